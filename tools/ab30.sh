mkdir -p gpurun_out/ab30
python __graft_entry__.py > gpurun_out/ab30/build.log 2>&1
timeout 1500 python tools/cluster_replay.py base 6000 > gpurun_out/ab30/cluster_base.json 2> gpurun_out/ab30/cluster_base.err
timeout 1500 python tools/cluster_replay.py roberta 6000 > gpurun_out/ab30/cluster_roberta.json 2> gpurun_out/ab30/cluster_roberta.err
timeout 1500 python tools/cluster_replay.py ablation 6000 > gpurun_out/ab30/ablation.json 2> gpurun_out/ab30/ablation.err
