mkdir -p gpurun_out/b1
timeout 1200 python tools/cluster_replay.py batch1 6000 > gpurun_out/b1/batch1.json 2> gpurun_out/b1/batch1.err
