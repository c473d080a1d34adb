mkdir -p gpurun_out/ab26
python __graft_entry__.py > gpurun_out/ab26/build.log 2>&1
timeout 1500 python tools/cluster_replay.py realloc 6000 > gpurun_out/ab26/realloc.json 2> gpurun_out/ab26/realloc.err
