mkdir -p gpurun_out/ab27
python __graft_entry__.py > gpurun_out/ab27/build.log 2>&1
timeout 1500 python tools/cluster_replay.py realloc 8000 16 0.97 > gpurun_out/ab27/realloc_G16.json 2> gpurun_out/ab27/realloc.err
