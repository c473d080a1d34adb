mkdir -p gpurun_out/ab25
python __graft_entry__.py > gpurun_out/ab25/build.log 2>&1
timeout 1200 python tools/cluster_replay.py realloc 6000 > gpurun_out/ab25/realloc.json 2> gpurun_out/ab25/realloc.err
timeout 900 python -m pytest tests -q -m gpu > gpurun_out/ab25/gpu_tests.log 2>&1; echo TESTS_RC=$? >> gpurun_out/ab25/gpu_tests.log
