mkdir -p gpurun_out/ab16
python __graft_entry__.py > gpurun_out/ab16/build.log 2>&1
python tools/dbg_head.py > gpurun_out/ab16/dbg.txt 2>&1
ARLO_NO_PDL=1 python tools/dbg_head.py > gpurun_out/ab16/dbg_nopdl.txt 2>&1
timeout 300 compute-sanitizer --tool racecheck python tools/dbg_head.py > gpurun_out/ab16/racecheck.txt 2>&1
timeout 900 python -m pytest tests -q -m gpu > gpurun_out/ab16/gpu_tests.log 2>&1; echo TESTS_RC=$? >> gpurun_out/ab16/gpu_tests.log
