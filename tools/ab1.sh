python __graft_entry__.py >/dev/null
timeout 600 python -m pytest tests -x -q -m gpu > gpurun_out/gpu_tests.log 2>&1; echo TESTS_RC=$? >> gpurun_out/gpu_tests.log
ARLO_LIB_VARIANT=e16 timeout 300 python -m pytest tests/test_gpu_ops.py -x -q -k gemm > gpurun_out/gpu_tests_e16.log 2>&1; echo RC=$? >> gpurun_out/gpu_tests_e16.log
for rep in 1 2; do for v in default e16 stg4 e16s4; do
  if [ $v = default ]; then python tools/ab_forward.py; else ARLO_LIB_VARIANT=$v python tools/ab_forward.py; fi
done; done > gpurun_out/ab1.txt 2>&1
ARLO_NO_SKINNY=1 python tools/ab_forward.py quick > gpurun_out/ab1_env.txt 2>&1
ARLO_NO_CLS_PRUNE=1 python tools/ab_forward.py quick >> gpurun_out/ab1_env.txt 2>&1
for v in default e16 e16s4; do for a in "32768 4096 1024 -256 1" "4096 3072 768 -256 1" "4096 3072 768 -256 0"; do
  if [ $v = default ]; then python tools/gemm_trace.py $a; else ARLO_LIB_VARIANT=$v python tools/gemm_trace.py $a; fi | grep -v "^tile"
done; done > gpurun_out/ab1_trace.txt 2>&1
python tools/gemm_sweep.py --set small --epi 0 0 1016 1032 1064 64 > gpurun_out/sweep_small.txt 2>&1
