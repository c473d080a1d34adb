python __graft_entry__.py >/dev/null
timeout 600 python -m pytest tests -x -q -m gpu > gpurun_out/gpu_tests.log 2>&1; echo TESTS_RC=$? >> gpurun_out/gpu_tests.log
python tools/gemm_sweep.py --set small 0 1016 1032 1064 64 128 -128 > gpurun_out/ab9_small.txt 2>&1
python tools/gemm_sweep.py --set base --epi 0 0 -256 -192 256 192 128 > gpurun_out/ab9_base.txt 2>&1
python tools/gemm_sweep.py --set large --epi 0 0 -256 256 > gpurun_out/ab9_large.txt 2>&1
for rep in 1 2; do for v in default prewmma; do
  if [ $v = default ]; then python tools/ab_forward.py; else ARLO_LIB_VARIANT=$v python tools/ab_forward.py; fi
done; done > gpurun_out/ab9_fwd.txt 2>&1
