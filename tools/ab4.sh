python __graft_entry__.py >/dev/null
ARLO_LIB_VARIANT=direct timeout 300 python -m pytest tests/test_gpu_ops.py -x -q -k gemm > gpurun_out/gpu_tests_direct.log 2>&1; echo RC=$? >> gpurun_out/gpu_tests_direct.log
for v in default direct gtanh; do
  for a in "32768 4096 1024 -256 1" "32768 4096 1024 -256 0" "4096 3072 768 -256 1" "4096 3072 768 -256 0" "4096 768 3072 -192 2"; do
    if [ $v = default ]; then python tools/gemm_trace.py $a; else ARLO_LIB_VARIANT=$v python tools/gemm_trace.py $a; fi | grep -v "^tile" | sed "s/^/$v /"
  done
done > gpurun_out/ab4_trace.txt 2>&1
for rep in 1 2; do for v in default direct gtanh; do
  if [ $v = default ]; then python tools/ab_forward.py; else ARLO_LIB_VARIANT=$v python tools/ab_forward.py; fi
done; done > gpurun_out/ab4.txt 2>&1
