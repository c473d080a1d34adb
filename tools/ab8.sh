python __graft_entry__.py >/dev/null
timeout 300 python -m pytest tests/test_gpu_ops.py -x -q -k gemm > gpurun_out/gpu_tests_gemm.log 2>&1; echo RC=$? >> gpurun_out/gpu_tests_gemm.log
ARLO_LIB_VARIANT=wmma timeout 300 python -m pytest tests/test_gpu_ops.py -x -q -k gemm > gpurun_out/gpu_tests_wmma.log 2>&1; echo RC=$? >> gpurun_out/gpu_tests_wmma.log
for v in default skold; do
  if [ $v = default ]; then python tools/gemm_sweep.py --set small --no-cublas 0 1016 1032; else ARLO_LIB_VARIANT=$v python tools/gemm_sweep.py --set small --no-cublas 0 1016 1032; fi | sed "s/^/$v /"
done > gpurun_out/ab8_small.txt 2>&1
for v in default wmma; do
  for a in "32768 4096 1024 -256 0" "4096 768 3072 -192 0" "4096 3072 768 -256 1"; do
    if [ $v = default ]; then python tools/gemm_trace.py $a; else ARLO_LIB_VARIANT=$v python tools/gemm_trace.py $a; fi | grep -v "^tile" | sed "s/^/$v /"
  done
done > gpurun_out/ab8_trace.txt 2>&1
