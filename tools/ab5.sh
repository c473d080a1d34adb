python __graft_entry__.py >/dev/null
timeout 600 python -m pytest tests -x -q -m gpu > gpurun_out/gpu_tests.log 2>&1; echo TESTS_RC=$? >> gpurun_out/gpu_tests.log
python tools/attn_trace.py 64 512 16 512 > gpurun_out/attn_trace.txt 2>&1
for v in default attn2 default attn2; do
  if [ $v = default ]; then python tools/op_bench.py; else ARLO_LIB_VARIANT=$v python tools/op_bench.py; fi | sed "s/^/$v /"
done > gpurun_out/ab5.txt 2>&1
for v in default attn2; do
  if [ $v = default ]; then python tools/ab_forward.py; else ARLO_LIB_VARIANT=$v python tools/ab_forward.py; fi
done > gpurun_out/ab5_fwd.txt 2>&1
