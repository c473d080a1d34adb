python __graft_entry__.py >/dev/null
timeout 300 python -m pytest tests/test_gpu_ops.py -x -q -k attention > gpurun_out/gpu_tests_attn.log 2>&1; echo RC=$? >> gpurun_out/gpu_tests_attn.log
python tools/attn_trace.py 64 512 16 512 > gpurun_out/attn_trace.txt 2>&1
for v in default attnold default attnold; do
  if [ $v = default ]; then python tools/op_bench.py; else ARLO_LIB_VARIANT=$v python tools/op_bench.py; fi | grep attention | sed "s/^/$v /"
done > gpurun_out/ab3.txt 2>&1
