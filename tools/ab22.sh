# attention L <= 128: P aliased over S, 128 TMEM columns, three CTAs per SM (A/B vs ARLO_ATTN_L128_NS2)
mkdir -p gpurun_out/ab22
python __graft_entry__.py > gpurun_out/ab22/build.log 2>&1
python -m paper_conf_icpp_tanlyl024_b200.build --variant ns2 -DARLO_ATTN_L128_NS2 >> gpurun_out/ab22/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_ops.py -q -m gpu -k attention > gpurun_out/ab22/attn_tests.log 2>&1; echo RC=$? >> gpurun_out/ab22/attn_tests.log
timeout 900 python -m pytest tests -q -m gpu > gpurun_out/ab22/gpu_tests.log 2>&1; echo TESTS_RC=$? >> gpurun_out/ab22/gpu_tests.log
for v in default ns2; do
  if [ $v = default ]; then python tools/op_bench.py; else ARLO_LIB_VARIANT=$v python tools/op_bench.py; fi | grep attention | sed "s/^/$v /"
done > gpurun_out/ab22/ops.txt 2>&1
for rep in 1 2; do for v in default ns2; do
  if [ $v = default ]; then python tools/ab_forward.py; else ARLO_LIB_VARIANT=$v python tools/ab_forward.py; fi
done; done > gpurun_out/ab22/fwd.txt 2>&1
python tools/attn_trace.py 32 128 12 128 > gpurun_out/ab22/attn_trace_128.txt 2>&1
