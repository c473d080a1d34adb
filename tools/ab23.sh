# attention chunk 0 from one TMEM read (A/B vs ARLO_ATTN_C0_TWOPASS); LayerNorm rows per CTA 8 / 16 / 32
mkdir -p gpurun_out/ab23
python __graft_entry__.py > gpurun_out/ab23/build.log 2>&1
python -m paper_conf_icpp_tanlyl024_b200.build --variant c0two -DARLO_ATTN_C0_TWOPASS >> gpurun_out/ab23/build.log 2>&1
python -m paper_conf_icpp_tanlyl024_b200.build --variant ln16 -DARLO_LN_ROWS=16 >> gpurun_out/ab23/build.log 2>&1
python -m paper_conf_icpp_tanlyl024_b200.build --variant ln32 -DARLO_LN_ROWS=32 >> gpurun_out/ab23/build.log 2>&1
python -m paper_conf_icpp_tanlyl024_b200.build --variant ln4 -DARLO_LN_ROWS=4 >> gpurun_out/ab23/build.log 2>&1
timeout 900 python -m pytest tests -q -m gpu > gpurun_out/ab23/gpu_tests.log 2>&1; echo TESTS_RC=$? >> gpurun_out/ab23/gpu_tests.log
for v in default c0two ln16 ln32 ln4; do
  if [ $v = default ]; then python tools/op_bench.py; else ARLO_LIB_VARIANT=$v python tools/op_bench.py; fi | sed "s/^/$v /"
done > gpurun_out/ab23/ops.txt 2>&1
for rep in 1 2; do for v in default c0two ln16 ln32; do
  if [ $v = default ]; then python tools/ab_forward.py; else ARLO_LIB_VARIANT=$v python tools/ab_forward.py; fi
done; done > gpurun_out/ab23/fwd.txt 2>&1
