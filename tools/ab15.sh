# LayerNorm two-rows-per-warp + paired fp32 (A/B vs ARLO_LN_V1), pooler/classifier rewrite, attention FFMA2
mkdir -p gpurun_out/ab15
python __graft_entry__.py > gpurun_out/ab15/build.log 2>&1
python -m paper_conf_icpp_tanlyl024_b200.build --variant lnv1 -DARLO_LN_V1 >> gpurun_out/ab15/build.log 2>&1
timeout 900 python -m pytest tests -x -q -m gpu > gpurun_out/ab15/gpu_tests.log 2>&1; echo TESTS_RC=$? >> gpurun_out/ab15/gpu_tests.log
for v in default lnv1; do
  if [ $v = default ]; then python tools/op_bench.py; else ARLO_LIB_VARIANT=$v python tools/op_bench.py; fi | sed "s/^/$v /"
done > gpurun_out/ab15/ops.txt 2>&1
for rep in 1 2; do for v in default lnv1; do
  if [ $v = default ]; then python tools/ab_forward.py; else ARLO_LIB_VARIANT=$v python tools/ab_forward.py; fi
done; done > gpurun_out/ab15/fwd.txt 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --cache-control none --clock-control none --csv \
   --log-file gpurun_out/ab15/base_128_32.csv python tools/forward_breakdown.py 128 32 2 > /dev/null 2>&1
python tools/forward_breakdown.py --summarize gpurun_out/ab15/base_128_32.csv > gpurun_out/ab15/base_128_32_summary.txt 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --cache-control none --clock-control none --csv \
   --log-file gpurun_out/ab15/base_128_1.csv python tools/forward_breakdown.py 128 1 2 > /dev/null 2>&1
python tools/forward_breakdown.py --summarize gpurun_out/ab15/base_128_1.csv > gpurun_out/ab15/base_128_1_summary.txt 2>&1
