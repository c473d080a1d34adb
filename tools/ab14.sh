# epilogue warp count A/B (8 default vs 12 / 16), attention setup before the PDL wait (tests), warm per-kernel breakdown
mkdir -p gpurun_out/ab14
python __graft_entry__.py > gpurun_out/ab14/build.log 2>&1
python -m paper_conf_icpp_tanlyl024_b200.build --variant e12 -DARLO_EPI_WARPS=12 >> gpurun_out/ab14/build.log 2>&1
python -m paper_conf_icpp_tanlyl024_b200.build --variant e16 -DARLO_EPI_WARPS=16 >> gpurun_out/ab14/build.log 2>&1
python -m paper_conf_icpp_tanlyl024_b200.build --variant e16s1 -DARLO_EPI_WARPS=16 -DARLO_STG_BUFS=1 >> gpurun_out/ab14/build.log 2>&1
timeout 900 python -m pytest tests -x -q -m gpu > gpurun_out/ab14/gpu_tests.log 2>&1; echo TESTS_RC=$? >> gpurun_out/ab14/gpu_tests.log
for v in default e12 e16 e16s1; do
  if [ $v = default ]; then unset ARLO_LIB_VARIANT; else export ARLO_LIB_VARIANT=$v; fi
  for e in 0 1 2; do
    python tools/gemm_sweep.py --set base --epi $e --no-cublas 0 2>&1 | sed "s/^/$v epi$e /"
    python tools/gemm_sweep.py --set large --epi $e --no-cublas 0 2>&1 | sed "s/^/$v epi$e /"
  done
done > gpurun_out/ab14/sweep.txt 2>&1
unset ARLO_LIB_VARIANT
for rep in 1 2; do for v in default e12 e16 e16s1; do
  if [ $v = default ]; then python tools/ab_forward.py; else ARLO_LIB_VARIANT=$v python tools/ab_forward.py; fi
done; done > gpurun_out/ab14/fwd.txt 2>&1
for c in "128 32" "64 32" "256 32"; do
  n=$(echo $c | tr ' ' _)
  timeout 600 ncu --metrics gpu__time_duration.sum --cache-control none --clock-control none --csv \
     --log-file gpurun_out/ab14/base_$n.csv python tools/forward_breakdown.py $c 2 > /dev/null 2>&1
  python tools/forward_breakdown.py --summarize gpurun_out/ab14/base_$n.csv > gpurun_out/ab14/base_${n}_summary.txt 2>&1
done
