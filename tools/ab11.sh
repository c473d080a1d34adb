# GEMM epilogue: CTA-scope accumulator release (no MEMBAR.ALL.GPU) + paired-fp32 epilogue math, A/B
mkdir -p gpurun_out/ab11
python __graft_entry__.py > gpurun_out/ab11/build.log 2>&1
python -m paper_conf_icpp_tanlyl024_b200.build --variant old -DARLO_EPI_SCALAR -DARLO_ARRIVE_RELEASE_CLUSTER >> gpurun_out/ab11/build.log 2>&1
python -m paper_conf_icpp_tanlyl024_b200.build --variant scalar -DARLO_EPI_SCALAR >> gpurun_out/ab11/build.log 2>&1
timeout 900 python -m pytest tests -x -q -m gpu > gpurun_out/ab11/gpu_tests.log 2>&1; echo TESTS_RC=$? >> gpurun_out/ab11/gpu_tests.log
for v in default old scalar; do
  if [ $v = default ]; then unset ARLO_LIB_VARIANT; else export ARLO_LIB_VARIANT=$v; fi
  for e in 0 1 2; do
    python tools/gemm_sweep.py --set base --epi $e --no-cublas 0 2>&1 | sed "s/^/$v epi$e /"
    python tools/gemm_sweep.py --set large --epi $e --no-cublas 0 2>&1 | sed "s/^/$v epi$e /"
  done
done > gpurun_out/ab11/sweep.txt 2>&1
unset ARLO_LIB_VARIANT
for rep in 1 2; do for v in default old scalar; do
  if [ $v = default ]; then python tools/ab_forward.py; else ARLO_LIB_VARIANT=$v python tools/ab_forward.py; fi
done; done > gpurun_out/ab11/fwd.txt 2>&1
for v in default old; do
  for a in "4096 3072 768 -256 1" "4096 768 3072 192 2" "32768 4096 1024 -256 1"; do
    if [ $v = default ]; then python tools/gemm_trace.py $a; else ARLO_LIB_VARIANT=$v python tools/gemm_trace.py $a; fi | grep -v "^tile" | sed "s/^/$v /"
  done
done > gpurun_out/ab11/trace.txt 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:gemm_tc_pair -s 2 -c 1 \
   -o gpurun_out/ab11/ffn1_base python tools/profile_ops.py gemm 4096 3072 768 1 > gpurun_out/ab11/ncu_ffn1.log 2>&1
