# pair GEMM: last tile split into two N-halves when a pair has 2..4 tiles (A/B vs ARLO_NO_SPLIT_LAST)
mkdir -p gpurun_out/ab24
python __graft_entry__.py > gpurun_out/ab24/build.log 2>&1
python -m paper_conf_icpp_tanlyl024_b200.build --variant nosplit -DARLO_NO_SPLIT_LAST >> gpurun_out/ab24/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_ops.py -q -m gpu -k gemm > gpurun_out/ab24/gemm_tests.log 2>&1; echo RC=$? >> gpurun_out/ab24/gemm_tests.log
for v in default nosplit; do
  if [ $v = default ]; then unset ARLO_LIB_VARIANT; else export ARLO_LIB_VARIANT=$v; fi
  for e in 0 1 2; do
    python tools/gemm_sweep.py --set base --epi $e --no-cublas 0 2>&1 | sed "s/^/$v epi$e /"
    python tools/gemm_sweep.py --set mid --epi $e --no-cublas 0 2>&1 | sed "s/^/$v epi$e /"
  done
done > gpurun_out/ab24/sweep.txt 2>&1
unset ARLO_LIB_VARIANT
for rep in 1 2; do for v in default nosplit; do
  if [ $v = default ]; then python tools/ab_forward.py; else ARLO_LIB_VARIANT=$v python tools/ab_forward.py; fi
done; done > gpurun_out/ab24/fwd.txt 2>&1
timeout 900 python -m pytest tests -q -m gpu > gpurun_out/ab24/gpu_tests.log 2>&1; echo TESTS_RC=$? >> gpurun_out/ab24/gpu_tests.log
