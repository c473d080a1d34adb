# GELU epilogue with 12 warps at M <= 16384 (A/B vs 8 everywhere), pooler register/occupancy fix
mkdir -p gpurun_out/ab18
python __graft_entry__.py > gpurun_out/ab18/build.log 2>&1
python -m paper_conf_icpp_tanlyl024_b200.build --variant ew8 -DARLO_GELU_EW12_MAX_M=0 >> gpurun_out/ab18/build.log 2>&1
timeout 900 python -m pytest tests -q -m gpu > gpurun_out/ab18/gpu_tests.log 2>&1; echo TESTS_RC=$? >> gpurun_out/ab18/gpu_tests.log
for v in default ew8; do
  if [ $v = default ]; then unset ARLO_LIB_VARIANT; else export ARLO_LIB_VARIANT=$v; fi
  python tools/gemm_sweep.py --set base --epi 1 --no-cublas 0 2>&1 | sed "s/^/$v /"
  python tools/gemm_sweep.py --set large --epi 1 --no-cublas 0 2>&1 | sed "s/^/$v /"
  python tools/gemm_sweep.py --set mid --epi 1 --no-cublas 0 2>&1 | sed "s/^/$v /"
done > gpurun_out/ab18/sweep.txt 2>&1
unset ARLO_LIB_VARIANT
for rep in 1 2; do for v in default ew8; do
  if [ $v = default ]; then python tools/ab_forward.py; else ARLO_LIB_VARIANT=$v python tools/ab_forward.py; fi
done; done > gpurun_out/ab18/fwd.txt 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum,launch__occupancy_limit_registers,launch__occupancy_limit_shared_mem --clock-control none -k regex:pooler -s 2 -c 1 python tools/profile_ops.py head 32 1 > gpurun_out/ab18/ncu_pooler.txt 2>&1
