# GEMM tile rasterisation N-fastest vs M-fastest (A/B), + bench
mkdir -p gpurun_out/ab13
python __graft_entry__.py > gpurun_out/ab13/build.log 2>&1
python -m paper_conf_icpp_tanlyl024_b200.build --variant rasm -DARLO_RASTER_M >> gpurun_out/ab13/build.log 2>&1
timeout 900 python -m pytest tests -x -q -m gpu > gpurun_out/ab13/gpu_tests.log 2>&1; echo TESTS_RC=$? >> gpurun_out/ab13/gpu_tests.log
for v in default rasm; do
  if [ $v = default ]; then unset ARLO_LIB_VARIANT; else export ARLO_LIB_VARIANT=$v; fi
  for e in 0 1 2; do
    python tools/gemm_sweep.py --set base --epi $e --no-cublas 0 2>&1 | sed "s/^/$v epi$e /"
    python tools/gemm_sweep.py --set large --epi $e --no-cublas 0 2>&1 | sed "s/^/$v epi$e /"
  done
done > gpurun_out/ab13/sweep.txt 2>&1
unset ARLO_LIB_VARIANT
for rep in 1 2; do for v in default rasm; do
  if [ $v = default ]; then python tools/ab_forward.py; else ARLO_LIB_VARIANT=$v python tools/ab_forward.py; fi
done; done > gpurun_out/ab13/fwd.txt 2>&1
M="--metrics gpu__time_duration.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active,l1tex__m_xbar2l1tex_read_bytes.sum,lts__t_bytes.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__cycles_elapsed.avg.per_second"
timeout 300 ncu $M --clock-control none -k regex:gemm_tc -s 2 -c 1 python tools/profile_ops.py gemm 32768 4096 1024 1 > gpurun_out/ab13/ncu_ffn1_large.txt 2>&1
timeout 900 python bench.py > gpurun_out/ab13/bench.json 2> gpurun_out/ab13/bench.err
