# Round-1 re-entry check + GELU epilogue A/B (AS 7.1.26 default vs AS 7.1.28 one-MUFU vs tanh (speed bound only))
mkdir -p gpurun_out/ab10
python __graft_entry__.py > gpurun_out/ab10/build.log 2>&1
python -m paper_conf_icpp_tanlyl024_b200.build --variant as28 -DARLO_GELU_AS28 >> gpurun_out/ab10/build.log 2>&1
python -m paper_conf_icpp_tanlyl024_b200.build --variant tanhx -DARLO_GELU_EXPERIMENT >> gpurun_out/ab10/build.log 2>&1
timeout 900 python -m pytest tests -x -q -m gpu > gpurun_out/ab10/gpu_tests.log 2>&1; echo TESTS_RC=$? >> gpurun_out/ab10/gpu_tests.log
for v in default as28 tanhx; do
  if [ $v = default ]; then unset ARLO_LIB_VARIANT; else export ARLO_LIB_VARIANT=$v; fi
  python tools/gemm_sweep.py --set base --epi 1 0 2>&1 | sed "s/^/$v /"
  python tools/gemm_sweep.py --set large --epi 1 0 2>&1 | sed "s/^/$v /"
done > gpurun_out/ab10/gelu_sweep.txt 2>&1
unset ARLO_LIB_VARIANT
for rep in 1 2; do for v in default as28 tanhx; do
  if [ $v = default ]; then python tools/ab_forward.py; else ARLO_LIB_VARIANT=$v python tools/ab_forward.py; fi
done; done > gpurun_out/ab10/fwd.txt 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:gemm_tc_pair -s 2 -c 1 \
   -o gpurun_out/ab10/ffn1_large python tools/profile_ops.py gemm 32768 4096 1024 1 > gpurun_out/ab10/ncu_ffn1.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/ab10/large512.csv \
   python tools/forward_breakdown.py 512 64 2 large > gpurun_out/ab10/large512.log 2>&1
python tools/forward_breakdown.py --summarize gpurun_out/ab10/large512.csv > gpurun_out/ab10/large512_summary.txt 2>&1
timeout 900 python bench.py > gpurun_out/ab10/bench.json 2> gpurun_out/ab10/bench.err
