# BN=96 single-CTA tiles (sweep vs chooser), head op timing, tests, forwards, bench
mkdir -p gpurun_out/ab19
python __graft_entry__.py > gpurun_out/ab19/build.log 2>&1
timeout 900 python -m pytest tests -q -m gpu > gpurun_out/ab19/gpu_tests.log 2>&1; echo TESTS_RC=$? >> gpurun_out/ab19/gpu_tests.log
for e in 0 1 2; do
  python tools/gemm_sweep.py --set base --epi $e --no-cublas 0 96 192 128 -256 -192 2>&1 | sed "s/^/epi$e /"
  python tools/gemm_sweep.py --set mid --epi $e --no-cublas 0 96 192 128 -256 -192 2>&1 | sed "s/^/epi$e /"
done > gpurun_out/ab19/sweep.txt 2>&1
python tools/op_bench.py > gpurun_out/ab19/ops.txt 2>&1
for rep in 1 2; do python tools/ab_forward.py; done > gpurun_out/ab19/fwd.txt 2>&1
timeout 900 python bench.py > gpurun_out/ab19/bench.json 2> gpurun_out/ab19/bench.err
