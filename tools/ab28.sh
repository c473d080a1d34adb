# residual prefetch before the accumulator wait (A/B via git stash is not possible on the box: compare with ab19/ab24 numbers)
mkdir -p gpurun_out/ab28
python __graft_entry__.py > gpurun_out/ab28/build.log 2>&1
timeout 900 python -m pytest tests -q -m gpu > gpurun_out/ab28/gpu_tests.log 2>&1; echo TESTS_RC=$? >> gpurun_out/ab28/gpu_tests.log
python tools/gemm_sweep.py --set base --epi 2 --no-cublas 0 > gpurun_out/ab28/sweep.txt 2>&1
python tools/gemm_sweep.py --set mid --epi 2 --no-cublas 0 >> gpurun_out/ab28/sweep.txt 2>&1
for rep in 1 2; do python tools/ab_forward.py; done > gpurun_out/ab28/fwd.txt 2>&1
