# pooler conflict-free staging; tests; ops; forwards; then the round profile (bench + ncu launch list + full captures)
mkdir -p gpurun_out/ab21
python __graft_entry__.py > gpurun_out/ab21/build.log 2>&1
timeout 900 python -m pytest tests -q -m gpu > gpurun_out/ab21/gpu_tests.log 2>&1; echo TESTS_RC=$? >> gpurun_out/ab21/gpu_tests.log
python tools/op_bench.py > gpurun_out/ab21/ops.txt 2>&1
for rep in 1 2; do python tools/ab_forward.py; done > gpurun_out/ab21/fwd.txt 2>&1
bash tools/profile_round.sh > gpurun_out/ab21/profile_round.log 2>&1
python tools/ncu_summary.py gpurun_out/prof/*.ncu-rep > gpurun_out/prof/ncu_summary.txt 2>&1
