# end-of-session round-1 artifacts: tests, smoke, round profile (bench + ncu launch list + full captures)
mkdir -p gpurun_out/final
python __graft_entry__.py > gpurun_out/final/build.log 2>&1
timeout 900 python -m pytest tests -q -m gpu > gpurun_out/final/gpu_tests.log 2>&1; echo TESTS_RC=$? >> gpurun_out/final/gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/final/smoke.log 2>&1; echo SMOKE_RC=$? >> gpurun_out/final/smoke.log
rm -rf gpurun_out/prof
bash tools/profile_round.sh > gpurun_out/final/profile_round.log 2>&1
python tools/ncu_summary.py gpurun_out/prof/*.ncu-rep > gpurun_out/prof/ncu_summary.txt 2>&1
python tools/op_bench.py > gpurun_out/final/ops.txt 2>&1
