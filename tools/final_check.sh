mkdir -p gpurun_out/check
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/check/build.log 2>&1
timeout 900 python -m pytest tests -x -q -m gpu > gpurun_out/check/gpu_tests.log 2>&1; echo TESTS_RC=$? >> gpurun_out/check/gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/check/smoke.log 2>&1; echo SMOKE_RC=$? >> gpurun_out/check/smoke.log
timeout 900 python bench.py > gpurun_out/check/bench.json 2> gpurun_out/check/bench.err; echo BENCH_RC=$? >> gpurun_out/check/bench.err
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/check/bench_ref.json 2> gpurun_out/check/bench_ref.err
