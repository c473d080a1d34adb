# One gpurun call: build, GPU tests, smoke, default bench (+ reference arm).  Results in gpurun_out/$1/.
out=gpurun_out/${1:-check}
mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
timeout 1500 python -m pytest tests -x -q -m gpu ${PYTEST_ARGS} > $out/gpu_tests.log 2>&1; echo TESTS_RC=$? >> $out/gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $out/smoke.log 2>&1; echo SMOKE_RC=$? >> $out/smoke.log
timeout 900 python bench.py --extras-out $out/bench_extras.json > $out/bench.json 2> $out/bench.err; echo BENCH_RC=$? >> $out/bench.err
timeout 600 python bench.py --impl reference > $out/bench_ref.json 2> $out/bench_ref.err
