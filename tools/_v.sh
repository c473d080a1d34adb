out=gpurun_out/v1; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1
timeout -s KILL 900 python -m pytest tests/test_gpu_fold.py tests/test_gpu_ops.py tests/test_gpu_runtime.py -q -x > $out/tests.log 2>&1; echo RC=$? >> $out/tests.log
timeout 900 python bench.py --extras-out $out/bench_extras.json > $out/bench.json 2> $out/bench.err; echo BENCH_RC=$? >> $out/bench.err
