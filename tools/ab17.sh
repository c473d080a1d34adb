mkdir -p gpurun_out/ab17
python __graft_entry__.py > gpurun_out/ab17/build.log 2>&1
python tools/dbg_head.py > gpurun_out/ab17/dbg.txt 2>&1
timeout 900 python -m pytest tests -q -m gpu > gpurun_out/ab17/gpu_tests.log 2>&1; echo TESTS_RC=$? >> gpurun_out/ab17/gpu_tests.log
for rep in 1 2; do python tools/ab_forward.py; done > gpurun_out/ab17/fwd.txt 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:pooler -s 2 -c 1 \
   -o gpurun_out/ab17/pooler python tools/profile_ops.py head 32 1 > gpurun_out/ab17/ncu_pooler.log 2>&1
