mkdir -p gpurun_out/ab20
python __graft_entry__.py > gpurun_out/ab20/build.log 2>&1
python tools/op_bench.py 2>&1 | grep head > gpurun_out/ab20/ops.txt
ARLO_NO_PDL=1 python tools/op_bench.py 2>&1 | grep head | sed "s/^/nopdl /" >> gpurun_out/ab20/ops.txt
timeout 300 ncu --set full --clock-control none --import-source on -k regex:pooler -s 2 -c 1 \
   -o gpurun_out/ab20/pooler python tools/profile_ops.py head 32 128 > gpurun_out/ab20/ncu_pooler.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:classifier -s 2 -c 1 \
   -o gpurun_out/ab20/classifier python tools/profile_ops.py head 32 128 > gpurun_out/ab20/ncu_cls.log 2>&1
B=32 L=256 python tools/attn_trace.py 32 256 12 256 > gpurun_out/ab20/attn_trace_256.txt 2>&1
python tools/attn_trace.py 32 128 12 128 > gpurun_out/ab20/attn_trace_128.txt 2>&1
python tools/attn_trace.py 64 512 16 512 > gpurun_out/ab20/attn_trace_512.txt 2>&1
