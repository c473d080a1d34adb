python __graft_entry__.py >/dev/null
python tools/attn_trace.py 64 512 16 512 > gpurun_out/attn_trace.txt 2>&1
python tools/attn_trace.py 32 128 12 128 >> gpurun_out/attn_trace.txt 2>&1
python tools/attn_trace.py 32 256 12 256 >> gpurun_out/attn_trace.txt 2>&1
python tools/ab_forward.py > gpurun_out/ab2.txt 2>&1
ARLO_FUSED_LN=1 python tools/ab_forward.py >> gpurun_out/ab2.txt 2>&1
