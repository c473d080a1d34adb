# Round profile artifacts (run under gpurun; results land in gpurun_out/prof/):
#   bench JSON, ncu launch list of the bench step (cold-cache, serialised: shares not absolutes),
#   ncu --set full of the top kernels, per-kernel metric summaries.
set -x
mkdir -p gpurun_out/prof
python __graft_entry__.py > /dev/null
timeout 900 python bench.py > gpurun_out/prof/bench.json 2> gpurun_out/prof/bench.err
ARLO_PROFILE_TIMED=1 timeout 900 ncu --profile-from-start off --metrics gpu__time_duration.sum --clock-control none -c 3000 --csv \
    --log-file gpurun_out/prof/launches.csv python bench.py --steps 2 --warmup 1 --no-extras --no-cpu-baseline \
    > gpurun_out/prof/bench_under_ncu.log 2>&1
python tools/forward_breakdown.py --summarize gpurun_out/prof/launches.csv > gpurun_out/prof/launches_summary.txt 2>&1
full() {  # name, kernel regex, command...
  name=$1; shift; k=$1; shift
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:$k -s 2 -c 1 \
      -o gpurun_out/prof/$name "$@" > gpurun_out/prof/$name.log 2>&1
}
full ffn1_gemm gemm_tc_pair python tools/profile_ops.py gemm 4096 3072 768 1
full ffn1_gemm_large gemm_tc_pair python tools/profile_ops.py gemm 32768 4096 1024 1
full skinny_gemm gemm_skinny python tools/profile_ops.py gemm 64 768 3072 0
full attn_l128 attn_tc python tools/profile_ops.py attn 32 128 12 128
full attn_l512 attn_tc python tools/profile_ops.py attn 64 512 16 512
full layernorm layernorm python tools/profile_ops.py ln 4096 768
full embed embed_ln python tools/profile_ops.py embed 32 128
full pooler pooler python tools/profile_ops.py head 32 128
