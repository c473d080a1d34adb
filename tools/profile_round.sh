# Round profile artifacts (one gpurun call; results in gpurun_out/${1:-prof}/):
#   bench JSON (+ extras), ncu launch list of the bench's timed steps (cold-cache, serialised: compare
#   SHARES, not absolutes), ncu --set full of the four GEMMs of the L=128 b=32 graph in the tile codes
#   the graph uses (from the bench extras) and of attention / LayerNorm, per-kernel metric summaries.
out=gpurun_out/${1:-prof}
mkdir -p $out
python __graft_entry__.py > /dev/null
timeout 900 python bench.py --extras-out $out/bench_extras.json > $out/bench.json 2> $out/bench.err
ARLO_PROFILE_TIMED=1 timeout 900 ncu --profile-from-start off --metrics gpu__time_duration.sum --clock-control none -c 3000 --csv \
    --log-file $out/launches.csv python bench.py --steps 2 --warmup 1 --no-extras --no-cpu-baseline \
    > $out/bench_under_ncu.log 2>&1
python tools/forward_breakdown.py --summarize $out/launches.csv > $out/launches_summary.txt 2>&1
full() {  # name, kernel regex, command...
  name=$1; shift; k=$1; shift
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:$k -s 2 -c 1 \
      -o $out/$name "$@" > $out/$name.log 2>&1
}
codes=$(python -c "import json; d=json.load(open('$out/bench_extras.json'))['gemm_tiles']['128']['32']; print(*d)")
set -- $codes
full qkv_L128b32 gemm python tools/profile_ops.py gemm 4096 2304 768 0 $1
full out_L128b32 gemm python tools/profile_ops.py gemm 4096 768 768 2 $2
full ffn1_L128b32 gemm python tools/profile_ops.py gemm 4096 3072 768 1 $3
full ffn2_L128b32 gemm python tools/profile_ops.py gemm 4096 768 3072 2 $4
full ffn1_large gemm_tc_pair python tools/profile_ops.py gemm 32768 4096 1024 1
full attn_l64 attn_tc python tools/profile_ops.py attn 32 64 12 64
full attn_l128 attn_tc python tools/profile_ops.py attn 32 128 12 128
full attn_l512 attn_tc python tools/profile_ops.py attn 64 512 16 512
full layernorm layernorm python tools/profile_ops.py ln 4096 768
python tools/ncu_summary.py $out/*.ncu-rep > $out/ncu_summary.txt 2>&1
# per-launch DRAM traffic of the four L=128 b=32 GEMMs, keyed as bench.py's roofline looks it up
cp profiles/traffic.json $out/traffic.json 2>/dev/null
python tools/ncu_summary.py --traffic $out/traffic.json qkv_L128_b32_tile$1_dram_bytes=$out/qkv_L128b32.ncu-rep \
    out_proj_L128_b32_tile$2_dram_bytes=$out/out_L128b32.ncu-rep ffn1_L128_b32_tile$3_dram_bytes=$out/ffn1_L128b32.ncu-rep \
    ffn2_L128_b32_tile$4_dram_bytes=$out/ffn2_L128b32.ncu-rep > $out/traffic.log 2>&1
ncu -i $out/ffn1_L128b32.ncu-rep --page source --csv > $out/ffn1_source.csv 2>/dev/null
# the build-time tile choice of a shape can differ between runs when two codes time within noise:
# capture the traffic of every candidate tile of the four GEMMs (metrics only, one launch each)
for g in "qkv 2304 768 0" "out_proj 768 768 2" "ffn1 3072 768 1" "ffn2 768 3072 2"; do
  set -- $g
  for code in -256 -192 -128 256 192 128 96; do
    [ $(( $2 % (code < 0 ? -code : code) )) -eq 0 ] || continue
    timeout 300 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none \
        -k regex:gemm -s 2 -c 1 -o $out/t_$1_$code python tools/profile_ops.py gemm 4096 $2 $3 $4 $code > /dev/null 2>&1 &&
      python tools/ncu_summary.py --traffic $out/traffic.json $1_L128_b32_tile${code}_dram_bytes=$out/t_$1_$code.ncu-rep \
        >> $out/traffic.log 2>&1
  done
done
# keep the pulled-back directory small (gpurun merges <= 64 MiB): the reports stay on the box
mkdir -p /tmp/ncu_reps && mv $out/*.ncu-rep /tmp/ncu_reps/ 2>/dev/null
