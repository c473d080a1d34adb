python __graft_entry__.py >/dev/null
for v in default same; do
  for a in "32768 4096 1024 -256 0" "4096 768 3072 -192 0" "16384 3072 768 -256 0"; do
    if [ $v = default ]; then python tools/gemm_trace.py $a; else ARLO_LIB_VARIANT=$v python tools/gemm_trace.py $a; fi | grep -v "^tile" | sed "s/^/$v /"
  done
done > gpurun_out/ab7_trace.txt 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:gemm_skinny -s 2 -c 1 -o gpurun_out/skinny python tools/profile_ops.py gemm 64 768 3072 0 > gpurun_out/skinny_ncu.log 2>&1
