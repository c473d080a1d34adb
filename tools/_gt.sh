out=gpurun_out/gt4; mkdir -p $out
cd tools && timeout 600 python fold_bench.py > ../$out/fb.txt 2>&1; cd ..
for cfg in "4096 2304 768 -256 3" "4096 768 768 192 5"; do echo "== $cfg" >> $out/t.txt; timeout 120 python tools/gemm_trace.py $cfg >> $out/t.txt 2>&1; done
