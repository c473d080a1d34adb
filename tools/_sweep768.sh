out=gpurun_out/sweep768; mkdir -p $out
for e in 2 0 1; do
  timeout 600 python tools/gemm_sweep.py --epi $e --set base 0 256 192 128 96 -256 -192 -128 > $out/base_epi$e.txt 2>&1
done
