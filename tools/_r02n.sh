mkdir -p gpurun_out/r02n
for v in default ln16g ln8g ln4g; do
  if [ $v = default ]; then unset ARLO_LIB_VARIANT; else export ARLO_LIB_VARIANT=$v; fi
  echo "== $v" >> gpurun_out/r02n/fwd.txt
  python tools/ab_forward.py quick >> gpurun_out/r02n/fwd.txt 2>&1
done
