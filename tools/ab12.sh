mkdir -p gpurun_out/ab12
python __graft_entry__.py > gpurun_out/ab12/build.log 2>&1
M="--metrics gpu__time_duration.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active,l1tex__m_xbar2l1tex_read_bytes.sum,lts__t_sectors.sum.pct_of_peak_sustained_elapsed,lts__t_bytes.sum,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_requests_srcunit_tex_op_read.sum,dram__bytes_read.sum,launch__cluster_dim_x,launch__cluster_dim_y,launch__grid_size,launch__block_size,sm__cycles_elapsed.avg.per_second"
for s in "32768 4096 1024" "4096 3072 768" "8192 8192 8192"; do
  timeout 300 ncu $M --clock-control none -s 2 -c 1 python tools/cublas_probe.py $s > gpurun_out/ab12/cublas_$(echo $s | tr ' ' _).txt 2>&1
  timeout 300 ncu $M --clock-control none -k regex:gemm_tc -s 2 -c 1 python tools/profile_ops.py gemm $s 0 > gpurun_out/ab12/ours_$(echo $s | tr ' ' _).txt 2>&1
done
python - > gpurun_out/ab12/occ.txt 2>&1 <<'PY'
import torch
p = torch.cuda.get_device_properties(0)
print(p)
PY
