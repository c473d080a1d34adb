// tma_bench.cu — cost of a burst of TMA / bulk requests from one CTA (the fused forward's
// activation loads), data L2-resident.
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lcuda -o tools/tma_bench tools/tma_bench.cu
//
// One thread issues N requests on one mbarrier and waits; time (clock64 -> ns at the measured
// SM clock) from the first issue to the barrier completing, and the issue time alone:
//   tile64    2-D tensor box {64 bf16, 64 rows} = 8 KB, 128B swizzle (an A k-block at T = 64)
//   tile128   2-D tensor box {64 bf16, 128 rows} = 16 KB (a weight k-block)
//   bulk512   1-D bulk copy of 512 B (a LayerNorm partial row)
//   bulk8k    1-D bulk copy of 8 KB
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>

__device__ __forceinline__ uint32_t su(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

template <int MODE>
__global__ void burst(const __grid_constant__ CUtensorMap tm64, const __grid_constant__ CUtensorMap tm128,
                      const char* src, int n, unsigned long long* out) {
  extern __shared__ __align__(1024) uint8_t smem[];
  __shared__ uint64_t bar;
  if (threadIdx.x != 0) return;
  for (int rep = 0; rep < 3; ++rep) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su(&bar)));
    asm volatile("fence.mbarrier_init.release.cluster;");
    const uint32_t bytes = MODE == 0 ? 8192 : MODE == 1 ? 16384 : MODE == 2 ? 512 : 8192;
    long long t0 = clock64();
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su(&bar)), "r"(bytes * n));
    for (int i = 0; i < n; ++i) {
      uint8_t* dst = smem + (size_t)i * 16384;
      if (MODE == 0)
        asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];"
                     ::"r"(su(dst)), "l"(&tm64), "r"(su(&bar)), "r"(0), "r"(i * 64) : "memory");
      else if (MODE == 1)
        asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];"
                     ::"r"(su(dst)), "l"(&tm128), "r"(su(&bar)), "r"(0), "r"(i * 128) : "memory");
      else
        asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                     ::"r"(su(dst)), "l"(src + (size_t)i * bytes), "r"(bytes), "r"(su(&bar)) : "memory");
    }
    long long t1 = clock64();
    asm volatile(
        "{\n\t.reg .pred p;\n\tW: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], 0;\n\t@!p bra W;\n\t}" ::"r"(su(&bar)));
    long long t2 = clock64();
    if (rep == 2) {
      out[0] = t1 - t0;
      out[1] = t2 - t0;
    }
  }
}

typedef CUresult (*Enc)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*,
                        const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                        CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

int main() {
  char* buf;
  cudaMalloc(&buf, 64 << 20);
  cudaMemset(buf, 1, 64 << 20);
  unsigned long long* out;
  cudaMalloc(&out, 64);
  void* fn = nullptr;
  cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q);
  Enc enc = (Enc)fn;
  CUtensorMap tm64, tm128;
  cuuint64_t dims[2] = {64, 1 << 14}, strides[1] = {128};
  cuuint32_t box64[2] = {64, 64}, box128[2] = {64, 128}, es[2] = {1, 1};
  enc(&tm64, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, buf, dims, strides, box64, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
      CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  enc(&tm128, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, buf, dims, strides, box128, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
      CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  int clk = 0;
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  const double ghz = clk / 1e6;
  const char* names[] = {"tile64", "tile128", "bulk512", "bulk8k"};
  auto k0 = burst<0>, k1 = burst<1>, k2 = burst<2>, k3 = burst<3>;
  for (auto k : {k0, k1, k2, k3}) cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
  printf("SM clock attribute %.3f GHz (cycles -> ns at that clock)\n", ghz);
  for (int mode = 0; mode < 4; ++mode)
    for (int n : {1, 2, 4, 8, 12}) {
      auto k = mode == 0 ? k0 : mode == 1 ? k1 : mode == 2 ? k2 : k3;
      k<<<1, 32, 200 * 1024>>>(tm64, tm128, buf, n, out);
      unsigned long long h[2];
      cudaMemcpy(h, out, 16, cudaMemcpyDeviceToHost);
      printf("%-8s n=%2d  issue %6.0f ns  complete %6.0f ns\n", names[mode], n, h[0] / ghz, h[1] / ghz);
    }
  printf("%s\n", cudaGetErrorString(cudaDeviceSynchronize()));
  return 0;
}
