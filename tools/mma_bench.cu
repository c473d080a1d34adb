// Microbenchmark: issue cost and completion time of back-to-back
// tcgen05.mma kind::f16 (M=128, N in {64,128,256}, K=16 per instruction) from
// smem operands, one CTA per SM.  Prints cycles per instruction for issue and
// for completion (commit -> mbarrier).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -I paper_conf_icpp_tanlyl024_b200/csrc \
//        -o tools/mma_bench tools/mma_bench.cu -lcuda
#include <cstdio>
#include <cstdint>
#include "ptx.cuh"

using namespace arlo;

__device__ __forceinline__ void mma_elect(uint32_t d_tmem, uint64_t a_desc, uint64_t b_desc, uint32_t idesc,
                                          uint32_t acc) {
  asm volatile(
      "{\n\t.reg .pred p, e;\n\t"
      "elect.sync _|e, 0xffffffff;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "@e tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(d_tmem),
      "l"(a_desc), "l"(b_desc), "r"(idesc), "r"(acc)
      : "memory");
}
__device__ __forceinline__ void commit_elect(uint64_t* bar) {
  asm volatile(
      "{\n\t.reg .pred e;\n\t"
      "elect.sync _|e, 0xffffffff;\n\t"
      "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n\t}" ::"r"(ptx::smem_u32(bar))
      : "memory");
}

// WARP: the whole warp 0 runs the issue loop (converged), one elected lane issues
// each MMA in the same asm block; else lane 0 alone runs it (divergent warp).
template <int N, bool WARP>
__global__ void __launch_bounds__(128, 1) k(int n_mma, long long* out) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  __shared__ uint64_t bar;
  __shared__ uint32_t slot;
  for (int i = threadIdx.x; i < (128 * 64 + N * 64) * 2 / 16; i += blockDim.x)
    reinterpret_cast<uint4*>(smem)[i] = make_uint4(0, 0, 0, 0);
  if (threadIdx.x == 0) {
    ptx::mbar_init(&bar, 1);
    ptx::fence_mbar_init();
  }
  if (threadIdx.x < 32) ptx::tmem_alloc(&slot, 256);
  ptx::fence_proxy_async_smem();
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = slot;
  if (WARP ? threadIdx.x < 32 : threadIdx.x == 0) {
    const uint32_t a = ptx::smem_u32(smem), b = ptx::smem_u32(smem + 128 * 128);
    constexpr uint32_t idesc = ptx::idesc_bf16_f32(128, N);
    // 8 bursts of n_mma MMAs, each committed and waited for; report the last burst
    long long t0 = 0, t1 = 0, t2 = 0;
    for (int rep = 0; rep < 8; ++rep) {
      t0 = clock64();
      for (int i = 0; i < n_mma; ++i) {
        if (WARP)
          mma_elect(tmem, ptx::desc_k_sw128(a + (i & 3) * 32), ptx::desc_k_sw128(b + (i & 3) * 32), idesc, i > 0);
        else
          ptx::mma_bf16_ss(tmem, ptx::desc_k_sw128(a + (i & 3) * 32), ptx::desc_k_sw128(b + (i & 3) * 32), idesc,
                           i > 0);
      }
      t1 = clock64();
      if (WARP)
        commit_elect(&bar);
      else
        ptx::mma_commit(&bar);
      ptx::mbar_wait(&bar, rep & 1);
      t2 = clock64();
      if (blockIdx.x == 0 && rep == 0 && threadIdx.x == 0) out[2] = t2 - t0;
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) {
      out[0] = t1 - t0;
      out[1] = t2 - t0;
    }
  }
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  if (threadIdx.x < 32) ptx::tmem_dealloc(tmem, 256);
}

template <int N, bool WARP = false>
void run(long long* d, int n_mma, int grid) {
  const int smem = (128 * 64 + N * 64) * 2 + 2048;
  cudaFuncSetAttribute(k<N, WARP>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  k<N, WARP><<<grid, 128, smem>>>(n_mma, d);
  printf("%s ", WARP ? "warp  " : "lane0 ");
  long long h[3];
  cudaMemcpy(h, d, 24, cudaMemcpyDeviceToHost);
  printf("N=%3d n_mma=%4d: 8th burst issue %.1f cyc/mma, complete %.1f cyc/mma (burst %lld cyc; 1st burst %lld; ideal %d/mma)"
         " err=%s\n", N, n_mma, (double)h[0] / n_mma, (double)h[1] / n_mma, h[1], h[2], 2 * 128 * N * 16 / 8192,
         cudaGetErrorString(cudaGetLastError()));
}

// NW warps issue concurrently, each its own bursts of n_mma (M=128, N=64) into
// its own TMEM columns, committed to its own mbarrier; cycles per burst per warp.
template <int NW>
__global__ void __launch_bounds__(128, 1) kmulti(int n_mma, long long* out) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  __shared__ uint64_t bar[4];
  __shared__ uint32_t slot;
  for (int i = threadIdx.x; i < (128 * 64 + 64 * 64) * 2 / 16; i += blockDim.x)
    reinterpret_cast<uint4*>(smem)[i] = make_uint4(0, 0, 0, 0);
  if (threadIdx.x == 0) {
    for (int i = 0; i < 4; ++i) ptx::mbar_init(&bar[i], 1);
    ptx::fence_mbar_init();
  }
  if (threadIdx.x < 32) ptx::tmem_alloc(&slot, 256);
  ptx::fence_proxy_async_smem();
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = slot;
  const int w = threadIdx.x >> 5;
  if (w < NW) {
    const uint32_t a = ptx::smem_u32(smem), b = ptx::smem_u32(smem + 128 * 128);
    constexpr uint32_t idesc = ptx::idesc_bf16_f32(128, 64);
    long long t0 = clock64();
    for (int rep = 0; rep < 32; ++rep) {
      for (int i = 0; i < n_mma; ++i)
        mma_elect(tmem + w * 64, ptx::desc_k_sw128(a + (i & 3) * 32), ptx::desc_k_sw128(b + (i & 3) * 32), idesc, i > 0);
      commit_elect(&bar[w]);
      ptx::mbar_wait(&bar[w], rep & 1);
    }
    long long t1 = clock64();
    if (blockIdx.x == 0 && (threadIdx.x & 31) == 0) out[w] = (t1 - t0) / 32;
  }
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  if (threadIdx.x < 32) ptx::tmem_dealloc(tmem, 256);
}

template <int NW>
void run_multi(long long* d, int n_mma) {
  const int smem = (128 * 64 + 64 * 64) * 2 + 2048;
  cudaFuncSetAttribute(kmulti<NW>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  kmulti<NW><<<148, 128, smem>>>(n_mma, d);
  long long h[4] = {0, 0, 0, 0};
  cudaMemcpy(h, d, 8 * NW, cudaMemcpyDeviceToHost);
  printf("%d issuing warps, bursts of %d (N=64): cycles per burst per warp:", NW, n_mma);
  for (int i = 0; i < NW; ++i) printf(" %lld", h[i]);
  printf("  err=%s\n", cudaGetErrorString(cudaGetLastError()));
}

// Operand-source variants at M=128, N=64, K=16, long streams from one converged
// warp: mode 0 SS (A, B K-major), 1 SS with B MN-major, 2 TS (A from TMEM) B
// K-major, 3 TS B MN-major.  Cycles per MMA.
__device__ __forceinline__ void mma_ts_elect(uint32_t d_tmem, uint32_t a_tmem, uint64_t b_desc, uint32_t idesc,
                                             uint32_t acc) {
  asm volatile(
      "{\n\t.reg .pred p, e;\n\t"
      "elect.sync _|e, 0xffffffff;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n\t}" ::"r"(d_tmem),
      "r"(a_tmem), "l"(b_desc), "r"(idesc), "r"(acc)
      : "memory");
}
template <int MODE>
__global__ void __launch_bounds__(128, 1) kmode(int n_mma, long long* out) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  __shared__ uint64_t bar;
  __shared__ uint32_t slot;
  for (int i = threadIdx.x; i < 65536 / 16; i += blockDim.x) reinterpret_cast<uint4*>(smem)[i] = make_uint4(0, 0, 0, 0);
  if (threadIdx.x == 0) {
    ptx::mbar_init(&bar, 1);
    ptx::fence_mbar_init();
  }
  if (threadIdx.x < 32) ptx::tmem_alloc(&slot, 256);
  ptx::fence_proxy_async_smem();
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = slot;
  if (threadIdx.x < 32) {
    const uint32_t a = ptx::smem_u32(smem), b = ptx::smem_u32(smem + 32768);
    constexpr bool bmn = MODE == 1 || MODE == 3;
    constexpr uint32_t idesc = bmn ? ptx::idesc_bf16_f32_bmn(128, 64) : ptx::idesc_bf16_f32(128, 64);
    long long t0 = clock64();
    for (int i = 0; i < n_mma; ++i) {
      const uint64_t bd = bmn ? ptx::desc_mn_sw128(b + (i & 3) * 2048, 0) : ptx::desc_k_sw128(b + (i & 3) * 32);
      if (MODE < 2)
        mma_elect(tmem, ptx::desc_k_sw128(a + (i & 3) * 32), bd, idesc, i > 0);
      else
        mma_ts_elect(tmem, tmem + 128 + (i & 3) * 8, bd, idesc, i > 0);
    }
    commit_elect(&bar);
    ptx::mbar_wait(&bar, 0);
    long long t1 = clock64();
    if (blockIdx.x == 0 && threadIdx.x == 0) out[0] = t1 - t0;
  }
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  if (threadIdx.x < 32) ptx::tmem_dealloc(tmem, 256);
}
template <int MODE>
void run_mode(long long* d, int n) {
  const int smem = 65536 + 2048;
  cudaFuncSetAttribute(kmode<MODE>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  kmode<MODE><<<148, 128, smem>>>(n, d);
  long long h = 0;
  cudaMemcpy(&h, d, 8, cudaMemcpyDeviceToHost);
  const char* names[] = {"SS  B K-major", "SS  B MN-major", "TS  B K-major", "TS  B MN-major"};
  printf("M=128 N=64 %s: %d MMAs %.1f cyc/mma  err=%s\n", names[MODE], n, (double)h / n,
         cudaGetErrorString(cudaGetLastError()));
}

int main() {
  long long* d;
  cudaMalloc(&d, 32);
  for (int n : {1, 4, 8, 16, 256}) {
    run<64>(d, n, 148);
    run<64, true>(d, n, 148);
    run<128>(d, n, 148);
    run<128, true>(d, n, 148);
  }
  for (int n : {4, 256}) {
    run_mode<0>(d, n);
    run_mode<1>(d, n);
    run_mode<2>(d, n);
    run_mode<3>(d, n);
  }
  for (int n : {4, 8}) {
    run_multi<1>(d, n);
    run_multi<2>(d, n);
    run_multi<4>(d, n);
  }
  return 0;
}
