// signal_bench.cu — inter-SM signalling latency on B200 (the fused forward's hop cost).
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/signal_bench tools/signal_bench.cu
//   tools/signal_bench
//
// Two CTAs (on different SMs) ping-pong a counter N times; per variant the round trip in ns
// (%globaltimer) / 2 = one signal -> observe hop:
//   relaxed    st.relaxed.gpu / ld.relaxed.gpu polling
//   release    red.release.gpu / ld.relaxed.gpu poll + fence.acq_rel.gpu
//   acquire    red.release.gpu / ld.acquire.gpu poll
//   fence+red  __threadfence + atomicAdd / ld.acquire.gpu poll  (cooperative-groups style)
//   +stores    'release' after each CTA writes `bytes` with 128 threads (16-byte stores), the
//              signal issued by thread 0 after __syncthreads: the drain of the stores is in the hop
//   rel+bg     'release' while warp 4 keeps bulk L2 prefetches of a 1 GB buffer in flight (the
//              fused kernel's producer streaming weights): does the release fence wait for them?
//   rlx+bg     'relaxed' with the same background traffic
#include <cstdio>
#include <cstdint>

__device__ __forceinline__ unsigned long long gt() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
__device__ __forceinline__ unsigned ld_relaxed(const unsigned* p) {
  unsigned v;
  asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ unsigned ld_acquire(const unsigned* p) {
  unsigned v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}

__device__ volatile int g_stop;
template <int MODE>
__global__ void pingpong(unsigned* flag, int iters, uint4* buf, int bytes, unsigned long long* out,
                         const char* big = nullptr) {
  if (threadIdx.x >= 128) {  // background: warp 4 lane 0 streams L2 prefetches until told to stop
    if ((MODE == 5 || MODE == 6) && threadIdx.x == 128) {
      size_t o = (size_t)blockIdx.x << 28;
      while (!g_stop) {
        asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(big + (o & ((1ull << 30) - 1))), "r"(65536u) : "memory");
        o += 65536;
      }
    }
    return;
  }
  const int me = blockIdx.x;  // 0 or 1
  unsigned* mine = flag + me * 32;
  unsigned* other = flag + (1 - me) * 32;
  uint4* dst = buf + (size_t)me * (bytes / 16);
  asm volatile("bar.sync 1, 128;" ::: "memory");
  unsigned long long t0 = gt();
  for (int i = 0; i < iters; ++i) {
    // CTA 0 speaks on even turns, CTA 1 answers
    if (me == 1 || i > 0) {
      if (threadIdx.x == 0) {
        const unsigned want = me == 0 ? i : i + 1;
        if (MODE == 2 || MODE == 3) {
          while (ld_acquire(other) < want) {}
        } else {
          while (ld_relaxed(other) < want) {}
          if (MODE == 1 || MODE == 4 || MODE == 5) asm volatile("fence.acq_rel.gpu;" ::: "memory");
        }
      }
      asm volatile("bar.sync 1, 128;" ::: "memory");
    }
    if (MODE == 4)
      for (int j = threadIdx.x; j < bytes / 16; j += 128) dst[j] = make_uint4(i, j, me, 0);
    asm volatile("bar.sync 1, 128;" ::: "memory");
    if (threadIdx.x == 0) {
      if (MODE == 0 || MODE == 6) asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(mine), "r"((unsigned)i + 1) : "memory");
      else if (MODE == 3) { __threadfence(); atomicAdd(mine, 1u); }
      else asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(mine) : "memory");
    }
  }
  if (threadIdx.x == 0 && me == 0) {
    while (ld_relaxed(other) < (unsigned)iters) {}
    out[0] = gt() - t0;
    g_stop = 1;
  }
}

int main() {
  unsigned* flag;
  uint4* buf;
  unsigned long long* out;
  cudaMalloc(&flag, 4096);
  cudaMalloc(&buf, 1 << 22);
  cudaMalloc(&out, 64);
  const int iters = 2000;
  char* big;
  cudaMalloc(&big, (1ull << 30) + (1 << 20));
  const char* names[] = {"relaxed", "release", "acquire", "fence+red", "+stores", "rel+bg", "rlx+bg"};
  for (int mode = 0; mode < 7; ++mode) {
    for (int bytes : {0, 4096, 16384, 32768}) {
      if (mode != 4 && bytes) continue;
      if (mode == 4 && !bytes) continue;
      cudaMemset(flag, 0, 4096);
      auto run = [&] {
        int zero = 0;
        cudaMemcpyToSymbol(g_stop, &zero, sizeof zero);
        switch (mode) {
          case 0: pingpong<0><<<2, 160>>>(flag, iters, buf, bytes, out, big); break;
          case 1: pingpong<1><<<2, 160>>>(flag, iters, buf, bytes, out, big); break;
          case 2: pingpong<2><<<2, 160>>>(flag, iters, buf, bytes, out, big); break;
          case 3: pingpong<3><<<2, 160>>>(flag, iters, buf, bytes, out, big); break;
          case 4: pingpong<4><<<2, 160>>>(flag, iters, buf, bytes, out, big); break;
          case 5: pingpong<5><<<2, 160>>>(flag, iters, buf, bytes, out, big); break;
          case 6: pingpong<6><<<2, 160>>>(flag, iters, buf, bytes, out, big); break;
        }
      };
      run();
      cudaDeviceSynchronize();
      cudaMemset(flag, 0, 4096);
      run();
      unsigned long long ns = 0;
      cudaMemcpy(&ns, out, 8, cudaMemcpyDeviceToHost);
      printf("%-10s bytes=%6d  hop %.0f ns\n", names[mode], bytes, ns / (2.0 * iters));
    }
  }
  cudaError_t e = cudaDeviceSynchronize();
  printf("%s\n", cudaGetErrorString(e));
  return 0;
}
