// Microbenchmark: latency of mbarrier.test_wait / try_wait polling from one
// thread, alone and while other warps spin or sleep on another barrier.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/mbar_bench tools/mbar_bench.cu
#include <cstdio>
#include <cstdint>

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ bool test(uint64_t* bar, uint32_t par) {
  uint32_t ok;
  asm volatile("{\n\t.reg .pred p;\n\tmbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}"
               : "=r"(ok) : "r"(su32(bar)), "r"(par) : "memory");
  return ok;
}
__device__ __forceinline__ bool trywait(uint64_t* bar, uint32_t par) {
  uint32_t ok;
  asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}"
               : "=r"(ok) : "r"(su32(bar)), "r"(par) : "memory");
  return ok;
}

// mode 0: thread 0 polls test_wait (parity 1 of a fresh barrier: completed -> true? use parity 0: not complete)
// others idle at __syncthreads.  mode 1: same with try_wait.  mode 2: test_wait while
// warps 1..nw-1 spin on test_wait of a second barrier.  mode 3: warps sleep in try_wait.
__global__ void k(int mode, int iters, long long* out) {
  __shared__ uint64_t bar[2];
  __shared__ volatile int stop;
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar[0])));
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar[1])));
    stop = 0;
  }
  __syncthreads();
  const int warp = threadIdx.x >> 5;
  if (warp == 0) {
    if (threadIdx.x == 0) {
      int hits = 0;
      long long t0 = clock64();
      for (int i = 0; i < iters; ++i) hits += (mode == 1) ? trywait(&bar[0], 0) : test(&bar[0], 0);
      long long t1 = clock64();
      out[0] = (t1 - t0);
      out[1] = hits;
      asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(su32(&bar[1])) : "memory");
    }
  } else if (mode >= 2) {
    if (mode == 2)
      while (!test(&bar[1], 0)) {}
    else
      while (!trywait(&bar[1], 0)) {}
  }
  __syncthreads();
}

int main() {
  long long* d;
  cudaMalloc(&d, 16);
  const int iters = 10000;
  const char* names[] = {"test_wait alone", "try_wait alone (not complete: suspends until timeout)",
                         "test_wait with 9 warps spinning test_wait", "test_wait with 9 warps in try_wait"};
  for (int mode = 0; mode < 4; ++mode) {
    if (mode == 1) {  // try_wait on an incomplete barrier suspends up to a timeout: use fewer iters
      k<<<1, 320>>>(mode, 100, d);
    } else {
      k<<<1, 320>>>(mode, iters, d);
    }
    long long h[2];
    cudaMemcpy(h, d, 16, cudaMemcpyDeviceToHost);
    printf("%-60s %.1f cycles/poll (hits %lld) err=%s\n", names[mode], (double)h[0] / (mode == 1 ? 100 : iters), h[1],
           cudaGetErrorString(cudaGetLastError()));
  }
  return 0;
}
