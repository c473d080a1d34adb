// pdl_chain_bench.cu — floor of a chain of dependent kernels in one CUDA graph on B200 (the
// batch-1 forward is 63-87 such launches: what does a launch cost before any work?).
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/pdl_chain_bench tools/pdl_chain_bench.cu
//   tools/pdl_chain_bench
//
// N = 64 launches of one kernel captured in a graph, replayed between CUDA events; per variant
// the time per launch (us, median of 20 replays):
//   pdl / plain   launched with / without programmatic stream serialization (the runtime's
//                 kernels use PDL: launch_dependents first, griddepcontrol.wait before global reads)
//   grid          CTAs per launch (1, 48 = the skinny N/16 grid of BERT-base N = 768, 148, 296)
//   work          0: the kernel only waits and exits; 1: each CTA then reads 16 KB that the
//                 previous launch wrote (L2-resident, like a GEMM's A operand) and writes 16 KB
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <vector>

__global__ void __launch_bounds__(128) link(const uint4* __restrict__ in, uint4* __restrict__ out, int work) {
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  asm volatile("griddepcontrol.wait;" ::: "memory");
  if (!work) return;
  const size_t base = (size_t)blockIdx.x * 1024;  // 16 KB per CTA
  uint4 acc = make_uint4(0, 0, 0, 0);
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    uint4 v;
    asm volatile("ld.global.v4.u32 {%0, %1, %2, %3}, [%4];"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
                 : "l"(in + base + i * 128 + threadIdx.x)
                 : "memory");
    acc.x += v.x; acc.y ^= v.y; acc.z += v.z; acc.w ^= v.w;
    out[base + i * 128 + threadIdx.x] = acc;
  }
}

static float run(bool pdl, int grid, int work, uint4* a, uint4* b) {
  const int N = 64;
  cudaStream_t s;
  cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
  cudaGraph_t g;
  cudaStreamBeginCapture(s, cudaStreamCaptureModeGlobal);
  for (int i = 0; i < N; ++i) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(grid);
    cfg.blockDim = dim3(128);
    cfg.stream = s;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at;
    cfg.numAttrs = pdl ? 1 : 0;
    const uint4* in = (i & 1) ? b : a;
    uint4* out = (i & 1) ? a : b;
    cudaLaunchKernelEx(&cfg, link, in, out, work);
  }
  cudaStreamEndCapture(s, &g);
  cudaGraphExec_t ge;
  cudaGraphInstantiate(&ge, g, 0);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  for (int i = 0; i < 3; ++i) cudaGraphLaunch(ge, s);
  std::vector<float> t;
  for (int r = 0; r < 20; ++r) {
    cudaEventRecord(e0, s);
    cudaGraphLaunch(ge, s);
    cudaEventRecord(e1, s);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    t.push_back(ms * 1e3f / N);
  }
  std::sort(t.begin(), t.end());
  cudaGraphExecDestroy(ge);
  cudaGraphDestroy(g);
  cudaStreamDestroy(s);
  return t[t.size() / 2];
}

int main() {
  uint4 *a, *b;
  const size_t bytes = (size_t)296 * 16384;
  cudaMalloc(&a, bytes);
  cudaMalloc(&b, bytes);
  cudaMemset(a, 1, bytes);
  cudaMemset(b, 2, bytes);
  printf("# us per launch, 64 dependent launches in one CUDA graph (median of 20 replays)\n");
  printf("%6s %5s %10s %10s\n", "grid", "work", "pdl", "plain");
  for (int grid : {1, 48, 148, 296})
    for (int work : {0, 1})
      printf("%6d %5d %10.2f %10.2f\n", grid, work, run(true, grid, work, a, b), run(false, grid, work, a, b));
  const cudaError_t e = cudaDeviceSynchronize();
  if (e != cudaSuccess) {
    printf("CUDA error: %s\n", cudaGetErrorString(e));
    return 1;
  }
  return 0;
}
