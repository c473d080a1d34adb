// Microbenchmark: MUFU ex2 / rcp and FFMA throughput per SM on this GPU.
#include <cstdio>
#include <cuda_runtime.h>
__global__ void k_ex2(float* out, int iters) {
  float a = threadIdx.x * 1e-3f, b = a + 1.f, c = a + 2.f, d = a + 3.f;
  for (int i = 0; i < iters; ++i) {
    asm volatile("ex2.approx.ftz.f32 %0, %0;" : "+f"(a)); asm volatile("ex2.approx.ftz.f32 %0, %0;" : "+f"(b));
    asm volatile("ex2.approx.ftz.f32 %0, %0;" : "+f"(c)); asm volatile("ex2.approx.ftz.f32 %0, %0;" : "+f"(d));
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = a + b + c + d;
}
__global__ void k_rcp(float* out, int iters) {
  float a = threadIdx.x * 1e-3f + 1.f, b = a + 1.f, c = a + 2.f, d = a + 3.f;
  for (int i = 0; i < iters; ++i) {
    asm volatile("rcp.approx.ftz.f32 %0, %0;" : "+f"(a)); asm volatile("rcp.approx.ftz.f32 %0, %0;" : "+f"(b));
    asm volatile("rcp.approx.ftz.f32 %0, %0;" : "+f"(c)); asm volatile("rcp.approx.ftz.f32 %0, %0;" : "+f"(d));
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = a + b + c + d;
}
__global__ void k_ffma(float* out, int iters) {
  float a = threadIdx.x * 1e-3f, b = a + 1.f, c = a + 2.f, d = a + 3.f, e = a + 4, f = a + 5, g = a + 6, h = a + 7;
  for (int i = 0; i < iters; ++i) {
    a = fmaf(a, 0.999f, 0.1f); b = fmaf(b, 0.999f, 0.1f); c = fmaf(c, 0.999f, 0.1f); d = fmaf(d, 0.999f, 0.1f);
    e = fmaf(e, 0.999f, 0.1f); f = fmaf(f, 0.999f, 0.1f); g = fmaf(g, 0.999f, 0.1f); h = fmaf(h, 0.999f, 0.1f);
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = a + b + c + d + e + f + g + h;
}
int main() {
  int sms = 0; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  int clk = 0; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  float* out; cudaMalloc(&out, sms * 4 * 1024 * 4);
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  const int iters = 4096;
  struct { const char* n; void (*k)(float*, int); int per; } ks[] = {{"ex2", k_ex2, 4}, {"rcp", k_rcp, 4}, {"ffma", k_ffma, 8}};
  for (auto& kk : ks) {
    kk.k<<<sms * 4, 1024>>>(out, 16);
    cudaEventRecord(a);
    kk.k<<<sms * 4, 1024>>>(out, iters);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b);
    double ops = (double)sms * 4 * 1024 * iters * kk.per;
    double per_sm_per_s = ops / (ms / 1e3) / sms;
    printf("%-5s %.3f ms  %.1f Gop/s/SM  = %.1f /clk/SM at %d MHz (max clock)\n", kk.n, ms, per_sm_per_s / 1e9,
           per_sm_per_s / (clk * 1e3), clk / 1000);
  }
  return 0;
}
