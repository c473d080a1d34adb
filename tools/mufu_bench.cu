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
// cvt.rn.bf16x2.f32 (F2FP): 1 op = one packed pair
__global__ void k_f2fp(float* out, int iters) {
  float a = threadIdx.x * 1e-3f, b = a + 1.f;
  unsigned acc = 0;
  for (int i = 0; i < iters; ++i) {
    unsigned r0, r1, r2, r3;
    asm volatile("cvt.rn.bf16x2.f32 %0, %1, %2;" : "=r"(r0) : "f"(a), "f"(b));
    asm volatile("cvt.rn.bf16x2.f32 %0, %1, %2;" : "=r"(r1) : "f"(b), "f"(a));
    asm volatile("cvt.rn.bf16x2.f32 %0, %1, %2;" : "=r"(r2) : "f"(a), "f"(a));
    asm volatile("cvt.rn.bf16x2.f32 %0, %1, %2;" : "=r"(r3) : "f"(b), "f"(b));
    acc ^= r0 ^ r1 ^ r2 ^ r3;
    a += 1e-7f;
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = (float)acc;
}
// softmax inner loop per element pair: 2 FFMA, 2 ex2, 2 FADD, 1 F2FP  (per = 2 elements)
__global__ void k_mix(float* out, int iters) {
  float s0 = threadIdx.x * 1e-3f, s1 = s0 + 0.5f, l0 = 0.f, l1 = 0.f;
  unsigned acc = 0;
  for (int i = 0; i < iters; ++i) {
    float p0, p1;
    asm volatile("ex2.approx.ftz.f32 %0, %1;" : "=f"(p0) : "f"(fmaf(s0, 0.18f, -1.f)));
    asm volatile("ex2.approx.ftz.f32 %0, %1;" : "=f"(p1) : "f"(fmaf(s1, 0.18f, -1.f)));
    l0 += p0; l1 += p1;
    unsigned r;
    asm volatile("cvt.rn.bf16x2.f32 %0, %1, %2;" : "=r"(r) : "f"(p1), "f"(p0));
    acc ^= r;
    s0 += 1e-6f; s1 -= 1e-6f;
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = l0 + l1 + (float)acc;
}
// ex2.approx.f16x2 / ex2.approx.ftz.bf16x2: 1 op = 2 exps (per counts exps)
__global__ void k_ex2_h2(float* out, int iters) {
  unsigned a = 0x3c003c00u + threadIdx.x, b = a ^ 0x10001u, c = a ^ 0x20002u, d = a ^ 0x30003u;
  for (int i = 0; i < iters; ++i) {
    asm volatile("ex2.approx.f16x2 %0, %0;" : "+r"(a)); asm volatile("ex2.approx.f16x2 %0, %0;" : "+r"(b));
    asm volatile("ex2.approx.f16x2 %0, %0;" : "+r"(c)); asm volatile("ex2.approx.f16x2 %0, %0;" : "+r"(d));
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = (float)(a ^ b ^ c ^ d);
}
__global__ void k_ex2_bh2(float* out, int iters) {
  unsigned a = 0x3f803f80u + threadIdx.x, b = a ^ 0x10001u, c = a ^ 0x20002u, d = a ^ 0x30003u;
  for (int i = 0; i < iters; ++i) {
    asm volatile("ex2.approx.ftz.bf16x2 %0, %0;" : "+r"(a)); asm volatile("ex2.approx.ftz.bf16x2 %0, %0;" : "+r"(b));
    asm volatile("ex2.approx.ftz.bf16x2 %0, %0;" : "+r"(c)); asm volatile("ex2.approx.ftz.bf16x2 %0, %0;" : "+r"(d));
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = (float)(a ^ b ^ c ^ d);
}
int main() {
  int sms = 0; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  int clk = 0; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  float* out; cudaMalloc(&out, sms * 4 * 1024 * 4);
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  const int iters = 4096;
  struct { const char* n; void (*k)(float*, int); int per; } ks[] = {{"ex2", k_ex2, 4}, {"rcp", k_rcp, 4}, {"ffma", k_ffma, 8},
               {"f2fp", k_f2fp, 4}, {"mix(elem)", k_mix, 2}, {"ex2h2", k_ex2_h2, 8}, {"ex2bh2", k_ex2_bh2, 8}};
  for (auto& kk : ks) {
    kk.k<<<sms * 4, 1024>>>(out, 16);
    cudaEventRecord(a);
    kk.k<<<sms * 4, 1024>>>(out, iters);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b);
    double ops = (double)sms * 4 * 1024 * iters * kk.per;
    double per_sm_per_s = ops / (ms / 1e3) / sms;
    printf("%-10s %.3f ms  %.1f Gop/s/SM  = %.1f /clk/SM at %d MHz (max clock)\n", kk.n, ms, per_sm_per_s / 1e9,
           per_sm_per_s / (clk * 1e3), clk / 1000);
  }
  return 0;
}
