// common.cuh — shared device helpers for the sm_100a kernels of libarlo.so.
#pragma once

#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include <atomic>
#include <utility>

namespace arlo {

using bf16 = __nv_bfloat16;

// Element-type traits: activations are either fp32 (check mode) or bf16.
template <typename T> struct Elem;
template <> struct Elem<float> {
  static __device__ __forceinline__ float to_f(float v) { return v; }
  static __device__ __forceinline__ float from_f(float v) { return v; }
};
template <> struct Elem<bf16> {
  static __device__ __forceinline__ float to_f(bf16 v) { return __bfloat162float(v); }
  static __device__ __forceinline__ bf16 from_f(float v) { return __float2bfloat16_rn(v); }
};

__device__ __forceinline__ float warp_sum(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}

__device__ __forceinline__ float warp_max(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = fmaxf(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}

// GELU, erf form (reading S2): 0.5 z (1 + erf(z / sqrt 2)), fp32.
__device__ __forceinline__ float gelu_erf(float z) {
  return 0.5f * z * (1.0f + erff(z * 0.70710678118654752440f));
}

// GELU, erf form, evaluated with Abramowitz & Stegun 7.1.26
//   erfc(a) = (a1 t + ... + a5 t^5) exp(-a^2),  t = 1 / (1 + p a),  |error| <= 1.5e-7
// for the bf16 tensor-core epilogues (output rounding 2^-9 relative dwarfs it).
// With a = |z|/sqrt 2 and h = 0.5 |z| erfc(a):  GELU(z) = max(z, 0) - h  for both signs.
// 2 MUFU (rcp, ex2) + ~10 FMA-pipe ops instead of erff's ~25 (its FSEL-selected
// two-branch polynomial); fp32 check mode keeps gelu_erf above.
__device__ __forceinline__ float rcp_approx(float x) {
  float r;
  asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x));
  return r;
}
__device__ __forceinline__ float2 f2c(float v) { return make_float2(v, v); }
__device__ __forceinline__ float ex2_approx(float x) {
  float r;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x));
  return r;
}

// 2^x for two values on the FMA pipe (no MUFU): x = j + f with j = rint(x) (the 1.5 * 2^23
// shifter), f in [-1/2, 1/2], 2^f by its degree-5 Taylor polynomial (relative error <= 2.4e-6,
// far below the bf16 rounding of P), then j added to the exponent field.  x is clamped at
// -127, where the result is 0 as ex2.approx.ftz gives.  The attention softmax evaluates a
// fixed subset of its exponentials this way (by key position only, so every runtime L
// computes a given key's p identically) to take load off the 16/clk/SM MUFU unit.
__device__ __forceinline__ float2 ex2_poly2(float2 x) {
  x = make_float2(fmaxf(x.x, -127.0f), fmaxf(x.y, -127.0f));
  const float2 t = __fadd2_rn(x, f2c(12582912.0f));
  const float2 j = __fadd2_rn(t, f2c(-12582912.0f));  // rint(x), exact
  const float2 f = __fadd2_rn(x, make_float2(-j.x, -j.y));  // exact
  float2 q = __ffma2_rn(f, f2c(1.3333558146e-3f), f2c(9.6181291076e-3f));
  q = __ffma2_rn(q, f, f2c(5.5504108665e-2f));
  q = __ffma2_rn(q, f, f2c(2.4022650696e-1f));
  q = __ffma2_rn(q, f, f2c(6.9314718056e-1f));
  q = __ffma2_rn(q, f, f2c(1.0f));
  return make_float2(__int_as_float(__float_as_int(q.x) + (__float_as_int(t.x) << 23)),
                     __int_as_float(__float_as_int(q.y) + (__float_as_int(t.y) << 23)));
}

__device__ __forceinline__ float gelu_erf_fast(float z) {
#if defined(ARLO_GELU_EXPERIMENT)  // A/B only: tanh-form GELU, 1 MUFU (NOT the erf form; reading S2)
  float th;
  asm("tanh.approx.f32 %0, %1;" : "=f"(th) : "f"(0.7978845608f * fmaf(0.044715f * z, z * z, z)));
  return 0.5f * z * (1.0f + th);
#elif defined(ARLO_GELU_AS28)
  // A&S 7.1.28: erf(a) = 1 - (1 + a1 a + ... + a6 a^6)^-16, |error| <= 3e-7; one MUFU (rcp)
  const float az = fabsf(z);
  const float a = az * 0.70710678118654752f;
  float p = fmaf(a, 0.0000430638f, 0.0002765672f);
  p = fmaf(a, p, 0.0001520143f);
  p = fmaf(a, p, 0.0092705272f);
  p = fmaf(a, p, 0.0422820123f);
  p = fmaf(a, p, 0.0705230784f);
  p = fmaf(a, p, 1.0f);
  float r = rcp_approx(p);
  r *= r;
  r *= r;
  r *= r;
  r *= r;  // (1 + ...)^-16 = erfc(a)
  return fmaf(-0.5f * az, r, fmaxf(z, 0.0f));
#else
  const float az = fabsf(z);
  const float t = rcp_approx(fmaf(az, 0.3275911f * 0.70710678118654752f, 1.0f));
  // coefficients pre-multiplied by 0.5
  float q = fmaf(t, 0.5f * 1.061405429f, 0.5f * -1.453152027f);
  q = fmaf(t, q, 0.5f * 1.421413741f);
  q = fmaf(t, q, 0.5f * -0.284496736f);
  q = fmaf(t, q, 0.5f * 0.254829592f);
  q *= t;
  const float e = ex2_approx(z * z * (-0.5f * 1.4426950408889634f));  // exp(-z^2/2) = exp(-a^2)
  return fmaxf(z, 0.0f) - az * q * e;
#endif
}

// GELU (erf form, reading S2) on two values with the sm_100 paired fp32 instructions (FFMA2 /
// FMUL2).  Every GEMM epilogue (single CTA, CTA pair, skinny, split-K, fused) uses this one
// function, so a given element is computed bitwise identically whatever tile produced it.
// Default: Abramowitz & Stegun 7.1.28, erfc(a) = (1 + c1 a + ... + c6 a^6)^-16, |erf error| <=
// 3e-7 (pinned against scipy in tests/test_gelu_fast.py): ONE MUFU op (rcp) per element.  The
// 7.1.26 form below (ARLO_GELU2_AS26) takes two (rcp, ex2); the GELU epilogue runs at the
// 16/clk/SM MUFU rate (gemm_trace: ~2000 of a chunk's cycles are its math), so halving the MUFU
// count shortens the exposed epilogue of the one- and two-round FFN1 GEMMs.
// GELU = max(z, 0) + (-0.5 |z| erfc(|z| / sqrt 2)).
__device__ __forceinline__ float2 f2(float v) { return make_float2(v, v); }
__device__ __forceinline__ float2 gelu2_erf_fast(float2 z) {
  const float2 az = make_float2(fabsf(z.x), fabsf(z.y));
#if !defined(ARLO_GELU2_AS26)
  // A&S 7.1.28; a = |z| / sqrt 2 is folded into the coefficients (c_k 2^(-k/2))
  float2 p = __ffma2_rn(az, f2(0.0000430638f * 0.125f), f2(0.0002765672f * 0.17677669529663687f));
  p = __ffma2_rn(az, p, f2(0.0001520143f * 0.25f));
  p = __ffma2_rn(az, p, f2(0.0092705272f * 0.35355339059327379f));
  p = __ffma2_rn(az, p, f2(0.0422820123f * 0.5f));
  p = __ffma2_rn(az, p, f2(0.0705230784f * 0.70710678118654752f));
  p = __ffma2_rn(az, p, f2(1.0f));
  float2 r = make_float2(rcp_approx(p.x), rcp_approx(p.y));
  r = __fmul2_rn(r, r);
  r = __fmul2_rn(r, r);
  r = __fmul2_rn(r, r);
  r = __fmul2_rn(r, r);  // erfc(a)
  return __ffma2_rn(__fmul2_rn(az, f2(-0.5f)), r, make_float2(fmaxf(z.x, 0.0f), fmaxf(z.y, 0.0f)));
#else  // A&S 7.1.26 (two MUFU ops)
  const float2 d = __ffma2_rn(az, f2(0.3275911f * 0.70710678118654752f), f2(1.0f));
  const float2 t = make_float2(rcp_approx(d.x), rcp_approx(d.y));
  float2 q = __ffma2_rn(t, f2(-0.5f * 1.061405429f), f2(-0.5f * -1.453152027f));
  q = __ffma2_rn(t, q, f2(-0.5f * 1.421413741f));
  q = __ffma2_rn(t, q, f2(-0.5f * -0.284496736f));
  q = __ffma2_rn(t, q, f2(-0.5f * 0.254829592f));
  const float2 s = __fmul2_rn(__fmul2_rn(z, z), f2(-0.5f * 1.4426950408889634f));
  const float2 e = make_float2(ex2_approx(s.x), ex2_approx(s.y));  // exp(-z^2/2) = exp(-a^2)
  const float2 h = __fmul2_rn(__fmul2_rn(q, t), az);                // -0.5 |z| erfc(a) / exp(-a^2)
  return __ffma2_rn(h, e, make_float2(fmaxf(z.x, 0.0f), fmaxf(z.y, 0.0f)));
#endif
}

// Pack two floats into a bf16x2 word (RNE), low half = a.
__device__ __forceinline__ uint32_t pack_bf16x2(float a, float b) {
  __nv_bfloat162 h = __floats2bfloat162_rn(a, b);
  return *reinterpret_cast<uint32_t*>(&h);
}

__device__ __forceinline__ float2 unpack_bf16x2(uint32_t w) {
  __nv_bfloat162 h = *reinterpret_cast<__nv_bfloat162*>(&w);
  return __bfloat1622float2(h);
}

// Programmatic dependent launch (PDL): every hot-path kernel is launched with
// programmatic stream serialization; it lets its dependents launch (their
// prologue then overlaps this kernel's tail) and waits for its predecessor's
// completion before touching global memory.
__device__ __forceinline__ void pdl_launch_dependents() {
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_begin() {
  pdl_launch_dependents();
  pdl_wait();
}

// 16-byte load of data a PREDECESSOR kernel produced (activations, residuals), for use
// after pdl_wait().  A volatile asm load is kept after the volatile griddepcontrol.wait;
// __ldg / const __restrict__ loads (ld.global.nc) are not: nvcc hoisted such loads above
// the wait (SASS: LDG.CONSTANT before ACQBULK), which read the pooled features before the
// pooler had written them.  Weights (never written by a kernel) keep __ldg.
__device__ __forceinline__ uint4 ld_dep_v4(const void* p) {
  uint4 v;
  asm volatile("ld.global.v4.u32 {%0, %1, %2, %3}, [%4];"
               : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
               : "l"(p)
               : "memory");
  return v;
}

__device__ __forceinline__ float4 ld_dep_f4(const void* p) {
  const uint4 u = ld_dep_v4(p);
  return make_float4(__uint_as_float(u.x), __uint_as_float(u.y), __uint_as_float(u.z), __uint_as_float(u.w));
}

__device__ __forceinline__ uint2 ld_dep_v2(const void* p) {
  uint2 v;
  asm volatile("ld.global.v2.u32 {%0, %1}, [%2];" : "=r"(v.x), "=r"(v.y) : "l"(p) : "memory");
  return v;
}

// Mean and 1/sqrt(var + eps) of a row from its granule statistics (FoldArgs; granule-major
// st[g][row][2], plane stride `ld` rows): the G = H/32 granules added in column order, var =
// E[y^2] - mean^2 (clamped at 0).  Loads go out in groups of 8 (a chain of dependent L2 loads
// under GEMM traffic cost microseconds per tile).
__device__ __forceinline__ float2 fold_row_stats(const float* st, size_t row, int ld, int G, int H, float eps) {
  const float2* p = reinterpret_cast<const float2*>(st) + row;
  float s1 = 0.f, s2 = 0.f;
  for (int g0 = 0; g0 < G; g0 += 8) {
    float2 v[8];
#pragma unroll
    for (int i = 0; i < 8; ++i)
      if (g0 + i < G) v[i] = __ldcg(p + (size_t)(g0 + i) * ld);
#pragma unroll
    for (int i = 0; i < 8; ++i)
      if (g0 + i < G) {
        s1 += v[i].x;
        s2 += v[i].y;
      }
  }
  const float mean = s1 / (float)H;
  const float var = fmaxf(s2 / (float)H - mean * mean, 0.f);
  return make_float2(mean, 1.0f / sqrtf(var + eps));
}

bool pdl_enabled();  // false when ARLO_NO_PDL is set in the environment (A/B measurements)

// Kernel attributes (the >48 KB dynamic shared memory opt-in, ...) belong to the CURRENT
// device's context, and runtimes of one process may live on several devices and be built
// from several host threads.  `done` keeps one bit per device index (a static per kernel
// instantiation); setting an attribute twice is harmless, so a race only repeats the call.
template <typename SetFn>
inline cudaError_t once_per_device(std::atomic<uint64_t>& done, SetFn set) {
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  const uint64_t bit = 1ull << (dev & 63);
  if (done.load(std::memory_order_acquire) & bit) return cudaSuccess;
  e = set();
  if (e == cudaSuccess) done.fetch_or(bit, std::memory_order_acq_rel);
  return e;
}

// Grid-wide barrier of a PERSISTENT grid (every CTA resident at once: grid <= one CTA per SM).
// bar[0] counts arrivals and is reset by the last arriver, bar[1] is a generation counter the
// waiters poll, so the same zero-initialised pair serves every later launch (graph replays).
// Each CTA's thread 0 reads the generation BEFORE arriving; release / acquire at gpu scope
// order the CTA's prior writes before the other CTAs' later reads.
__device__ __forceinline__ unsigned ld_acquire_gpu(const unsigned* p) {
  unsigned v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void grid_barrier(unsigned* bar) {
  __syncthreads();
  if (threadIdx.x == 0) {
    const unsigned gen = ld_acquire_gpu(bar + 1);
    __threadfence();
    if (atomicAdd(bar, 1u) == gridDim.x * gridDim.y * gridDim.z - 1) {
      atomicExch(bar, 0u);
      __threadfence();
      atomicAdd(bar + 1, 1u);
    } else {
      while (ld_acquire_gpu(bar + 1) == gen) __nanosleep(20);
    }
    __threadfence();
  }
  __syncthreads();
}

template <typename... KArgs, typename... Args>
inline cudaError_t launch_k(void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t s,
                            Args&&... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = pdl_enabled() ? 1 : 0;
  return cudaLaunchKernelEx(&cfg, kern, std::forward<Args>(args)...);
}

}  // namespace arlo
