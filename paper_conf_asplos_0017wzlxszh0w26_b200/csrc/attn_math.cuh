// Helpers shared by the attention kernels (k_attn.cu, k_attn_pair.cu): packed f32x2 math
// (FFMA2 / FADD2), 3-input max, MUFU and FMA-pipe exp2, the work-item record of the plan.
#pragma once
#include <cuda_runtime.h>
#include <cstdint>

namespace bat {
namespace {

__device__ __forceinline__ float ex2(float x) {
  float y;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}

// ---- packed f32x2 math (FFMA2 / FADD2) and 3-input max (FMNMX3), sm_100a
__device__ __forceinline__ uint64_t pk2(float a, float b) {
  uint64_t r;
  asm("mov.b64 %0, {%1, %2};" : "=l"(r) : "f"(a), "f"(b));
  return r;
}
__device__ __forceinline__ void up2(uint64_t v, float& a, float& b) {
  asm("mov.b64 {%0, %1}, %2;" : "=f"(a), "=f"(b) : "l"(v));
}
__device__ __forceinline__ uint64_t ffma2(uint64_t a, uint64_t b, uint64_t c) {
  uint64_t d;
  asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(d) : "l"(a), "l"(b), "l"(c));
  return d;
}
__device__ __forceinline__ uint64_t fadd2(uint64_t a, uint64_t b) {
  uint64_t d;
  asm("add.f32x2 %0, %1, %2;" : "=l"(d) : "l"(a), "l"(b));
  return d;
}
__device__ __forceinline__ float fmax3(float a, float b, float c) {
  float d;
  asm("max.f32 %0, %1, %2, %3;" : "=f"(d) : "f"(a), "f"(b), "f"(c));
  return d;
}
// 2^x for a pair on the FMA pipe (offloads the MUFU): x = j + f, j = rint(x) by the
// 1.5*2^23 trick, 2^f on [-0.5, 0.5] by a degree-3 minimax polynomial (rel. err 1.1e-4, far
// below the bf16 rounding of P), exponent inserted with an integer multiply-add.  x is clamped
// at -126 so the inserted exponent never underflows the field: p(0) = 0.99992 < 1 has biased
// exponent 126, so j = -127 would wrap into the sign bit (a NaN, seen with rows whose scores
// span > 126 log2 units — tests/test_gpu_attn_rescale.py); 2^-126 is far below P's bf16 ulp.
__device__ __forceinline__ uint64_t exp2_poly2(uint64_t x) {
  float x0, x1;
  up2(x, x0, x1);
  x = pk2(fmaxf(x0, -126.0f), fmaxf(x1, -126.0f));
  const uint64_t magic = pk2(12582912.0f, 12582912.0f);
  const uint64_t t = fadd2(x, magic);
  const uint64_t jf = fadd2(t, pk2(-12582912.0f, -12582912.0f));
  float j0, j1;
  up2(jf, j0, j1);
  const uint64_t f = fadd2(x, pk2(-j0, -j1));
  uint64_t p = ffma2(pk2(0.05592204f, 0.05592204f), f, pk2(0.24264008f, 0.24264008f));
  p = ffma2(p, f, pk2(0.69312103f, 0.69312103f));
  p = ffma2(p, f, pk2(0.99992448f, 0.99992448f));
  float p0, p1, t0, t1;
  up2(p, p0, p1);
  up2(t, t0, t1);
  const uint32_t r0 = __float_as_uint(p0) + (__float_as_uint(t0) << 23);
  const uint32_t r1 = __float_as_uint(p1) + (__float_as_uint(t1) << 23);
  return pk2(__uint_as_float(r0), __uint_as_float(r1));
}

struct WorkItem {
  int b, kvh, q0, q1, kt_off, kt_n, tp_off, km_off;
};
__device__ __forceinline__ WorkItem load_work(const int32_t* work, int w) {
  const int4 a = *reinterpret_cast<const int4*>(work + int64_t(w) * 8);
  const int4 c = *reinterpret_cast<const int4*>(work + int64_t(w) * 8 + 4);
  return WorkItem{a.x, a.y, a.z, a.w, c.x, c.y, c.z, c.w};
}

}  // namespace
}  // namespace bat
