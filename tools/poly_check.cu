// Stand-alone device check of the attention kernel's exp2 paths (poly on FMA pipe vs MUFU).
#include <cstdio>
#include <cstdint>
#include <cmath>
#include <vector>
__device__ __forceinline__ uint64_t pk2(float a, float b) { uint64_t r; asm("mov.b64 %0, {%1, %2};" : "=l"(r) : "f"(a), "f"(b)); return r; }
__device__ __forceinline__ void up2(uint64_t v, float& a, float& b) { asm("mov.b64 {%0, %1}, %2;" : "=f"(a), "=f"(b) : "l"(v)); }
__device__ __forceinline__ uint64_t ffma2(uint64_t a, uint64_t b, uint64_t c) { uint64_t d; asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(d) : "l"(a), "l"(b), "l"(c)); return d; }
__device__ __forceinline__ uint64_t fadd2(uint64_t a, uint64_t b) { uint64_t d; asm("add.f32x2 %0, %1, %2;" : "=l"(d) : "l"(a), "l"(b)); return d; }
__device__ __forceinline__ uint64_t exp2_poly2(uint64_t x) {
  float x0, x1; up2(x, x0, x1);
  x = pk2(fmaxf(x0, -127.0f), fmaxf(x1, -127.0f));
  const uint64_t magic = pk2(12582912.0f, 12582912.0f);
  const uint64_t t = fadd2(x, magic);
  const uint64_t jf = fadd2(t, pk2(-12582912.0f, -12582912.0f));
  float j0, j1; up2(jf, j0, j1);
  const uint64_t f = fadd2(x, pk2(-j0, -j1));
  uint64_t p = ffma2(pk2(0.05592204f, 0.05592204f), f, pk2(0.24264008f, 0.24264008f));
  p = ffma2(p, f, pk2(0.69312103f, 0.69312103f));
  p = ffma2(p, f, pk2(0.99992448f, 0.99992448f));
  float p0, p1, t0, t1; up2(p, p0, p1); up2(t, t0, t1);
  const uint32_t r0 = __float_as_uint(p0) + (__float_as_uint(t0) << 23);
  const uint32_t r1 = __float_as_uint(p1) + (__float_as_uint(t1) << 23);
  return pk2(__uint_as_float(r0), __uint_as_float(r1));
}
__global__ void k(const float* x, float* y, int n) {
  int i = 2 * (blockIdx.x * blockDim.x + threadIdx.x);
  if (i + 1 >= n) return;
  uint64_t e = exp2_poly2(pk2(x[i], x[i + 1]));
  up2(e, y[i], y[i + 1]);
}
int main() {
  const int n = 1 << 20;
  std::vector<float> hx(n), hy(n);
  for (int i = 0; i < n; ++i) hx[i] = -30.0f + 38.0f * i / n;
  float *dx, *dy; cudaMalloc(&dx, n * 4); cudaMalloc(&dy, n * 4);
  cudaMemcpy(dx, hx.data(), n * 4, cudaMemcpyHostToDevice);
  k<<<n / 512, 256>>>(dx, dy, n);
  cudaMemcpy(hy.data(), dy, n * 4, cudaMemcpyDeviceToHost);
  double worst = 0; float wx = 0;
  for (int i = 0; i < n; ++i) { double r = std::fabs(hy[i] / std::exp2((double)hx[i]) - 1); if (r > worst) { worst = r; wx = hx[i]; } }
  printf("poly exp2 max rel err %.3g at x=%g (%s)\n", worst, wx, cudaGetErrorString(cudaGetLastError()));
  for (float v : {-7.5f, -1.0f, -0.5f, 0.0f, 0.25f, 3.7f}) { cudaMemcpy(dx, &v, 4, cudaMemcpyHostToDevice); }
  return 0;
}
