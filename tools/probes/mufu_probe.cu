// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o mufu_probe mufu_probe.cu
// Throughput probe: the softmax inner step (FFMA + exp2 + FADD over 64 register-resident scores)
// with WARPS warps per CTA, one CTA per SM; exp2 by MUFU (ex2.approx) or by the FMA-pipe
// polynomial for every POLY-th element.  Prints cycles per element per SM.
#include <cstdio>
#include <cuda_runtime.h>
__device__ __forceinline__ float ex2(float x) { float y; asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x)); return y; }
__device__ __forceinline__ float exp2_poly(float x) {
  x = fmaxf(x, -126.f);
  const float t = x + 12582912.f;
  const float f = x - (t - 12582912.f);
  const float p = fmaf(fmaf(fmaf(0.0551703f, f, 0.242608f), f, 0.693261f), f, 0.999928f);
  return __int_as_float(__float_as_int(p) + (__float_as_int(t) << 23));
}
template <int POLY>
__global__ void probe(float* out, int iters, float scale, long long* cyc) {
  float s[64];
  for (int e = 0; e < 64; ++e) s[e] = -0.01f * (threadIdx.x + e);
  float acc = 0.f;
  long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
    float r8[8] = {0, 0, 0, 0, 0, 0, 0, 0};
#pragma unroll
    for (int e = 0; e < 64; ++e) {
      const float x = fmaf(s[e], scale, -acc * 1e-30f);
      const float p = (POLY > 0 && (e % POLY) == POLY - 1) ? exp2_poly(x) : ex2(x);
      r8[e & 7] += p;
      s[e] = p * 0.5f - 1.f;
    }
    acc += ((r8[0] + r8[1]) + (r8[2] + r8[3])) + ((r8[4] + r8[5]) + (r8[6] + r8[7]));
  }
  long long t1 = clock64();
  if (threadIdx.x == 0 && blockIdx.x == 0) *cyc = t1 - t0;
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}
int main() {
  float* out; long long* cyc; cudaMalloc(&out, 148 * 1024 * 4); cudaMallocManaged(&cyc, 8);
  const int iters = 2000;
  for (int warps : {4, 8, 16}) {
    for (int poly : {0, 4, 2}) {
      auto run = [&](auto k) { k<<<148, warps * 32>>>(out, iters, 0.18f, cyc); cudaDeviceSynchronize(); k<<<148, warps * 32>>>(out, iters, 0.18f, cyc); cudaDeviceSynchronize(); };
      if (poly == 0) run(probe<0>); else if (poly == 4) run(probe<4>); else run(probe<2>);
      const double el = double(iters) * 64 * warps * 32;
      printf("warps %2d poly 1/%d: %.3f elements/clk/SM (%lld cycles)\n", warps, poly, el / *cyc, *cyc);
    }
  }
  return 0;
}
