// One LayerNorm row per warp: fp32 statistics, two-pass variance, gamma/beta from shared
// memory.  Shared by the LayerNorm kernel (K4) and the GEMM epilogue that normalises complete
// rows (K2 + K4 fused), so the fused and unfused paths are bit-identical.
#pragma once
#include "dtype.cuh"

namespace dp {

// 8 elements at index i of a T or fp32 array through L2 only (coherent with stores made by
// other CTAs of the running grid, unlike the read-only path).
template <class T>
__device__ __forceinline__ void load8_cg(const void* base, size_t i, float* f, int f32) {
  if (f32) {
    const float4* p = reinterpret_cast<const float4*>(static_cast<const float*>(base) + i);
    const float4 a = __ldcg(p), b = __ldcg(p + 1);
    f[0] = a.x; f[1] = a.y; f[2] = a.z; f[3] = a.w; f[4] = b.x; f[5] = b.y; f[6] = b.z; f[7] = b.w;
  } else {
    uint4 u = __ldcg(reinterpret_cast<const uint4*>(static_cast<const T*>(base) + i));
    unpack8<T>(u, f);
  }
}

// 8 elements through a generic pointer (e.g. a row staged in shared memory).
template <class T>
__device__ __forceinline__ void load8_generic(const void* base, size_t i, float* f, int f32) {
  if (f32) {
    const float4* p = reinterpret_cast<const float4*>(static_cast<const float*>(base) + i);
    const float4 a = p[0], b = p[1];
    f[0] = a.x; f[1] = a.y; f[2] = a.z; f[3] = a.w; f[4] = b.x; f[5] = b.y; f[6] = b.z; f[7] = b.w;
  } else {
    unpack8<T>(*reinterpret_cast<const uint4*>(static_cast<const T*>(base) + i), f);
  }
}

// y[yoff .. yoff+n) = LN(x[off ..] (+ r[off ..])) * gamma + beta.  VPL >= ceil(n / 256); lanes
// past n are skipped (not added as zeros), so any VPL gives the same arithmetic sequence.
// SRC: 0 = read-only global path, 1 = L2-coherent global, 2 = generic (shared memory).
template <class T, int VPL, int SRC>
__device__ __forceinline__ void ln_row_warp(const void* x, const void* r, size_t off, int n, float eps, int in_f32,
                                            const uint4* gb, T* y, size_t yoff, float* y32 = nullptr) {
  const int lane = threadIdx.x & 31, nv = n / 8;
  float v[VPL][8];
  float sum = 0.f;
#pragma unroll
  for (int k = 0; k < VPL; ++k) {
    const int c = lane + 32 * k;
    if (c < nv) {
      if (SRC == 1)
        load8_cg<T>(x, off + 8 * c, v[k], in_f32);
      else if (SRC == 2)
        load8_generic<T>(x, off + 8 * c, v[k], in_f32);
      else
        load8<T>(x, off + 8 * c, v[k], in_f32);
      if (r) {
        float a[8];
        load8<T>(r, off + 8 * c, a, in_f32);
#pragma unroll
        for (int e = 0; e < 8; ++e) v[k][e] += a[e];
      }
#pragma unroll
      for (int e = 0; e < 8; ++e) sum += v[k][e];
    }
  }
  const float mean = warp_sum(sum) / n;
  float sq = 0.f;
#pragma unroll
  for (int k = 0; k < VPL; ++k) {
    const int c = lane + 32 * k;
    if (c < nv) {
#pragma unroll
      for (int e = 0; e < 8; ++e) {
        const float d = v[k][e] - mean;
        sq += d * d;
      }
    }
  }
  const float rstd = rsqrtf(warp_sum(sq) / n + eps);
#pragma unroll
  for (int k = 0; k < VPL; ++k) {
    const int c = lane + 32 * k;
    if (c < nv) {
      float gg[8], bb[8], o[8];
      unpack8<T>(gb[c], gg);
      unpack8<T>(gb[nv + c], bb);
#pragma unroll
      for (int e = 0; e < 8; ++e) o[e] = (v[k][e] - mean) * rstd * gg[e] + bb[e];
      reinterpret_cast<uint4*>(y + yoff)[c] = pack8<T>(o);
      if (y32 != nullptr) store8<T>(y32, yoff + 8 * c, o, 1);  // fp32 residual-stream copy
    }
  }
}

}  // namespace dp
