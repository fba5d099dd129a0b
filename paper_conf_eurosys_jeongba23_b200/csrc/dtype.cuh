// fp16 / bf16 <-> fp32 helpers on 16-byte vectors (8 elements).
#pragma once
#include <cuda_bf16.h>
#include <cuda_fp16.h>
#include <cstdint>

#include "kernels.h"

namespace dp {

template <class T>
struct Cvt;

template <>
struct Cvt<__half> {
  static __device__ __forceinline__ float2 to2(uint32_t v) {
    __half2 h = *reinterpret_cast<__half2*>(&v);
    return __half22float2(h);
  }
  static __device__ __forceinline__ uint32_t from2(float a, float b) {
    __half2 h = __floats2half2_rn(a, b);
    return *reinterpret_cast<uint32_t*>(&h);
  }
  static __device__ __forceinline__ float to1(__half v) { return __half2float(v); }
  static __device__ __forceinline__ __half from1(float v) { return __float2half_rn(v); }
};

template <>
struct Cvt<__nv_bfloat16> {
  static __device__ __forceinline__ float2 to2(uint32_t v) {
    __nv_bfloat162 h = *reinterpret_cast<__nv_bfloat162*>(&v);
    return __bfloat1622float2(h);
  }
  static __device__ __forceinline__ uint32_t from2(float a, float b) {
    __nv_bfloat162 h = __floats2bfloat162_rn(a, b);
    return *reinterpret_cast<uint32_t*>(&h);
  }
  static __device__ __forceinline__ float to1(__nv_bfloat16 v) { return __bfloat162float(v); }
  static __device__ __forceinline__ __nv_bfloat16 from1(float v) { return __float2bfloat16_rn(v); }
};

template <class T>
__device__ __forceinline__ void unpack8(const uint4& u, float* f) {
  float2 a = Cvt<T>::to2(u.x), b = Cvt<T>::to2(u.y), c = Cvt<T>::to2(u.z), d = Cvt<T>::to2(u.w);
  f[0] = a.x; f[1] = a.y; f[2] = b.x; f[3] = b.y; f[4] = c.x; f[5] = c.y; f[6] = d.x; f[7] = d.y;
}

template <class T>
__device__ __forceinline__ uint4 pack8(const float* f) {
  uint4 u;
  u.x = Cvt<T>::from2(f[0], f[1]);
  u.y = Cvt<T>::from2(f[2], f[3]);
  u.z = Cvt<T>::from2(f[4], f[5]);
  u.w = Cvt<T>::from2(f[6], f[7]);
  return u;
}

// 16-byte read-only load; works on HBM and on host-mapped (zero-copy) addresses.
__device__ __forceinline__ uint4 ldg16(const void* p) {
  uint4 r;
  asm volatile("ld.global.nc.v4.u32 {%0, %1, %2, %3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
               : "l"(p));
  return r;
}

// 8 consecutive elements at element index i of a T or fp32 array (f32 selects).
template <class T>
__device__ __forceinline__ void load8(const void* base, size_t i, float* f, int f32) {
  if (f32) {
    const float4* p = reinterpret_cast<const float4*>(static_cast<const float*>(base) + i);
    const float4 a = p[0], b = p[1];
    f[0] = a.x; f[1] = a.y; f[2] = a.z; f[3] = a.w; f[4] = b.x; f[5] = b.y; f[6] = b.z; f[7] = b.w;
  } else {
    unpack8<T>(ldg16(static_cast<const T*>(base) + i), f);
  }
}

template <class T>
__device__ __forceinline__ void store8(void* base, size_t i, const float* f, int f32) {
  if (f32) {
    float4* p = reinterpret_cast<float4*>(static_cast<float*>(base) + i);
    p[0] = make_float4(f[0], f[1], f[2], f[3]);
    p[1] = make_float4(f[4], f[5], f[6], f[7]);
  } else {
    *reinterpret_cast<uint4*>(static_cast<T*>(base) + i) = pack8<T>(f);
  }
}

template <class T>
__device__ __forceinline__ float load1(const void* base, size_t i, int f32) {
  return f32 ? static_cast<const float*>(base)[i] : Cvt<T>::to1(static_cast<const T*>(base)[i]);
}

template <class T>
__device__ __forceinline__ void store1(void* base, size_t i, float v, int f32) {
  if (f32)
    static_cast<float*>(base)[i] = v;
  else
    static_cast<T*>(base)[i] = Cvt<T>::from1(v);
}

// Thread-block clusters: this CTA's rank, and the broadcast of rank 0's shared-memory buffer to
// every rank (DSMEM reads between two cluster barriers).  Used so that rows every CTA needs (LN
// gamma / beta, the token-type row) cross the host link ONCE per cluster when they live in host
// memory (DHA), instead of once per CTA.
__device__ __forceinline__ uint32_t cta_cluster_rank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}

__device__ __forceinline__ void cluster_bcast_from_rank0(uint4* buf, int n16) {
  // (1) rank 0's buffer is written and visible cluster-wide
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
  if (cta_cluster_rank() != 0) {
    const uint32_t base = static_cast<uint32_t>(__cvta_generic_to_shared(buf));
    uint32_t remote;
    asm volatile("mapa.shared::cluster.u32 %0, %1, 0;" : "=r"(remote) : "r"(base));
    for (int i = threadIdx.x; i < n16; i += blockDim.x) {
      uint4 v;
      asm volatile("ld.shared::cluster.v4.u32 {%0, %1, %2, %3}, [%4];"
                   : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
                   : "r"(remote + 16u * i)
                   : "memory");
      buf[i] = v;
    }
  }
  // (2) every rank has its copy (rank 0 may exit; this CTA's copy is visible to its threads)
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}

// 2^x on the MUFU, flushing subnormal results to zero (exp2f adds the subnormal-range fix-up --
// two FMULs and a select per call -- which the softmax numerators never need: p < 2^-126 is
// irrelevant next to the row maximum's 1).  2^-inf = +0.
__device__ __forceinline__ float fast_exp2(float x) {
  float y;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}

__device__ __forceinline__ float warp_sum(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}

__device__ __forceinline__ float gelu_erf(float x) { return 0.5f * x * (1.0f + erff(x * 0.70710678118654752f)); }
// 0.5 x (1 + tanh(u)) == x / (1 + exp(-2u)) exactly (1 + tanh(u) = 2 / (1 + exp(-2u))), so the
// tanh form of GELU is one exponential and one division: MUFU ex2 + rcp instead of the libm tanhf
// (~25 instructions with branches) that dominated the GPT-2 fc epilogues.  Relative error a few
// fp32 ulps; exp overflow at very negative x gives x / inf = -0, the exact limit.
__device__ __forceinline__ float gelu_tanh(float x) {
  const float c2 = 2.f * 0.7978845608028654f;  // 2 sqrt(2/pi)
  const float e = __expf(-c2 * (x + 0.044715f * x * x * x));
  return __fdividef(x, 1.f + e);
}

// Compile-time activation: an epilogue specialised per activation stays small (a runtime
// switch inlined per element made the GEMM epilogue ~4 K instructions, instruction-fetch bound).
template <int ACT>
__device__ __forceinline__ float apply_act_c(float v) {
  if constexpr (ACT == ACT_GELU_ERF) return gelu_erf(v);
  else if constexpr (ACT == ACT_GELU_TANH) return gelu_tanh(v);
  else if constexpr (ACT == ACT_TANH) return tanhf(v);
  else return v;
}

__device__ __forceinline__ float apply_act(float v, int act) {
  switch (act) {
    case ACT_GELU_ERF: return gelu_erf(v);
    case ACT_GELU_TANH: return gelu_tanh(v);
    case ACT_TANH: return tanhf(v);
    default: return v;
  }
}

}  // namespace dp
