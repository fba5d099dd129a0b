// fp32 storage path (DP_FP32): the paper's own precision (Table 1's byte counts are fp32
// HF tensors; 417 MB = fp32 BERT-Base).  SURVEY §8(d) C1 runs tiny BERT in
// fp32 at <= 1e-4 relative to the oracle.
//
// There is no fp32 kind of tcgen05.mma (tf32 rounds the operands to 10 mantissa bits, ~1e-3
// relative), so every fp32 kernel is a CUDA-core kernel with fp32 FMA:
//   * embedding gather + LayerNorm (K1) and LayerNorm (K4): one warp per row, the row staged in
//     shared memory, gamma / beta / the token-type row staged once per CTA (DHA: every host
//     byte crosses the link once per CTA);
//   * linear (K3 / resident): a CTA owns 8 weight rows, streams them ONCE (host-mapped or HBM)
//     with coalesced 16-byte loads into shared memory before the grid-dependency wait, then
//     every warp computes 4 tokens x 8 rows per pass (W is never re-read, so the same kernel is
//     the DHA linear and the resident one: DHA vs loaded execution is bit-identical);
//   * attention (K5): 32 query rows per CTA, 32-key tiles of K / V in shared memory, fp32 online
//     softmax (one key per lane for the scores, one output column pair per lane for P.V).
// These are the correctness path of the paper's precision, not a tuned one: an fp32 cold start
// is host-link bound (twice the bytes of fp16) and the CUDA-core compute overlaps the loads.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdint>

#include "common.h"
#include "kernels.h"
#include "launch.cuh"

namespace dp {

namespace {

__device__ __forceinline__ float wsum(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}
__device__ __forceinline__ float wmax(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = fmaxf(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}
__device__ __forceinline__ float4 ld4(const float* p) {  // read-only 16-byte load (HBM or host-mapped)
  float4 r;
  asm volatile("ld.global.nc.v4.f32 {%0, %1, %2, %3}, [%4];" : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w) : "l"(p));
  return r;
}

// LayerNorm of the row in `row` (shared memory, n floats) by one warp: two-pass variance.
__device__ __forceinline__ void ln_warp_f32(const float* row, int n, float eps, const float* g, const float* b,
                                            float* y, float* y32, int lane) {
  float s = 0.f;
  for (int i = lane; i < n; i += 32) s += row[i];
  const float mean = wsum(s) / n;
  float q = 0.f;
  for (int i = lane; i < n; i += 32) {
    const float d = row[i] - mean;
    q += d * d;
  }
  const float rstd = rsqrtf(wsum(q) / n + eps);
  for (int i = lane; i < n; i += 32) {
    const float v = (row[i] - mean) * rstd * g[i] + b[i];
    y[i] = v;
    if (y32) y32[i] = v;
  }
}

constexpr int kWarps = 8;

// K1 fp32: x[t] = LN(word[id] + pos[p] + type[0]) (BERT / RoBERTa) or wte[id] + wpe[p] (GPT-2).
__global__ void __launch_bounds__(256) embed_f32_kernel(const int32_t* __restrict__ ids, int ntok, int seq,
                                                        int pos_off, const float* word, const float* pos,
                                                        const float* type, const float* g, const float* b, int H,
                                                        float eps, float* __restrict__ out, float* __restrict__ out32,
                                                        int vocab) {
  extern __shared__ float sm_e[];  // [type | gamma | beta] (3H) + kWarps rows (H each)
  pdl_trigger();
  float* st = sm_e;
  float* sg = sm_e + H;
  float* sb = sm_e + 2 * H;
  float* rows = sm_e + 3 * H;
  const int H4 = H / 4;
  for (int i = threadIdx.x; i < 3 * H4; i += blockDim.x) {  // shared rows: once per CTA
    const int which = i / H4, c = i - which * H4;
    const float* src = which == 0 ? type : (which == 1 ? g : b);
    if (src) reinterpret_cast<float4*>(sm_e)[i] = ld4(src + 4 * c);
  }
  pdl_wait();
  __syncthreads();
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int t = blockIdx.x * kWarps + warp;
  if (t >= ntok) return;
  int id = ids[t];
  if (vocab > 0) id = min(max(id, 0), vocab - 1);
  const int p = pos_off + t % seq;
  float* row = rows + warp * H;
  for (int c = lane; c < H4; c += 32) {
    const float4 w = ld4(word + (size_t)id * H + 4 * c), q = ld4(pos + (size_t)p * H + 4 * c);
    float4 v = make_float4(w.x + q.x, w.y + q.y, w.z + q.z, w.w + q.w);
    if (type) {
      const float4 y = reinterpret_cast<const float4*>(st)[c];
      v = make_float4(v.x + y.x, v.y + y.y, v.z + y.z, v.w + y.w);
    }
    reinterpret_cast<float4*>(row)[c] = v;
  }
  __syncwarp();
  float* o = out + (size_t)t * H;
  if (!g) {
    for (int i = lane; i < H; i += 32) o[i] = row[i];
    return;
  }
  ln_warp_f32(row, H, eps, sg, sb, o, out32 ? out32 + (size_t)t * H : nullptr, lane);
}

// K4 fp32: y = LN(x (+ r)) * g + b.
__global__ void __launch_bounds__(256) layernorm_f32_kernel(const float* __restrict__ x, const float* __restrict__ r,
                                                            const float* g, const float* b, float* __restrict__ y,
                                                            float* __restrict__ y32, int rows, int n, float eps) {
  extern __shared__ float sm_l[];  // gamma | beta | kWarps rows
  pdl_trigger();
  const int n4 = n / 4;
  for (int i = threadIdx.x; i < 2 * n4; i += blockDim.x)
    reinterpret_cast<float4*>(sm_l)[i] = ld4((i < n4 ? g : b) + 4 * (i < n4 ? i : i - n4));
  pdl_wait();
  __syncthreads();
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  float* row = sm_l + 2 * n + warp * n;
  for (int rr = blockIdx.x * kWarps + warp; rr < rows; rr += gridDim.x * kWarps) {
    const float* xr = x + (size_t)rr * n;
    const float* rs = r ? r + (size_t)rr * n : nullptr;
    for (int c = lane; c < n4; c += 32) {
      float4 v = reinterpret_cast<const float4*>(xr)[c];
      if (rs) {
        const float4 u = reinterpret_cast<const float4*>(rs)[c];
        v = make_float4(v.x + u.x, v.y + u.y, v.z + u.z, v.w + u.w);
      }
      reinterpret_cast<float4*>(row)[c] = v;
    }
    __syncwarp();
    ln_warp_f32(row, n, eps, sm_l, sm_l + n, y + (size_t)rr * n, y32 ? y32 + (size_t)rr * n : nullptr, lane);
    __syncwarp();
  }
}

__device__ __forceinline__ float act_f32(float v, int act) {
  switch (act) {
    case ACT_GELU_ERF: return 0.5f * v * (1.0f + erff(v * 0.70710678118654752f));
    case ACT_GELU_TANH: return 0.5f * v * (1.0f + tanhf(0.7978845608028654f * (v + 0.044715f * v * v * v)));
    case ACT_TANH: return tanhf(v);
    default: return v;
  }
}

constexpr int LR = 8;   // weight rows per CTA
constexpr int LT = 4;   // tokens per warp pass

// Linear fp32: Y[M,N] = act(X W^T + b) + res, W [N,K] read once (host-mapped or HBM).  res may
// alias Y (GPT-2's in-place residual stream): each element is read and then written by one thread.
__global__ void __launch_bounds__(256) linear_f32_kernel(const float* __restrict__ X, int ldx, const float* W,
                                                         const float* bias, const float* res, int ldr,
                                                         float* Y, int ldy, int M, int N, int K,
                                                         int act) {
  extern __shared__ float sw[];  // [LR][K]
  pdl_trigger();
  const int n0 = blockIdx.x * LR;
  const int rows = min(LR, N - n0);
  const int K4 = K / 4;
  const int total = rows * K4;
  const float* src = W + (size_t)n0 * K;  // the CTA's rows are one contiguous block
  for (int base = threadIdx.x; base < total; base += 8 * 256) {  // up to 8 loads in flight per thread
    float4 v[8];
#pragma unroll
    for (int j = 0; j < 8; ++j)
      if (base + j * 256 < total) v[j] = ld4(src + 4 * (base + j * 256));
#pragma unroll
    for (int j = 0; j < 8; ++j)
      if (base + j * 256 < total) reinterpret_cast<float4*>(sw)[base + j * 256] = v[j];
  }
  __shared__ float sbias[LR];
  if (threadIdx.x < LR) sbias[threadIdx.x] = (bias && threadIdx.x < rows) ? bias[n0 + threadIdx.x] : 0.f;
  pdl_wait();
  __syncthreads();
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  for (int m0 = warp * LT; m0 < M; m0 += kWarps * LT) {
    float acc[LT][LR];
#pragma unroll
    for (int t = 0; t < LT; ++t)
#pragma unroll
      for (int r = 0; r < LR; ++r) acc[t][r] = 0.f;
    for (int c = lane; c < K4; c += 32) {
      float4 xv[LT];
#pragma unroll
      for (int t = 0; t < LT; ++t)
        xv[t] = m0 + t < M ? reinterpret_cast<const float4*>(X + (size_t)(m0 + t) * ldx)[c] : make_float4(0, 0, 0, 0);
#pragma unroll
      for (int r = 0; r < LR; ++r) {
        if (r < rows) {
          const float4 w = reinterpret_cast<const float4*>(sw + r * K)[c];
#pragma unroll
          for (int t = 0; t < LT; ++t) {
            acc[t][r] = fmaf(xv[t].x, w.x, acc[t][r]);
            acc[t][r] = fmaf(xv[t].y, w.y, acc[t][r]);
            acc[t][r] = fmaf(xv[t].z, w.z, acc[t][r]);
            acc[t][r] = fmaf(xv[t].w, w.w, acc[t][r]);
          }
        }
      }
    }
#pragma unroll
    for (int t = 0; t < LT; ++t) {
      float mine = 0.f;
#pragma unroll
      for (int r = 0; r < LR; ++r) {
        const float v = wsum(acc[t][r]);
        if (lane == r) mine = v;
      }
      const int m = m0 + t;
      if (lane < rows && m < M) {
        const int n = n0 + lane;
        float v = act_f32(mine + sbias[lane], act);
        if (res) v += res[(size_t)m * ldr + n];
        Y[(size_t)m * ldy + n] = v;
      }
    }
  }
}

constexpr int AQ = 32, AK = 32, AD = 64;

// Attention fp32: ctx = softmax(q k^T / sqrt(64) [causal]) v per head.  grid (heads, q tiles, batch).
__global__ void __launch_bounds__(128) attention_f32_kernel(const float* __restrict__ qkv, int ldqkv,
                                                            float* __restrict__ ctx, int seq, int H, int causal) {
  __shared__ float sq[AQ][AD];
  __shared__ float sk[AK][AD + 1];  // +1: lane j reads row j without bank conflicts
  __shared__ float sv[AK][AD];
  pdl_trigger();
  pdl_wait();  // q, k, v come from the previous kernels
  const int head = blockIdx.x, q0 = blockIdx.y * AQ, bidx = blockIdx.z;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const size_t tok0 = (size_t)bidx * seq;
  const float* qb = qkv + tok0 * ldqkv + head * AD;
  const float* kb = qb + H;
  const float* vb = qb + 2 * H;
  for (int i = tid; i < AQ * AD; i += 128) {
    const int r = i / AD, c = i % AD;
    sq[r][c] = q0 + r < seq ? qb[(size_t)(q0 + r) * ldqkv + c] * 0.125f : 0.f;  // 1/sqrt(64): exact
  }
  constexpr int RW = AQ / 4;  // query rows per warp
  float mrow[RW], lrow[RW], o0[RW], o1[RW];
#pragma unroll
  for (int j = 0; j < RW; ++j) mrow[j] = -INFINITY, lrow[j] = 0.f, o0[j] = 0.f, o1[j] = 0.f;
  int nkt = (seq + AK - 1) / AK;
  if (causal) nkt = min(nkt, (q0 + AQ - 1) / AK + 1);
  for (int kt = 0; kt < nkt; ++kt) {
    const int k0 = kt * AK;
    __syncthreads();  // the previous tile is consumed (and sq is visible on the first pass)
    for (int i = tid; i < AK * AD; i += 128) {
      const int r = i / AD, c = i % AD;
      const bool ok = k0 + r < seq;
      sk[r][c] = ok ? kb[(size_t)(k0 + r) * ldqkv + c] : 0.f;
      sv[r][c] = ok ? vb[(size_t)(k0 + r) * ldqkv + c] : 0.f;
    }
    __syncthreads();
#pragma unroll
    for (int j = 0; j < RW; ++j) {
      const int r = warp * RW + j, qrow = q0 + r;
      if (qrow >= seq) continue;  // warp-uniform
      const int key = k0 + lane;
      float s = 0.f;
#pragma unroll 16
      for (int d = 0; d < AD; ++d) s = fmaf(sq[r][d], sk[lane][d], s);
      const bool valid = key < seq && (!causal || key <= qrow);
      s = valid ? s : -INFINITY;
      const float mnew = fmaxf(mrow[j], wmax(s));
      if (mnew == -INFINITY) continue;  // every key of this tile masked
      const float alpha = mrow[j] == -INFINITY ? 0.f : expf(mrow[j] - mnew);
      const float p = valid ? expf(s - mnew) : 0.f;
      lrow[j] = lrow[j] * alpha + wsum(p);
      float a0 = o0[j] * alpha, a1 = o1[j] * alpha;
#pragma unroll 8
      for (int kk = 0; kk < AK; ++kk) {
        const float pk = __shfl_sync(0xffffffffu, p, kk);
        a0 = fmaf(pk, sv[kk][lane], a0);
        a1 = fmaf(pk, sv[kk][lane + 32], a1);
      }
      o0[j] = a0, o1[j] = a1;
      mrow[j] = mnew;
    }
  }
#pragma unroll
  for (int j = 0; j < RW; ++j) {
    const int qrow = q0 + warp * RW + j;
    if (qrow >= seq) continue;
    const float inv = lrow[j] > 0.f ? 1.f / lrow[j] : 0.f;
    float* c = ctx + (tok0 + qrow) * H + head * AD;
    c[lane] = o0[j] * inv;
    c[lane + 32] = o1[j] * inv;
  }
}

}  // namespace

void launch_embed_f32(const int32_t* ids, int ntok, int seq, int pos_off, const void* word, const void* pos,
                      const void* type, const void* g, const void* b, int H, float eps, void* out, void* out32,
                      int vocab, cudaStream_t s) {
  DP_CHECK(H % 4 == 0, DP_ERR_INVALID, "fp32 embedding: hidden must be a multiple of 4");
  const size_t smem = size_t(3 + kWarps) * H * 4;
  DP_CHECK(smem <= 200 * 1024, DP_ERR_UNSUPPORTED, "fp32 embedding: hidden too large");
  static std::atomic<unsigned> attr{0};
  if (first_on_device(attr))
    DP_CUDA(cudaFuncSetAttribute(embed_f32_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024));
  launch_kernel(embed_f32_kernel, dim3((ntok + kWarps - 1) / kWarps), dim3(256), smem, s, ids, ntok, seq, pos_off,
                (const float*)word, (const float*)pos, (const float*)type, (const float*)g, (const float*)b, H, eps,
                (float*)out, (float*)out32, vocab);
  DP_CUDA(cudaGetLastError());
}

void launch_layernorm_f32(const void* x, const void* r, const void* g, const void* b, void* y, int rows, int n,
                          float eps, cudaStream_t s, void* y32) {
  DP_CHECK(n % 4 == 0, DP_ERR_INVALID, "fp32 LayerNorm: width must be a multiple of 4");
  const size_t smem = size_t(2 + kWarps) * n * 4;
  DP_CHECK(smem <= 200 * 1024, DP_ERR_UNSUPPORTED, "fp32 LayerNorm: width too large");
  static std::atomic<unsigned> attr{0};
  if (first_on_device(attr))
    DP_CUDA(cudaFuncSetAttribute(layernorm_f32_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024));
  const int grid = std::max(1, std::min((rows + kWarps - 1) / kWarps, 148 * 8));
  launch_kernel(layernorm_f32_kernel, dim3(grid), dim3(256), smem, s, (const float*)x, (const float*)r,
                (const float*)g, (const float*)b, (float*)y, (float*)y32, rows, n, eps);
  DP_CUDA(cudaGetLastError());
}

void launch_linear_f32(const void* x, int ldx, const void* w, const void* bias, const void* res, int ldr, void* y,
                       int ldy, int M, int N, int K, int act, cudaStream_t s) {
  DP_CHECK(K % 4 == 0 && ldx % 4 == 0, DP_ERR_INVALID, "fp32 linear: K and ldx must be multiples of 4");
  const size_t smem = size_t(LR) * K * 4;
  DP_CHECK(smem <= 200 * 1024, DP_ERR_UNSUPPORTED, "fp32 linear: K too large");
  static std::atomic<unsigned> attr{0};
  if (first_on_device(attr))
    DP_CUDA(cudaFuncSetAttribute(linear_f32_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024));
  launch_kernel(linear_f32_kernel, dim3((N + LR - 1) / LR), dim3(256), smem, s, (const float*)x, ldx,
                (const float*)w, (const float*)bias, (const float*)res, ldr, (float*)y, ldy, M, N, K, act);
  DP_CUDA(cudaGetLastError());
}

void launch_attention_f32(const void* qkv, int ldqkv, void* ctx, int batch, int seq, int H, int heads, bool causal,
                          cudaStream_t s) {
  DP_CHECK(heads > 0 && H % heads == 0 && H / heads == AD, DP_ERR_UNSUPPORTED, "attention needs head dim 64");
  launch_kernel(attention_f32_kernel, dim3(heads, (seq + AQ - 1) / AQ, batch), dim3(128), 0, s, (const float*)qkv,
                ldqkv, (float*)ctx, seq, H, causal ? 1 : 0);
  DP_CUDA(cudaGetLastError());
}

}  // namespace dp
