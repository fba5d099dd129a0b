// K5t: attention core on the 5th-generation tensor cores (tcgen05 + TMEM + TMA), d = 64.
//
//   ctx[q, h*64 : h*64+64] = softmax(q_h k_h^T / 8 [+ causal mask]) v_h
//
// One CTA (256 threads) per (head, 128-query tile, sequence).  Per 128-key tile j:
//   1. S = Q K_j^T on tcgen05 (M = 128 queries, N = 128 keys, K = 64), fp32 in TMEM columns
//      [0, 128); Q and K_j arrive by TMA (128-byte swizzle), K double-buffered;
//   2. two threads own query row r = TMEM lane r (warps w and w + 4 read the lane quarter w % 4),
//      each half of its S row (tcgen05.ld): masks, the online softmax in fp32 with exp2 (the
//      halves' maxima meet in shared memory; each keeps a partial row sum under the same
//      corrections);
//      the numerators P (storage type) go to shared memory as the next MMA's A operand, written
//      in the 128-byte-swizzled K-major layout by hand; V_j arrives by TMA as [keys][head dims]
//      and is the MN-major B operand as it lands (no transpose);
//   3. O_j = P V_j on tcgen05 (M = 128, N = 64, K = 128 keys) into TMEM columns [128, 192);
//   4. thread r accumulates o_r = o_r * corr + O_j[r] in registers.
// After the last key tile o_r / l_r is stored (128 bytes per row).  Arithmetic contract: S and
// O_j in fp32, P rounded to the storage type before P V (as the mma.sync K5), row sums in fp32.
#include <cuda.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstring>

#include "common.h"
#include "dtype.cuh"
#include "kernels.h"
#include "launch.cuh"
#include "tc.cuh"

namespace dp {

namespace {

constexpr int TQ = 128;  // queries per CTA (MMA M, TMEM lanes)
constexpr int TK = 128;  // keys per tile (MMA N of S, K of P V)
constexpr int TD = 64;   // head dim
constexpr uint32_t Q_BYTES = TQ * TD * 2;      // 16 KB
constexpr uint32_t K_BYTES = TK * TD * 2;      // 16 KB
constexpr uint32_t P_BYTES = TQ * TK * 2;      // 32 KB: two [128][64] swizzled K-blocks
constexpr uint32_t V_BYTES = TK * TD * 2;      // 16 KB: [128 keys][64] swizzled (MN-major B operand)
constexpr uint32_t SMEM_BYTES = Q_BYTES + 2 * K_BYTES + P_BYTES + 2 * V_BYTES + 1024;

// byte offset of element (r, k) of a K-major [rows][64] tile with the 128-byte swizzle
__device__ __forceinline__ uint32_t sw128_off(int r, int k) {
  return uint32_t(r) * 128u + ((uint32_t((k >> 3) ^ (r & 7))) << 4) + uint32_t(k & 7) * 2u;
}

template <class T>
__global__ void __launch_bounds__(256, 1)
    attention_tc_kernel(const __grid_constant__ CUtensorMap tmQK, const T* __restrict__ qkv, int ldqkv,
                        T* __restrict__ ctx, int seq, int H, int causal, float scale_log2) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  uint8_t* sQ = smem;
  uint8_t* sK = sQ + Q_BYTES;           // [2][TK][64]
  uint8_t* sP = sK + 2 * K_BYTES;       // [2 k-blocks][TQ][64]
  uint8_t* sV = sP + P_BYTES;           // [2][TK][64]: V tiles as TMA lands them (keys x head dims)
  __shared__ __align__(8) uint64_t bar_q, bar_k[2], bar_v[2], bar_s[2], bar_o[2];
  __shared__ uint32_t tmem_base_sh;
  __shared__ float red[2][TQ];          // per column half: partial row max (and at the end: row sum)
  // kind::f16, fp32 accumulate, A/B K-major; S: M 128 x N 128; O: M 128 x N 64
  constexpr uint32_t IDESC_S = (1u << 4) | (FmtBits<T>::v << 7) | (FmtBits<T>::v << 10) | (uint32_t(TK >> 3) << 17) |
                               (uint32_t(TQ >> 4) << 24);
  // O: B = V_j is MN-major (head dims contiguous, keys along K): the transpose-B bit (16)
  constexpr uint32_t IDESC_O = (1u << 4) | (FmtBits<T>::v << 7) | (FmtBits<T>::v << 10) | (1u << 16) |
                               (uint32_t(TD >> 3) << 17) | (uint32_t(TQ >> 4) << 24);

  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  // grid (heads, query tiles, batch); causal query tiles longest first
  const int head = blockIdx.x, bidx = blockIdx.z;
  const int qt = causal ? (int)gridDim.y - 1 - (int)blockIdx.y : (int)blockIdx.y;
  const int q0 = qt * TQ;
  const int tok0 = bidx * seq;
  int nkt = (seq + TK - 1) / TK;
  if (causal) nkt = min(nkt, (q0 + TQ - 1) / TK + 1);

  if (tid == 0) {
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&tmQK)) : "memory");
    mbar_init(&bar_q, 1);
    mbar_init(&bar_k[0], 1);
    mbar_init(&bar_k[1], 1);
    mbar_init(&bar_v[0], 1);
    mbar_init(&bar_v[1], 1);
    mbar_init(&bar_s[0], 1);
    mbar_init(&bar_s[1], 1);
    mbar_init(&bar_o[0], 1);
    mbar_init(&bar_o[1], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&tmem_base_sh)),
                 "r"(512));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tmem = tmem_base_sh;
  // TMEM: S double buffer in columns [0, 256), O double buffer in [256, 384)
  auto t_s = [&](int b) { return tmem + 128u * uint32_t(b); };
  auto t_o = [&](int b) { return tmem + 256u + 64u * uint32_t(b); };
  pdl_trigger();
  pdl_wait();  // q, k, v come from the previous kernel

  const int qcol = head * TD, kcol = H + head * TD;
  const int vcol = 2 * H + head * TD;
  // thread (warp w, lane l): query row r = 32 (w % 4) + l (its TMEM lane), column half h = w / 4
  // -- keys [64 h, 64 h + 64) of each S tile, head dims [32 h, 32 h + 32) of O
  const int r = (warp & 3) * 32 + lane, h = warp >> 2;
  const uint32_t lane_base = uint32_t((warp & 3) * 32) << 16;
  const int qrow = q0 + r;
  auto issue_s = [&](int jj) {  // S_jj = Q K_jj^T into TMEM buffer jj & 1 (K_jj must be landing)
    mbar_wait_spin(&bar_k[jj & 1], (jj >> 1) & 1);
    asm volatile("tcgen05.fence::after_thread_sync;");
    const uint64_t dq = sw128_desc(sQ), dk = sw128_desc(sK + (jj & 1) * K_BYTES);
#pragma unroll
    for (int kk = 0; kk < TD / 16; ++kk) umma_f16(t_s(jj & 1), dq + 2 * kk, dk + 2 * kk, IDESC_S, kk != 0);
    umma_commit(&bar_s[jj & 1]);
  };
  if (tid == 0) {
    mbar_expect_tx(&bar_q, Q_BYTES);
    tma_load_2d(&tmQK, &bar_q, sQ, qcol, tok0 + q0);
    for (int jj = 0; jj < 2 && jj < nkt; ++jj) {
      mbar_expect_tx(&bar_k[jj], K_BYTES);
      tma_load_2d(&tmQK, &bar_k[jj], sK + jj * K_BYTES, kcol, tok0 + jj * TK);
      mbar_expect_tx(&bar_v[jj], V_BYTES);
      tma_load_2d(&tmQK, &bar_v[jj], sV + jj * V_BYTES, vcol, tok0 + jj * TK);
    }
    mbar_wait_spin(&bar_q, 0);
    issue_s(0);
  }
  float o[TD / 2];
#pragma unroll
  for (int d = 0; d < TD / 2; ++d) o[d] = 0.f;
  float mrow = -INFINITY, lrow = 0.f;  // lrow: this half's partial row sum (same corrections)
  float corr_prev = 0.f;               // the correction that goes with the O tile in flight

  // Software pipeline per key tile j: S_{j+1} is computed on the tensor core while the threads run
  // the softmax of tile j, and O_j = P_j V_j is added to the registers one iteration later.
  for (int j = 0; j < nkt; ++j) {
    const int k0 = j * TK;
    // (1) the next S on the tensor core (its buffer was last read in iteration j - 1)
    if (tid == 0 && j + 1 < nkt) issue_s(j + 1);
    // (2) S_j ready; K_j's buffer is free again -> K_{j+2}
    mbar_wait_spin(&bar_s[j & 1], (j >> 1) & 1);
    asm volatile("tcgen05.fence::after_thread_sync;");
    if (tid == 0 && j + 2 < nkt) {
      mbar_expect_tx(&bar_k[j & 1], K_BYTES);
      tma_load_2d(&tmQK, &bar_k[j & 1], sK + (j & 1) * K_BYTES, kcol, tok0 + k0 + 2 * TK);
    }
    // (3) this half of the S row -> online softmax
    float s[TK / 2];
    {
      uint32_t v[TK / 2];
#pragma unroll
      for (int c = 0; c < TK / 2; c += 16) tmem_ld16_nowait(t_s(j & 1) + lane_base + 64 * h + c, v + c);
      tmem_ld_wait();
#pragma unroll
      for (int e = 0; e < TK / 2; ++e) s[e] = __uint_as_float(v[e]);  // scaled inside the exponent
    }
    const int kbase = k0 + 64 * h;
    if (kbase + 64 > seq || (causal && kbase + 63 > qrow)) {  // only where a key can be invalid
#pragma unroll
      for (int e = 0; e < TK / 2; ++e) {
        const int key = kbase + e;
        if (key >= seq || (causal && key > qrow)) s[e] = -INFINITY;
      }
    }
    float mx = -INFINITY;
#pragma unroll
    for (int e = 0; e < TK / 2; ++e) mx = fmaxf(mx, s[e]);
    red[h][r] = mx;
    __syncthreads();
    const float mnew = fmaxf(mrow, fmaxf(red[0][r], red[1][r]) * scale_log2);
    const float corr = (mrow == -INFINITY) ? 0.f : fast_exp2(mrow - mnew);
    const float mref = (mnew == -INFINITY) ? 0.f : mnew;  // a fully masked row: every p = 2^-inf = 0
    float rs = 0.f;
#pragma unroll
    for (int e = 0; e < TK / 2; ++e) {
      const float p = fast_exp2(fmaf(s[e], scale_log2, -mref));
      rs += p;
      s[e] = p;
    }
    lrow = lrow * corr + rs;
    mrow = mnew;
    // (4) O_{j-1} has landed: add it (with the correction of its own tile); P and V^T are free
    if (j > 0) {
      mbar_wait_spin(&bar_o[(j - 1) & 1], ((j - 1) >> 1) & 1);
      asm volatile("tcgen05.fence::after_thread_sync;");
      uint32_t v[TD / 2];
#pragma unroll
      for (int c = 0; c < TD / 2; c += 16) tmem_ld16_nowait(t_o((j - 1) & 1) + lane_base + 32 * h + c, v + c);
      tmem_ld_wait();
#pragma unroll
      for (int e = 0; e < TD / 2; ++e) o[e] = o[e] * corr_prev + __uint_as_float(v[e]);
      // V_{j-1}'s buffer is free (O_{j-1} done): V_{j+1} into it
      if (tid == 0 && j + 1 < nkt) {
        mbar_expect_tx(&bar_v[(j + 1) & 1], V_BYTES);
        tma_load_2d(&tmQK, &bar_v[(j + 1) & 1], sV + ((j + 1) & 1) * V_BYTES, vcol, tok0 + k0 + TK);
      }
    }
    corr_prev = corr;
    // (5) P_j row half (K-block h) into the A-operand tile
    {
      uint8_t* pt = sP + h * (TQ * 64 * 2);
#pragma unroll
      for (int c = 0; c < 8; ++c) {
        const float* pp = s + c * 8;
        uint4 u;
        u.x = Cvt<T>::from2(pp[0], pp[1]);
        u.y = Cvt<T>::from2(pp[2], pp[3]);
        u.z = Cvt<T>::from2(pp[4], pp[5]);
        u.w = Cvt<T>::from2(pp[6], pp[7]);
        *reinterpret_cast<uint4*>(pt + sw128_off(r, c * 8)) = u;
      }
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // P -> the tensor core
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    // (6) O_j = P_j V_j into TMEM buffer j & 1
    if (tid == 0) {
      mbar_wait_spin(&bar_v[j & 1], (j >> 1) & 1);
      asm volatile("tcgen05.fence::after_thread_sync;");
      // V_j as the MN-major B operand: 128-byte swizzle atoms of 8 keys x 64 head dims, 1024 B apart
      // along K (SBO); a 16-key step advances 2048 B (128 in descriptor units)
      const uint64_t dv = sw128_desc(sV + (j & 1) * V_BYTES);
#pragma unroll
      for (int kb = 0; kb < 2; ++kb) {
        const uint64_t dp_ = sw128_desc(sP + kb * (TQ * 64 * 2));
#pragma unroll
        for (int kk = 0; kk < 4; ++kk)
          umma_f16(t_o(j & 1), dp_ + 2 * kk, dv + 128 * (kb * 4 + kk), IDESC_O, (kb | kk) != 0);
      }
      umma_commit(&bar_o[j & 1]);
    }
  }
  {  // the last O tile
    const int jl = nkt - 1;
    mbar_wait_spin(&bar_o[jl & 1], (jl >> 1) & 1);
    asm volatile("tcgen05.fence::after_thread_sync;");
    uint32_t v[TD / 2];
#pragma unroll
    for (int c = 0; c < TD / 2; c += 16) tmem_ld16_nowait(t_o(jl & 1) + lane_base + 32 * h + c, v + c);
    tmem_ld_wait();
#pragma unroll
    for (int e = 0; e < TD / 2; ++e) o[e] = o[e] * corr_prev + __uint_as_float(v[e]);
  }
  red[h][r] = lrow;  // the two halves' partial sums
  __syncthreads();
  if (qrow < seq) {
    const float l = red[0][r] + red[1][r];
    const float inv = l > 0.f ? 1.f / l : 0.f;
    uint4* dst = reinterpret_cast<uint4*>(ctx + (size_t)(tok0 + qrow) * H + head * TD + 32 * h);
#pragma unroll
    for (int c = 0; c < 4; ++c) {
      uint4 u;
      u.x = Cvt<T>::from2(o[c * 8 + 0] * inv, o[c * 8 + 1] * inv);
      u.y = Cvt<T>::from2(o[c * 8 + 2] * inv, o[c * 8 + 3] * inv);
      u.z = Cvt<T>::from2(o[c * 8 + 4] * inv, o[c * 8 + 5] * inv);
      u.w = Cvt<T>::from2(o[c * 8 + 6] * inv, o[c * 8 + 7] * inv);
      dst[c] = u;
    }
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(512));
}

}  // namespace

bool attention_tc_supported(int ldqkv, int H, int heads, const void* qkv) {
  return heads > 0 && H % heads == 0 && H / heads == TD && ldqkv % 8 == 0 && ((uintptr_t)qkv % 16) == 0;
}

void launch_attention_tc(int dtype, const void* qkv, int ldqkv, void* ctx, int batch, int seq, int H, int heads,
                         bool causal, cudaStream_t s) {
  const int T = batch * seq;
  // one map over the whole qkv matrix: box [128 rows][64 columns] with the 128-byte swizzle, for
  // the Q tile (columns h*64) and the K tiles (columns H + h*64); rows past T read as zeros
  const CUtensorMap m = make_kmajor_map(qkv, dtype, T, 3 * H, ldqkv, 128);
  const float scale_log2 = 1.4426950408889634f / 8.0f;  // log2(e) / sqrt(64)
  const dim3 grid(heads, (seq + TQ - 1) / TQ, batch);
  auto go = [&](auto tag) {
    using T = decltype(tag);
    static std::atomic<unsigned> attr{0};
    if (first_on_device(attr))
      DP_CUDA(cudaFuncSetAttribute(attention_tc_kernel<T>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                   (int)SMEM_BYTES));
    launch_kernel(attention_tc_kernel<T>, grid, dim3(256), SMEM_BYTES, s, m, (const T*)qkv, ldqkv, (T*)ctx, seq, H,
                  causal ? 1 : 0, scale_log2);
  };
  if (dtype == DP_BF16)
    go(__nv_bfloat16{});
  else
    go(__half{});
  DP_CUDA(cudaGetLastError());
}

}  // namespace dp
