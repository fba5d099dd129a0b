// K5t: attention core on the 5th-generation tensor cores (tcgen05 + TMEM + TMA), d = 64.
//
//   ctx[q, h*64 : h*64+64] = softmax(q_h k_h^T / 8 [+ causal mask]) v_h
//
// One CTA (128 threads) per (head, 128-query tile, sequence).  Per 128-key tile j:
//   1. S = Q K_j^T on tcgen05 (M = 128 queries, N = 128 keys, K = 64), fp32 in TMEM columns
//      [0, 128); Q and K_j arrive by TMA (128-byte swizzle), K double-buffered;
//   2. thread r owns query row r = TMEM lane r: it reads its whole row of S (tcgen05.ld), masks,
//      and runs the online softmax in fp32 with exp2 (no shuffles: the row is in one thread);
//      the numerators P (storage type) go to shared memory as the next MMA's A operand, written
//      in the 128-byte-swizzled K-major layout by hand; V_j (loaded to registers under step 1) is
//      written transposed (V_j^T: d rows, keys along K) as the B operand;
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
constexpr uint32_t VT_BYTES = TD * TK * 2;     // 16 KB: two [64][64] swizzled K-blocks
constexpr uint32_t SMEM_BYTES = Q_BYTES + 2 * K_BYTES + P_BYTES + VT_BYTES + 1024;

// byte offset of element (r, k) of a K-major [rows][64] tile with the 128-byte swizzle
__device__ __forceinline__ uint32_t sw128_off(int r, int k) {
  return uint32_t(r) * 128u + ((uint32_t((k >> 3) ^ (r & 7))) << 4) + uint32_t(k & 7) * 2u;
}

template <class T>
__global__ void __launch_bounds__(128, 1)
    attention_tc_kernel(const __grid_constant__ CUtensorMap tmQK, const T* __restrict__ qkv, int ldqkv,
                        T* __restrict__ ctx, int seq, int H, int causal, float scale_log2) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  uint8_t* sQ = smem;
  uint8_t* sK = sQ + Q_BYTES;           // [2][TK][64]
  uint8_t* sP = sK + 2 * K_BYTES;       // [2 k-blocks][TQ][64]
  uint8_t* sVt = sP + P_BYTES;          // [2 k-blocks][TD][64]
  __shared__ __align__(8) uint64_t bar_q, bar_k[2], bar_s, bar_o;
  __shared__ uint32_t tmem_base_sh;
  // kind::f16, fp32 accumulate, A/B K-major; S: M 128 x N 128; O: M 128 x N 64
  constexpr uint32_t IDESC_S = (1u << 4) | (FmtBits<T>::v << 7) | (FmtBits<T>::v << 10) | (uint32_t(TK >> 3) << 17) |
                               (uint32_t(TQ >> 4) << 24);
  constexpr uint32_t IDESC_O = (1u << 4) | (FmtBits<T>::v << 7) | (FmtBits<T>::v << 10) | (uint32_t(TD >> 3) << 17) |
                               (uint32_t(TQ >> 4) << 24);

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
    mbar_init(&bar_s, 1);
    mbar_init(&bar_o, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&tmem_base_sh)),
                 "r"(256));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tmem = tmem_base_sh;
  const uint32_t t_s = tmem, t_o = tmem + 128;
  pdl_trigger();
  pdl_wait();  // q, k, v come from the previous kernel

  const int qcol = head * TD, kcol = H + head * TD;
  const T* vbase = qkv + (size_t)tok0 * ldqkv + 2 * H + head * TD;
  if (tid == 0) {
    mbar_expect_tx(&bar_q, Q_BYTES);
    tma_load_2d(&tmQK, &bar_q, sQ, qcol, tok0 + q0);
    mbar_expect_tx(&bar_k[0], K_BYTES);
    tma_load_2d(&tmQK, &bar_k[0], sK, kcol, tok0);
  }
  const int r = warp * 32 + lane;  // query row of this thread (TMEM lane)
  const int qrow = q0 + r;
  float o[TD];
#pragma unroll
  for (int d = 0; d < TD; ++d) o[d] = 0.f;
  float mrow = -INFINITY, lrow = 0.f;

  for (int j = 0; j < nkt; ++j) {
    const int k0 = j * TK;
    // V_j: thread t loads key k0 + t (its 128-byte row) into registers under the S MMA
    uint4 vr[8];
    {
      const bool ok = k0 + tid < seq;
      const uint4* src = reinterpret_cast<const uint4*>(vbase + (size_t)(ok ? k0 + tid : 0) * ldqkv);
#pragma unroll
      for (int c = 0; c < 8; ++c) vr[c] = ok ? src[c] : make_uint4(0, 0, 0, 0);
    }
    if (tid == 0) {
      if (j + 1 < nkt) {  // next key tile into the other buffer (its last reader, S_{j-1}, is done)
        mbar_expect_tx(&bar_k[(j + 1) & 1], K_BYTES);
        tma_load_2d(&tmQK, &bar_k[(j + 1) & 1], sK + ((j + 1) & 1) * K_BYTES, kcol, tok0 + k0 + TK);
      }
      if (j == 0) mbar_wait(&bar_q, 0);
      mbar_wait(&bar_k[j & 1], (j >> 1) & 1);
      asm volatile("tcgen05.fence::after_thread_sync;");
      const uint64_t dq = sw128_desc(sQ), dk = sw128_desc(sK + (j & 1) * K_BYTES);
#pragma unroll
      for (int kk = 0; kk < TD / 16; ++kk) umma_f16(t_s, dq + 2 * kk, dk + 2 * kk, IDESC_S, kk != 0);
      umma_commit(&bar_s);
    }
    // V_j^T into the B-operand tile: element (d, key t) of K-block t / 64
    {
      uint8_t* vt = sVt + (tid >> 6) * (TD * 64 * 2);
      const int kk = tid & 63;
#pragma unroll
      for (int c = 0; c < 8; ++c) {
        const uint32_t w4[4] = {vr[c].x, vr[c].y, vr[c].z, vr[c].w};
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          const int d = c * 8 + e * 2;
          *reinterpret_cast<uint16_t*>(vt + sw128_off(d, kk)) = uint16_t(w4[e] & 0xFFFFu);
          *reinterpret_cast<uint16_t*>(vt + sw128_off(d + 1, kk)) = uint16_t(w4[e] >> 16);
        }
      }
    }
    // S row -> online softmax -> P row (one thread spins on the MMA, the CTA barrier releases all)
    if (tid == 0) mbar_wait_spin(&bar_s, j & 1);
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;");
    float s[TK];
    {
      uint32_t v[TK];  // all 8 loads in flight, one completion wait
#pragma unroll
      for (int c = 0; c < TK; c += 16) tmem_ld16_nowait(t_s + (uint32_t(warp * 32) << 16) + c, v + c);
      tmem_ld_wait();
#pragma unroll
      for (int e = 0; e < TK; ++e) s[e] = __uint_as_float(v[e]) * scale_log2;
    }
    // masking only where a key can be invalid: the sequence's last tile, or the causal diagonal
    if (k0 + TK > seq || (causal && k0 + TK - 1 > q0)) {
#pragma unroll
      for (int e = 0; e < TK; ++e) {
        const int key = k0 + e;
        if (key >= seq || (causal && key > qrow)) s[e] = -INFINITY;
      }
    }
    float mx = -INFINITY;
#pragma unroll
    for (int e = 0; e < TK; ++e) mx = fmaxf(mx, s[e]);
    const float mnew = fmaxf(mrow, mx);
    const float corr = (mrow == -INFINITY) ? 0.f : exp2f(mrow - mnew);
    float rs = 0.f;
#pragma unroll
    for (int e = 0; e < TK; e += 2) {
      const float p0 = (mnew == -INFINITY) ? 0.f : exp2f(s[e] - mnew);
      const float p1 = (mnew == -INFINITY) ? 0.f : exp2f(s[e + 1] - mnew);
      rs += p0 + p1;
      s[e] = p0;
      s[e + 1] = p1;
    }
    lrow = lrow * corr + rs;
    mrow = mnew;
#pragma unroll
    for (int kb = 0; kb < 2; ++kb) {  // P row r into K-blocks kb (keys 64 kb .. 64 kb + 63)
      uint8_t* pt = sP + kb * (TQ * 64 * 2);
#pragma unroll
      for (int c = 0; c < 8; ++c) {
        const float* pp = s + kb * 64 + c * 8;
        uint4 u;
        u.x = Cvt<T>::from2(pp[0], pp[1]);
        u.y = Cvt<T>::from2(pp[2], pp[3]);
        u.z = Cvt<T>::from2(pp[4], pp[5]);
        u.w = Cvt<T>::from2(pp[6], pp[7]);
        *reinterpret_cast<uint4*>(pt + sw128_off(r, c * 8)) = u;
      }
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // P, V^T -> the tensor core
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    if (tid == 0) {
      asm volatile("tcgen05.fence::after_thread_sync;");
#pragma unroll
      for (int kb = 0; kb < 2; ++kb) {
        const uint64_t dp_ = sw128_desc(sP + kb * (TQ * 64 * 2)), dv = sw128_desc(sVt + kb * (TD * 64 * 2));
#pragma unroll
        for (int kk = 0; kk < 4; ++kk) umma_f16(t_o, dp_ + 2 * kk, dv + 2 * kk, IDESC_O, (kb | kk) != 0);
      }
      umma_commit(&bar_o);
    }
    if (tid == 0) mbar_wait_spin(&bar_o, j & 1);
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;");
    {
      uint32_t v[TD];
#pragma unroll
      for (int c = 0; c < TD; c += 16) tmem_ld16_nowait(t_o + (uint32_t(warp * 32) << 16) + c, v + c);
      tmem_ld_wait();
#pragma unroll
      for (int e = 0; e < TD; ++e) o[e] = o[e] * corr + __uint_as_float(v[e]);
    }
    // every thread has read S and O_j before the next tile's MMAs overwrite them
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;");
  }
  if (qrow < seq) {
    const float inv = lrow > 0.f ? 1.f / lrow : 0.f;
    uint4* dst = reinterpret_cast<uint4*>(ctx + (size_t)(tok0 + qrow) * H + head * TD);
#pragma unroll
    for (int c = 0; c < 8; ++c) {
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
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(256));
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
    launch_kernel(attention_tc_kernel<T>, grid, dim3(128), SMEM_BYTES, s, m, (const T*)qkv, ldqkv, (T*)ctx, seq, H,
                  causal ? 1 : 0, scale_log2);
  };
  if (dtype == DP_BF16)
    go(__nv_bfloat16{});
  else
    go(__half{});
  DP_CUDA(cudaGetLastError());
}

}  // namespace dp
