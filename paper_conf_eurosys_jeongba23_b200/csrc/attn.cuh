// Shared device code: cp.async helpers and the flash-attention tile (K5) used by the
// standalone attention kernel (kernels.cu) and the persistent layer-program kernel (persist.cu).
//
// Attention tile, flash-style, d = 64: (64 query rows, head, sequence) on 4 warps x 16 rows;
// K/V tiles of 64 keys in padded shared memory; S = Q K^T and O += P V on mma.sync m16n8k16
// (fp32 accumulate), online softmax in fp32 with exp2.  `sync` is the barrier of the 128
// participating threads (__syncthreads in the standalone kernel, a named barrier in K6).
#pragma once
#include <cuda_runtime.h>

#include <cstdint>

#include "dtype.cuh"

namespace dp {

// cp.async (global -> shared, 16 bytes, bypassing L1); the zero-fill form writes zeros when
// !valid (src is not read)
__device__ __forceinline__ void cp_async16(void* dst, const void* src) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(static_cast<uint32_t>(__cvta_generic_to_shared(dst))),
               "l"(src)
               : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() {
  asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory");
}
__device__ __forceinline__ void cp_async16_zfill(void* dst, const void* src, bool valid) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(static_cast<uint32_t>(__cvta_generic_to_shared(dst))),
               "l"(src), "r"(valid ? 16 : 0)
               : "memory");
}

template <class T>
struct MmaOp;
template <>
struct MmaOp<__half> {
  static __device__ __forceinline__ void mma(float* c, const uint32_t* a, const uint32_t* b) {
    asm volatile(
        "mma.sync.aligned.m16n8k16.row.col.f32.f16.f16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
        "{%0,%1,%2,%3};"
        : "+f"(c[0]), "+f"(c[1]), "+f"(c[2]), "+f"(c[3])
        : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b[0]), "r"(b[1]));
  }
};
template <>
struct MmaOp<__nv_bfloat16> {
  static __device__ __forceinline__ void mma(float* c, const uint32_t* a, const uint32_t* b) {
    asm volatile(
        "mma.sync.aligned.m16n8k16.row.col.f32.bf16.bf16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
        "{%0,%1,%2,%3};"
        : "+f"(c[0]), "+f"(c[1]), "+f"(c[2]), "+f"(c[3])
        : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b[0]), "r"(b[1]));
  }
};

__device__ __forceinline__ void ldsm_x4(uint32_t* r, const void* p) {
  const uint32_t a = static_cast<uint32_t>(__cvta_generic_to_shared(p));
  asm volatile("ldmatrix.sync.aligned.m8n8.x4.shared.b16 {%0,%1,%2,%3}, [%4];"
               : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3])
               : "r"(a));
}
__device__ __forceinline__ void ldsm_x4_t(uint32_t* r, const void* p) {
  const uint32_t a = static_cast<uint32_t>(__cvta_generic_to_shared(p));
  asm volatile("ldmatrix.sync.aligned.m8n8.x4.trans.shared.b16 {%0,%1,%2,%3}, [%4];"
               : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3])
               : "r"(a));
}

constexpr int ATT_D = 64, ATT_BQ = 64, ATT_BK = 64, ATT_LD = 72;  // padded row (144 B): no ldmatrix conflicts

// One key tile of the online-softmax flash step for one warp's 16 query rows (rows qrow0 and
// qrow0 + 8 per lane): S = Q K^T, mask, running max / sum, O = O * corr + P V.
template <class T>
__device__ __forceinline__ void attention_key_tile(const T* skt, const T* svt, const uint32_t (&qa)[4][4],
                                                   float (&o)[8][4], float (&mrow)[2], float (&lrow)[2], int k0,
                                                   int qrow0, int seq, int causal, float scale_log2, int lane) {
    float s[8][4];
#pragma unroll
    for (int nb = 0; nb < 8; ++nb) s[nb][0] = s[nb][1] = s[nb][2] = s[nb][3] = 0.f;
#pragma unroll
    for (int kk = 0; kk < 4; ++kk) {
#pragma unroll
      for (int nb = 0; nb < 8; nb += 2) {
        uint32_t bfr[4];
        const int key = nb * 8 + (lane & 7) + (lane >> 4) * 8;
        ldsm_x4(bfr, &skt[key * ATT_LD + kk * 16 + ((lane >> 3) & 1) * 8]);
        MmaOp<T>::mma(s[nb], qa[kk], bfr);
        MmaOp<T>::mma(s[nb + 1], qa[kk], bfr + 2);
      }
    }
    // mask + online softmax (rows qrow0, qrow0+8; each row spread over 4 lanes).  Scores stay
    // unscaled until the exponent: p = exp2(s * scale_log2 - m) is one FFMA + MUFU per element.
    // Only the sequence's last key tile and the causal diagonal need the mask (the warp's rows
    // start at qrow0 - lane / 4); the running max is kept in scaled units.
    const bool need_mask = k0 + 64 > seq || (causal && k0 + 63 > qrow0 - (lane >> 2));
    if (need_mask) {
#pragma unroll
      for (int nb = 0; nb < 8; ++nb) {
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          const int key = k0 + nb * 8 + (lane & 3) * 2 + (e & 1);
          const int qr = qrow0 + (e >> 1) * 8;
          if (key >= seq || (causal && key > qr)) s[nb][e] = -INFINITY;
        }
      }
    }
    float mx[2] = {-INFINITY, -INFINITY};
#pragma unroll
    for (int nb = 0; nb < 8; ++nb) {
      mx[0] = fmaxf(mx[0], fmaxf(s[nb][0], s[nb][1]));
      mx[1] = fmaxf(mx[1], fmaxf(s[nb][2], s[nb][3]));
    }
    float corr[2], mref[2];
#pragma unroll
    for (int h = 0; h < 2; ++h) {
      mx[h] = fmaxf(mx[h], __shfl_xor_sync(0xffffffffu, mx[h], 1));
      mx[h] = fmaxf(mx[h], __shfl_xor_sync(0xffffffffu, mx[h], 2));
      const float mnew = fmaxf(mrow[h], mx[h] * scale_log2);
      corr[h] = (mrow[h] == -INFINITY) ? 0.f : fast_exp2(mrow[h] - mnew);
      mrow[h] = mnew;
      mref[h] = (mnew == -INFINITY) ? 0.f : mnew;  // a fully masked row: every p is exp2(-inf) = 0
    }
    float rs[2] = {0.f, 0.f};
#pragma unroll
    for (int nb = 0; nb < 8; ++nb) {
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        const int h = e >> 1;
        const float p = fast_exp2(fmaf(s[nb][e], scale_log2, -mref[h]));
        s[nb][e] = p;
        rs[h] += p;
      }
    }
#pragma unroll
    for (int h = 0; h < 2; ++h) lrow[h] = lrow[h] * corr[h] + rs[h];  // per-lane partial sums
#pragma unroll
    for (int db = 0; db < 8; ++db) {
      o[db][0] *= corr[0];
      o[db][1] *= corr[0];
      o[db][2] *= corr[1];
      o[db][3] *= corr[1];
    }
    // O += P V : P from registers as A fragments (keys = k dimension)
#pragma unroll
    for (int kk = 0; kk < 4; ++kk) {
      uint32_t pa[4];
      pa[0] = Cvt<T>::from2(s[2 * kk][0], s[2 * kk][1]);
      pa[1] = Cvt<T>::from2(s[2 * kk][2], s[2 * kk][3]);
      pa[2] = Cvt<T>::from2(s[2 * kk + 1][0], s[2 * kk + 1][1]);
      pa[3] = Cvt<T>::from2(s[2 * kk + 1][2], s[2 * kk + 1][3]);
#pragma unroll
      for (int db = 0; db < 8; db += 2) {
        uint32_t bfr[4];
        const int key = kk * 16 + (lane & 7) + ((lane >> 3) & 1) * 8;
        ldsm_x4_t(bfr, &svt[key * ATT_LD + (db + (lane >> 4)) * 8]);
        MmaOp<T>::mma(o[db], pa, bfr);
        MmaOp<T>::mma(o[db + 1], pa, bfr + 2);
      }
    }
}

template <class T, class Sync>
__device__ __forceinline__ void attention_tile(const T* __restrict__ qkv, int ldqkv, T* __restrict__ ctx, int seq,
                                               int H, int causal, float scale_log2, int qt, int head, int bidx,
                                               T* sq, T* sk_, T* sv_, int tid, Sync sync) {
  // Q tile + a 2-deep ring of (K, V) tiles, all filled with cp.async: the Q tile and the
  // first two key tiles are in flight together (one L2 round trip, not one per tile), and
  // tile kt+2 streams in while tile kt is computed.  Rows past `seq` are zero-filled.
  T* sk[2] = {sk_, sk_ + ATT_BK * ATT_LD};
  T* sv[2] = {sv_, sv_ + ATT_BK * ATT_LD};
  const int lane = tid & 31, warp = tid >> 5;
  sync();  // the previous tile's readers are done with the buffers
  const size_t tok0 = (size_t)bidx * seq;
  const int q0 = qt * ATT_BQ;
  const T* qbase = qkv + tok0 * ldqkv + head * ATT_D;
  const T* kbase = qbase + H;
  const T* vbase = qbase + 2 * H;
  int nkt = (seq + ATT_BK - 1) / ATT_BK;
  if (causal) nkt = min(nkt, (q0 + ATT_BQ - 1) / ATT_BK + 1);
  auto load_kv = [&](int kt) {
    const int k0 = kt * ATT_BK;
    for (int i = tid; i < ATT_BK * 8; i += 128) {
      const int r = i >> 3, c = i & 7;
      const bool ok = k0 + r < seq;
      const size_t off = (size_t)(ok ? k0 + r : 0) * ldqkv + c * 8;
      cp_async16_zfill(&sk[kt & 1][r * ATT_LD + c * 8], kbase + off, ok);
      cp_async16_zfill(&sv[kt & 1][r * ATT_LD + c * 8], vbase + off, ok);
    }
  };
  for (int i = tid; i < ATT_BQ * 8; i += 128) {  // Q: 64 rows x 64 d = 512 vectors of 16 B
    const int r = i >> 3, c = i & 7;
    const bool ok = q0 + r < seq;
    cp_async16_zfill(&sq[r * ATT_LD + c * 8], qbase + (size_t)(ok ? q0 + r : 0) * ldqkv + c * 8, ok);
  }
  load_kv(0);
  cp_async_commit();
  if (nkt > 1) load_kv(1);
  cp_async_commit();
  cp_async_wait<1>();
  sync();
  uint32_t qa[4][4];  // A fragments: 16 rows of this warp x 64 d (4 k-steps)
  {
    const int r = warp * 16 + (lane & 7) + ((lane >> 3) & 1) * 8;
#pragma unroll
    for (int kk = 0; kk < 4; ++kk) ldsm_x4(qa[kk], &sq[r * ATT_LD + kk * 16 + (lane >> 4) * 8]);
  }
  float o[8][4];
#pragma unroll
  for (int i = 0; i < 8; ++i) o[i][0] = o[i][1] = o[i][2] = o[i][3] = 0.f;
  float mrow[2] = {-INFINITY, -INFINITY}, lrow[2] = {0.f, 0.f};
  const int qrow0 = q0 + warp * 16 + (lane >> 2);  // rows qrow0 and qrow0 + 8
  for (int kt = 0; kt < nkt; ++kt) {
    const int k0 = kt * ATT_BK;
    if (kt > 0) {
      cp_async_wait<1>();  // tile kt landed (tile kt+1 may still be in flight)
      sync();
    }
    attention_key_tile<T>(sk[kt & 1], sv[kt & 1], qa, o, mrow, lrow, k0, qrow0, seq, causal, scale_log2, lane);
    if (kt + 2 < nkt) {
      sync();  // every warp is done with slot kt & 1
      load_kv(kt + 2);
    }
    cp_async_commit();
  }
  // finalize: full row sums across the 4 lanes of a row
#pragma unroll
  for (int h = 0; h < 2; ++h) {
    lrow[h] += __shfl_xor_sync(0xffffffffu, lrow[h], 1);
    lrow[h] += __shfl_xor_sync(0xffffffffu, lrow[h], 2);
  }
  const float inv0 = lrow[0] > 0.f ? 1.f / lrow[0] : 0.f, inv1 = lrow[1] > 0.f ? 1.f / lrow[1] : 0.f;
  T* cbase = ctx + tok0 * H + head * ATT_D;
#pragma unroll
  for (int db = 0; db < 8; ++db) {
    const int col = db * 8 + (lane & 3) * 2;
    if (qrow0 < seq)
      *reinterpret_cast<uint32_t*>(cbase + (size_t)qrow0 * H + col) = Cvt<T>::from2(o[db][0] * inv0, o[db][1] * inv0);
    if (qrow0 + 8 < seq)
      *reinterpret_cast<uint32_t*>(cbase + (size_t)(qrow0 + 8) * H + col) =
          Cvt<T>::from2(o[db][2] * inv1, o[db][3] * inv1);
  }
}

}  // namespace dp
