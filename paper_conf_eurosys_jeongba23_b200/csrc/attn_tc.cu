// K5t: attention core on the 5th-generation tensor cores (tcgen05 + TMEM + TMA), d = 64.
//
//   ctx[q, h*64 : h*64+64] = softmax(q_h k_h^T / 8 [+ causal mask]) v_h
//
// One CTA (320 threads, warp-specialised) per (head, 128-query tile, sequence); keys in tiles of
// 64.  The key tiles alternate between two softmax warpgroups, each with its own running row
// max / sum / output (merged once at the end, like K5b's key-tile groups), so two independent
// softmax chains share the SM while the tensor core serves both:
//   warp 8 (one lane)  : TMA -- Q once, then K_j / V_j into a 4-stage ring;
//   warp 9 (one lane)  : tcgen05.mma -- S_j = Q K_j^T (M 128, N 64, K 64) into the owning
//                        group's TMEM S buffer (two per group: S_{j+2} is computed while the
//                        group works on S_j), and O_g += P_j V_j (M 128, N 64, K 64 keys) into
//                        the group's TMEM accumulator once the group has published P_j;
//   warps 0-3 / 4-7    : group g = even / odd key tiles; thread r owns query row r (TMEM lane
//                        r): it reads its 64 scores (tcgen05.ld), masks, runs the online
//                        softmax in fp32 with exp2 and writes the numerators P (storage type, two
//                        per column) back over its S row (tcgen05.st): P V takes A from TMEM.
// MUFU (16 exponentials per clock per SM, profiles/r02_mufu_probe.txt) bounds the softmax: the
// two groups' exponentials run at ~12 per clock per SM (profiles/r02_attn_tc_trace.jsonl).
// Measured and dropped: the groups taking strict turns on the exponentials (named barriers), and
// a quarter / half of the exponentials as a degree-3 polynomial on the FMA pipe (both slower).
// The softmax reference max of a row moves only when the row max grows by more than 2^8 (then
// the thread rescales its O row in TMEM, tcgen05.ld / st, and its row sum): between moves the
// numerators stay <= 2^8, so the O accumulator never leaves TMEM (no per-tile correction pass).
// V_j lands as [keys][head dims] and is the MN-major B operand as is (no transpose).  TMEM: three S
// buffers per group in columns [0, 384), the two O accumulators in [384, 512).  Arithmetic contract: S and
// O in fp32, P rounded to the storage type before P V (as the mma.sync K5), row sums in fp32.
#include <cuda.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstring>
#include <type_traits>

#include "common.h"
#include "dtype.cuh"
#include "kernels.h"
#include "launch.cuh"
#include "tc.cuh"

namespace dp {

namespace {

#ifdef DP_ATT_TRACE
// per-CTA globaltimer stamps (tools/att_trace.py): 0 entry, 1 after setup + PDL wait, 2 / 3 group
// 0 / 1 first scores read, 4 / 5 group 0 / 1 last P published, 6 / 7 group 0 / 1 accumulator
// read, 8 stored, 9 MMA warp done issuing, 10 loader done issuing; [15] = key tiles
__device__ unsigned long long g_att_trace[2048][64];
#define ATRACE(i)                                                                                \
  do {                                                                                           \
    unsigned long long t_;                                                                       \
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_));                                       \
    const int b_ = (blockIdx.z * gridDim.y + blockIdx.y) * gridDim.x + blockIdx.x;               \
    if (b_ < 2048 && (i) < 64) g_att_trace[b_][i] = t_;                                          \
  } while (0)
#else
#define ATRACE(i) \
  do {            \
  } while (0)
#endif

constexpr int TQ = 128;  // queries per CTA (MMA M, TMEM lanes)
constexpr int TK = 64;   // keys per tile (MMA N of S, K of P V)
constexpr int TD = 64;   // head dim
constexpr int NS = 6;    // stages of the K ring and of the V ring
constexpr int SB = 3;    // TMEM S buffers per softmax group
constexpr uint32_t Q_BYTES = TQ * TD * 2;   // 16 KB
constexpr uint32_t KV_BYTES = TK * TD * 2;  // 8 KB each for K_j and V_j
constexpr uint32_t MERGE_BYTES = TQ * 68 * 4;  // group 1's (o[64], m, l) per row
constexpr uint32_t SMEM_BYTES = Q_BYTES + 2 * NS * KV_BYTES + MERGE_BYTES + 1024;
constexpr int NTHR = 352;  // 8 softmax warps, the TMA warp, two MMA warps


// One lane polls the barrier and releases its warp: 256 softmax threads polling the same
// barriers flooded the shared-memory barrier unit and delayed the MMA warp's own polls.
__device__ __forceinline__ void warp_wait(uint64_t* bar, uint32_t phase) {
  if ((threadIdx.x & 31) == 0) mbar_wait(bar, phase);
  __syncwarp();
}

__device__ __forceinline__ void named_sync(int id, int n) {
  asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(n) : "memory");
}


// CAUSAL and SPLIT (nsplit > 1) are compile-time: each variant carries only its masking and
// merge code (a CTA runs its code once; cold instruction fetch is on its critical path).
template <class T, bool CAUSAL, bool SPLIT>
__global__ void __launch_bounds__(NTHR, 1)
    attention_tc_kernel(const __grid_constant__ CUtensorMap tmQ, const __grid_constant__ CUtensorMap tmKV,
                        T* __restrict__ ctx, int seq, int H, float scale_log2, int nsplit_rt) {
  constexpr bool causal = CAUSAL;
  const int nsplit = SPLIT ? nsplit_rt : 1;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  uint8_t* sQ = smem;
  uint8_t* sK = sQ + Q_BYTES;               // [NS][64 keys][64]: freed by S_j
  uint8_t* sV = sK + NS * KV_BYTES;         // [NS][64 keys][64]: freed by P_j V_j
  float* xs = reinterpret_cast<float*>(sV + NS * KV_BYTES);  // [128][68]
  __shared__ __align__(8) uint64_t bar_q, k_full[NS], k_empty[NS], v_full[NS], v_empty[NS], s_full[2][SB], p_full[2][SB],
      o_full[2][2], recv_bar;
  __shared__ uint32_t tmem_base_sh;
  // kind::f16, fp32 accumulate; S: A = Q, B = K_j both K-major, M 128 x N 64
  constexpr uint32_t IDESC_S = (1u << 4) | (FmtBits<T>::v << 7) | (FmtBits<T>::v << 10) | (uint32_t(TK >> 3) << 17) |
                               (uint32_t(TQ >> 4) << 24);
  // O: A = P K-major, B = V_j MN-major (head dims contiguous, keys along K): transpose-B bit 16
  constexpr uint32_t IDESC_O = (1u << 4) | (FmtBits<T>::v << 7) | (FmtBits<T>::v << 10) | (1u << 16) |
                               (uint32_t(TD >> 3) << 17) | (uint32_t(TQ >> 4) << 24);

  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  if (tid == 0) ATRACE(0);
  // grid (heads, query tiles x nsplit, batch); causal query tiles longest first.  With nsplit > 1
  // the nsplit CTAs of a query tile form a cluster along y and take consecutive key ranges
  // (split = cluster rank); their partial (o, m, l) rows are merged over DSMEM at the end.
  const int head = blockIdx.x, bidx = blockIdx.z;
  const int qidx = (int)blockIdx.y / nsplit, split = (int)blockIdx.y - qidx * nsplit;
  const int nqt = (int)gridDim.y / nsplit;
  const int qt = causal ? nqt - 1 - qidx : qidx;
  const int q0 = qt * TQ;
  const int tok0 = bidx * seq;
  int nkt_all = (seq + TK - 1) / TK;
  if (causal) nkt_all = min(nkt_all, (q0 + TQ - 1) / TK + 1);
  const int kt_lo = split * nkt_all / nsplit;                // this CTA's key tiles [kt_lo, kt_lo + nkt)
  const int nkt = (split + 1) * nkt_all / nsplit - kt_lo;

  if (tid == 0) {
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&tmQ)) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&tmKV)) : "memory");
    mbar_init(&bar_q, 1);
    mbar_init(&recv_bar, 1);  // cluster merge: the peers' partial rows (bulk DSMEM pushes) land here
    for (int i = 0; i < NS; ++i) {
      mbar_init(&k_full[i], 1);
      mbar_init(&k_empty[i], 1);
      mbar_init(&v_full[i], 1);
      mbar_init(&v_empty[i], 1);
    }
    for (int g = 0; g < 2; ++g) {
      for (int b = 0; b < 2; ++b) mbar_init(&o_full[g][b], 1);
      for (int b = 0; b < SB; ++b) {
        mbar_init(&s_full[g][b], 1);
        mbar_init(&p_full[g][b], 4);  // one arrival per warp of the group
      }
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 9) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&tmem_base_sh)),
                 "r"(512));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tmem = tmem_base_sh;
  auto t_s = [&](int g, int b) { return tmem + 64u * uint32_t(SB * g + b); };
  auto t_o = [&](int g) { return tmem + 64u * uint32_t(2 * SB + g); };
  pdl_trigger();
  pdl_wait();  // q, k, v come from the previous kernel
  if (tid == 0) ATRACE(1);
#ifdef DP_ATT_TRACE
  if (tid == 0) {
    const int b_ = (blockIdx.z * gridDim.y + blockIdx.y) * gridDim.x + blockIdx.x;
    if (b_ < 2048) g_att_trace[b_][15] = (unsigned long long)nkt;
  }
#endif

  const int qcol = head * TD, kcol = H + head * TD, vcol = 2 * H + head * TD;
  if (warp == 8) {
    // TMA producer: Q, then K_j and V_j in key order into their rings (a K stage is free once
    // S_j is done, a V stage once P_j V_j is done)
    if (lane == 0) {
      mbar_expect_tx(&bar_q, Q_BYTES);
      tma_load_2d(&tmQ, &bar_q, sQ, qcol, tok0 + q0);
      for (int j = 0; j < nkt; ++j) {  // j: local key tile (absolute kt_lo + j)
        const int st = j % NS;
        if (j >= NS) mbar_wait(&k_empty[st], ((j / NS) - 1) & 1);
        mbar_expect_tx(&k_full[st], KV_BYTES);
        tma_load_2d(&tmKV, &k_full[st], sK + st * KV_BYTES, kcol, tok0 + (kt_lo + j) * TK);
        if (j >= NS) mbar_wait(&v_empty[st], ((j / NS) - 1) & 1);
        mbar_expect_tx(&v_full[st], KV_BYTES);
        tma_load_2d(&tmKV, &v_full[st], sV + st * KV_BYTES, vcol, tok0 + (kt_lo + j) * TK);
      }
      ATRACE(10);
    }
  } else if (warp >= 9) {
    // MMA issuers, one thread per softmax group (warp 9: group 0, warp 10: group 1), each in its
    // group's order: S_0, S_1, then P_i V_i and S_{i+2} as P_i is published and S_i's buffer is
    // read.  One issuer alternating between the groups could not keep up: a tcgen05.mma issue costs
    // ~80 cycles and a commit ~50 (profiles/r02_attn_tc_trace.jsonl), against ~0.5 us of softmax
    // per 64-key tile.
    if (lane == 0) {
      const int g = warp - 9;
      mbar_wait(&bar_q, 0);
      const uint64_t dq = sw128_desc(sQ);
      const int nl = (nkt - g + 1) / 2;
      auto issue_s = [&](int i) {
        const int j = 2 * i + g, b = i % SB, st = j % NS;
        if (j < 8) ATRACE(56 + j);
        mbar_wait(&k_full[st], (j / NS) & 1);
        // (S buffer b held P_{i-SB}: this MMA executes after that tile's P V, issued before it)
        asm volatile("tcgen05.fence::after_thread_sync;");
        const uint64_t dk = sw128_desc(sK + st * KV_BYTES);
#pragma unroll
        for (int kk = 0; kk < TD / 16; ++kk) umma_f16(t_s(g, b), dq + 2 * kk, dk + 2 * kk, IDESC_S, kk != 0);
        umma_commit(&s_full[g][b]);
        umma_commit(&k_empty[st]);  // K_j consumed
      };
      auto issue_pv = [&](int i) {
        const int j = 2 * i + g, b = i & 1, sb = i % SB, st = j % NS;
        mbar_wait(&p_full[g][sb], (i / SB) & 1);
        mbar_wait(&v_full[st], (j / NS) & 1);
        asm volatile("tcgen05.fence::after_thread_sync;");
        // A = P_j from TMEM (the S buffer's first 32 columns: 2 numerators per column, a 16-key
        // step = 8 columns); B = V_j as the MN-major operand: 128-byte swizzle atoms of 8 keys x 64
        // head dims, 1024 B apart along K (SBO), a 16-key step = 2048 B (128 in descriptor units)
        const uint64_t dv = sw128_desc(sV + st * KV_BYTES);
#pragma unroll
        for (int kk = 0; kk < TK / 16; ++kk)
          umma_f16_ts(t_o(g), t_s(g, sb) + 8 * kk, dv + 128 * kk, IDESC_O, (i | kk) != 0);
        umma_commit(&o_full[g][b]);  // O holds tiles <= j
        umma_commit(&v_empty[st]);   // V_j consumed
      };
      for (int i = 0; i < nl && i < SB; ++i) issue_s(i);
      for (int i = 0; i < nl; ++i) {
        issue_pv(i);
        if (i + SB < nl) issue_s(i + SB);
      }
      if (g == 0) ATRACE(9);
    }
  } else {
    // softmax group g = warp / 4: key tiles g, g + 2, g + 4, ...; thread r = query row r
    const int g = warp >> 2, r = (warp & 3) * 32 + lane;
    const uint32_t lane_base = uint32_t((warp & 3) * 32) << 16;
    const int qrow = q0 + r;
    float mref = -INFINITY, lrow = 0.f;  // the row's softmax reference max (scaled units) and sum
    const int nloc = (nkt - g + 1) / 2;
    for (int i = 0; i < nloc; ++i) {
      const int j = 2 * i + g, b = i & 1, sb = i % SB, k0 = (kt_lo + j) * TK;
      warp_wait(&s_full[g][sb], (i / SB) & 1);
      if (tid == 0 && i < 8) ATRACE(16 + 4 * i);
      asm volatile("tcgen05.fence::after_thread_sync;");
      float s[TK];
      {
        uint32_t v[TK];
#pragma unroll
        for (int c = 0; c < TK; c += 16) tmem_ld16_nowait(t_s(g, sb) + lane_base + c, v + c);
        tmem_ld_wait();
#pragma unroll
        for (int e = 0; e < TK; ++e) s[e] = __uint_as_float(v[e]);  // scaled inside the exponent
      }
      if (tid == 0 && i < 8) ATRACE(17 + 4 * i);
      if (i == 0 && r == 0) ATRACE(2 + g);
      if (r == 0 && j < 8) ATRACE(48 + j);
      if (k0 + TK > seq || (causal && k0 + TK - 1 > qrow)) {  // only where a key can be invalid
#pragma unroll
        for (int e = 0; e < TK; ++e) {
          const int key = k0 + e;
          if (key >= seq || (causal && key > qrow)) s[e] = -INFINITY;
        }
      }
      float mx;
      {  // 8 independent chains, not one 64-long dependency chain
        float m8[8];
#pragma unroll
        for (int q = 0; q < 8; ++q) m8[q] = s[q];
#pragma unroll
        for (int e = 8; e < TK; ++e) m8[e & 7] = fmaxf(m8[e & 7], s[e]);
        mx = fmaxf(fmaxf(fmaxf(m8[0], m8[1]), fmaxf(m8[2], m8[3])), fmaxf(fmaxf(m8[4], m8[5]), fmaxf(m8[6], m8[7])));
      }
      mx *= scale_log2;
      // P V of tile i - 2 has completed: each O barrier is then at most one phase behind, so the
      // parity wait for tile i - 1 below (and the next iteration's) is unambiguous
      if (i >= 2) warp_wait(&o_full[g][i & 1], ((i - 2) >> 1) & 1);
      // move the reference only when the row max outgrows it by > 2^8 (or on the first finite max);
      // O and the row sum then scale by f = 2^(old - new)
      float f = 1.f;
      const bool move = mx > mref + 8.f;
      if (move) {
        f = (mref == -INFINITY) ? 0.f : fast_exp2(mref - mx);
        lrow *= f;
        mref = mx;
      }
      if (i > 0 && __any_sync(0xffffffffu, move)) {  // collective: a lane that keeps its reference scales by 1
        // the group's previous P V (into the O rows being rescaled) has completed
        warp_wait(&o_full[g][(i - 1) & 1], ((i - 1) >> 1) & 1);
        asm volatile("tcgen05.fence::after_thread_sync;");
#pragma unroll
        for (int c = 0; c < TD; c += 16) {
          uint32_t v[16];
          tmem_ld16(t_o(g) + lane_base + c, v);
#pragma unroll
          for (int e = 0; e < 16; ++e) v[e] = __float_as_uint(__uint_as_float(v[e]) * f);
          tmem_st16(t_o(g) + lane_base + c, v);
        }
        asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
      }
      const float mr = (mref == -INFINITY) ? 0.f : mref;  // a fully masked row: every p = 2^-inf = 0
      float r8[8] = {0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f};
#pragma unroll
      for (int e = 0; e < TK; ++e) {
        const float pv = fast_exp2(fmaf(s[e], scale_log2, -mr));
        r8[e & 7] += pv;
        s[e] = pv;
      }
      lrow += ((r8[0] + r8[1]) + (r8[2] + r8[3])) + ((r8[4] + r8[5]) + (r8[6] + r8[7]));
      if (tid == 0 && i < 8) ATRACE(18 + 4 * i);
      // P_j (row r, storage type, 2 per column) over the S row it came from: the A operand of P V
      {
        uint32_t pk[TK / 2];
#pragma unroll
        for (int c = 0; c < TK / 2; ++c) pk[c] = Cvt<T>::from2(s[2 * c], s[2 * c + 1]);
        tmem_st16(t_s(g, sb) + lane_base, pk);
        tmem_st16(t_s(g, sb) + lane_base + 16, pk + 16);
        asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
      }
      asm volatile("tcgen05.fence::before_thread_sync;");
      __syncwarp();
      if (lane == 0) mbar_arrive(&p_full[g][sb]);
      if (tid == 0 && i < 8) ATRACE(19 + 4 * i);
    }
    if (r == 0) ATRACE(4 + g);
    float o[TD];
    if (nloc > 0) {
      warp_wait(&o_full[g][(nloc - 1) & 1], ((nloc - 1) >> 1) & 1);
      asm volatile("tcgen05.fence::after_thread_sync;");
      uint32_t v[TD];
#pragma unroll
      for (int c = 0; c < TD; c += 16) tmem_ld16_nowait(t_o(g) + lane_base + c, v + c);
      tmem_ld_wait();
#pragma unroll
      for (int e = 0; e < TD; ++e) o[e] = __uint_as_float(v[e]);
    } else {
#pragma unroll
      for (int e = 0; e < TD; ++e) o[e] = 0.f;
    }
    const float mrow = mref;
    if (r == 0) ATRACE(6 + g);
    // merge the two groups (group 1 publishes, group 0 combines in a fixed order) and store
    if (g == 1) {
      float* mine = xs + r * 68;
#pragma unroll
      for (int e = 0; e < TD; e += 4) *reinterpret_cast<float4*>(mine + e) = make_float4(o[e], o[e + 1], o[e + 2], o[e + 3]);
      mine[64] = mrow;
      mine[65] = lrow;
    }
    named_sync(1, 256);
    if (g == 0) {
      float* ot = xs + r * 68;
      const float m1 = ot[64], l1 = ot[65];
      const float m = fmaxf(mrow, m1);
      const float a0 = (mrow == -INFINITY) ? 0.f : fast_exp2(mrow - m);
      const float a1 = (m1 == -INFINITY) ? 0.f : fast_exp2(m1 - m);
      const float l = lrow * a0 + l1 * a1;
      if constexpr (!SPLIT) {
        if (qrow < seq) {
          const float inv = l > 0.f ? 1.f / l : 0.f;
          const float c0 = a0 * inv, c1 = a1 * inv;
          uint4* dst = reinterpret_cast<uint4*>(ctx + (size_t)(tok0 + qrow) * H + head * TD);
#pragma unroll
          for (int c = 0; c < TD / 8; ++c) {
            float v[8];
#pragma unroll
            for (int e = 0; e < 8; ++e) v[e] = o[c * 8 + e] * c0 + ot[c * 8 + e] * c1;
            uint4 u;
            u.x = Cvt<T>::from2(v[0], v[1]);
            u.y = Cvt<T>::from2(v[2], v[3]);
            u.z = Cvt<T>::from2(v[4], v[5]);
            u.w = Cvt<T>::from2(v[6], v[7]);
            dst[c] = u;
          }
        }
      } else {
        // this CTA's key range merged: unnormalised o, reference max m, sum l, published in place
        // for the cluster merge below
#pragma unroll
        for (int e = 0; e < TD; e += 4) {
          const float4 t = *reinterpret_cast<const float4*>(ot + e);
          *reinterpret_cast<float4*>(ot + e) =
              make_float4(o[e] * a0 + t.x * a1, o[e + 1] * a0 + t.y * a1, o[e + 2] * a0 + t.z * a1, o[e + 3] * a0 + t.w * a1);
        }
        ot[64] = m;
        ot[65] = l;
      }
    }
    if (tid == 0) ATRACE(8);
  }
  if constexpr (SPLIT) {
    // Cluster merge: the nsplit CTAs of a query tile hold (o, m, l) of consecutive key ranges in
    // their xs rows ([128][68] fp32).  Rank k finalises query rows [k*128/n, (k+1)*128/n): every
    // CTA pushes the rows each peer owns with ONE bulk copy (cp.async.bulk shared::cta ->
    // shared::cluster, completing on the peer's recv_bar) into the peer's K ring -- idle by now:
    // every S MMA finished before the O accumulators were read -- and the owner merges the ranks'
    // rows in rank order from its own shared memory (deterministic).  (Remote loads by the owner
    // instead -- latency-bound ld.shared::cluster -- cost ~3-4 us per CTA, tools/att_waves.py.)
    const int rows_max = (TQ + nsplit - 1) / nsplit;
    const int rlo = split * TQ / nsplit, rhi = (split + 1) * TQ / nsplit;
    float* recv = reinterpret_cast<float*>(sK);  // [nsplit - 1][rows_max][68]
    if (tid == 0)
      asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(&recv_bar)),
                   "r"(uint32_t(nsplit - 1) * uint32_t(rhi - rlo) * 68u * 4u)
                   : "memory");
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // xs rows -> async proxy
    // every rank's rows are final and its K ring and recv_bar are ready
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
    if (tid == 0) {
      ATRACE(11);
      for (int k = 0; k < nsplit; ++k) {
        if (k == split) continue;
        const int klo = k * TQ / nsplit, khi = (k + 1) * TQ / nsplit;
        const int slot = split < k ? split : split - 1;  // this rank's slot in rank k's receive area
        uint32_t dst, bar;
        asm volatile("mapa.shared::cluster.u32 %0, %1, %2;"
                     : "=r"(dst)
                     : "r"(smem_u32(recv + size_t(slot) * rows_max * 68)), "r"(k));
        asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(bar) : "r"(smem_u32(&recv_bar)), "r"(k));
        asm volatile(
            "cp.async.bulk.shared::cluster.shared::cta.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst),
            "r"(smem_u32(xs + klo * 68)), "r"(uint32_t(khi - klo) * 68u * 4u), "r"(bar)
            : "memory");
      }
      asm volatile("cp.async.bulk.commit_group;" ::: "memory");
      mbar_wait_spin(&recv_bar, 0);
    }
    __syncthreads();
    if (warp < 8) {
      // (row, 32-column half) per thread
      const int rr = rlo + (tid >> 1), half = tid & 1;
      const int qrow = q0 + rr;
      if (rr < rhi && qrow < seq) {
        const float* src[4];
        float m = -INFINITY;
#pragma unroll
        for (int k = 0; k < 4; ++k) {  // (nsplit <= 4; unrolled so the row pointers stay in registers)
          src[k] = nullptr;
          if (k >= nsplit) continue;
          src[k] = k == split ? xs + rr * 68 : recv + (size_t(k < split ? k : k - 1) * rows_max + (rr - rlo)) * 68;
          m = fmaxf(m, src[k][64]);
        }
        float l = 0.f, acc[32];
#pragma unroll
        for (int e = 0; e < 32; ++e) acc[e] = 0.f;
#pragma unroll
        for (int k = 0; k < 4; ++k) {
          if (k >= nsplit) continue;
          const float mk = src[k][64];
          const float a = (mk == -INFINITY) ? 0.f : fast_exp2(mk - m);
          l += src[k][65] * a;
#pragma unroll
          for (int e = 0; e < 32; e += 4) {
            const float4 t = *reinterpret_cast<const float4*>(src[k] + 32 * half + e);
            acc[e] += t.x * a;
            acc[e + 1] += t.y * a;
            acc[e + 2] += t.z * a;
            acc[e + 3] += t.w * a;
          }
        }
        const float inv = l > 0.f ? 1.f / l : 0.f;
        uint4* dst = reinterpret_cast<uint4*>(ctx + (size_t)(tok0 + qrow) * H + head * TD + 32 * half);
#pragma unroll
        for (int c = 0; c < 4; ++c) {
          uint4 u;
          u.x = Cvt<T>::from2(acc[8 * c] * inv, acc[8 * c + 1] * inv);
          u.y = Cvt<T>::from2(acc[8 * c + 2] * inv, acc[8 * c + 3] * inv);
          u.z = Cvt<T>::from2(acc[8 * c + 4] * inv, acc[8 * c + 5] * inv);
          u.w = Cvt<T>::from2(acc[8 * c + 6] * inv, acc[8 * c + 7] * inv);
          dst[c] = u;
        }
      }
    }
    // the pushes must have read this CTA's rows before it exits (every push INTO this CTA has
    // landed: recv_bar completed)
    if (tid == 0) asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
  }
#ifdef DP_ATT_TRACE
  if (tid == 0) {
    ATRACE(12);
    unsigned smid;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
    const int b_ = (blockIdx.z * gridDim.y + blockIdx.y) * gridDim.x + blockIdx.x;
    if (b_ < 2048) g_att_trace[b_][14] = smid;
  }
#endif
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (warp == 9) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(512));
}

}  // namespace

bool attention_tc_supported(int ldqkv, int H, int heads, const void* qkv) {
  return heads > 0 && H % heads == 0 && H / heads == TD && ldqkv % 8 == 0 && ((uintptr_t)qkv % 16) == 0;
}

void launch_attention_tc(int dtype, const void* qkv, int ldqkv, void* ctx, int batch, int seq, int H, int heads,
                         bool causal, cudaStream_t s) {
  const int T = batch * seq;
  // maps over the whole qkv matrix with the 128-byte swizzle: box [128 rows][64 columns] for the Q
  // tile (columns h*64), [64 rows][64 columns] for the K / V tiles (columns H + h*64, 2H + h*64);
  // rows past T read as zeros
  const CUtensorMap mq = make_kmajor_map(qkv, dtype, T, 3 * H, ldqkv, TQ);
  const CUtensorMap mkv = make_kmajor_map(qkv, dtype, T, 3 * H, ldqkv, TK);
  const float scale_log2 = 1.4426950408889634f / 8.0f;  // log2(e) / sqrt(64)
  // Key-range split (round 2): one CTA per SM (512 TMEM columns), so a grid with fewer query
  // tiles than SMs leaves SMs idle.  Each query tile's keys are split over a cluster of 2 or 4
  // CTAs when the grid still fits ONE wave and every CTA keeps >= 4 key tiles: the merge costs
  // ~2 us (cluster barrier ~0.6 + push / merge / store ~1.5, tools/att_waves.py), a key-tile pair
  // ~1.2 us.  Measured (warm forwards, profiles/r02_attn_split_waves.jsonl,
  // r02_warm_ab_attention_split.jsonl): GPT-2 S512 0.611 -> 0.596 ms, BERT-Base S512 0.629 ->
  // 0.609; BERT-Large S384 (3 key tiles per half) 1.266 -> 1.281 and causal S1024 in two waves
  // (1.78 -> 1.90) slower, so neither splits; clusters of 3 also packed badly into the GPCs
  // (13 SMs idle, 9 CTAs in a second wave).
  const int nqt = (seq + TQ - 1) / TQ, nkt = (seq + TK - 1) / TK;
  const int ctas = heads * nqt * batch;
  int nsplit = 1;
  for (int n : {4, 2})
    if (ctas * n <= 148 && nkt >= 4 * n) {
      nsplit = n;
      break;
    }
  if (const int forced = experiment_env("DP_ATT_SPLIT", 0); forced > 0) nsplit = std::min(forced, 4);
  const dim3 grid(heads, nqt * nsplit, batch);
  auto go2 = [&](auto tag, auto ctag, auto stag) {
    using T = decltype(tag);
    constexpr bool C = decltype(ctag)::value, SP = decltype(stag)::value;
    auto kern = attention_tc_kernel<T, C, SP>;
    static std::atomic<unsigned> attr{0};
    if (first_on_device(attr))
      DP_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)SMEM_BYTES));
    if (SP)
      launch_kernel_cluster(kern, grid, dim3(NTHR), SMEM_BYTES, dim3(1, nsplit, 1), s, mq, mkv, (T*)ctx, seq, H,
                            scale_log2, nsplit);
    else
      launch_kernel(kern, grid, dim3(NTHR), SMEM_BYTES, s, mq, mkv, (T*)ctx, seq, H, scale_log2, 1);
  };
  auto go = [&](auto tag) {
    using B = std::bool_constant<true>;
    using F = std::bool_constant<false>;
    if (causal)
      nsplit > 1 ? go2(tag, B{}, B{}) : go2(tag, B{}, F{});
    else
      nsplit > 1 ? go2(tag, F{}, B{}) : go2(tag, F{}, F{});
  };
  if (dtype == DP_BF16)
    go(__nv_bfloat16{});
  else
    go(__half{});
  DP_CUDA(cudaGetLastError());
}

}  // namespace dp

#ifdef DP_ATT_TRACE
extern "C" __attribute__((visibility("default"))) int dp_debug_att_trace(void* host, int nblocks) {
  if (nblocks > 2048) nblocks = 2048;
  return (int)cudaMemcpyFromSymbol(host, dp::g_att_trace, size_t(nblocks) * 64 * sizeof(unsigned long long));
}
#endif
