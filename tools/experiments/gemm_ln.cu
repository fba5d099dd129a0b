// K2+K4 fused: resident tcgen05 GEMM whose epilogue applies the LayerNorm that follows it
// (BERT/RoBERTa post-LN after attn-out and fc2; GPT-2 pre-LN after the residual projections),
// removing the LayerNorm launch (SURVEY §8(a) a12 + a14).
//
//   z[m, n]   = x[m, :] . W[n, :] + b[n] + res[m, n]                  (fp32)
//   out[m, n] = (z[m, n] - mean_m) * rstd_m * gamma[n] + beta[n]     (storage dtype, + fp32 copy)
//   y[m, n]   = z[m, n]                                             (optional: GPT-2's residual stream)
//
// A LayerNorm needs whole rows (N = hidden = 6..8 W tiles of 128), so the CTAs that own one
// token tile form a thread-block cluster (N/128 x 1 x splits): cluster rank (nx, sp) computes W
// rows [128 nx, 128 nx + 128) over K-split sp.  Split partials are summed over DSMEM by their
// owner (rank sp owns tile rows [sp*128/S, (sp+1)*128/S)), so every element of z has exactly
// one owner CTA.  The row statistics are exchanged, not the data: each CTA publishes its
// per-token partial sums (BN floats) in shared memory, one cluster barrier later every CTA sums
// all ranks' partials in rank order (deterministic) over DSMEM -> mean; the same again for the
// squared deviations -> rstd (two-pass variance, as K4).  DSMEM traffic per CTA: 2 x CS x BN
// floats (+ the split partial rows when S > 1).  The previous "last CTA normalises the rows"
// fusion was measured slower (a serial tail behind every other CTA, K2).
#include <cuda.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstdlib>
#include <cstring>

#include "common.h"
#include "dtype.cuh"
#include "kernels.h"
#include "launch.cuh"
#include "tc.cuh"

namespace dp {

namespace {

constexpr int LBM = 128;  // W rows per tile
constexpr int LBK = 64;   // K per stage

template <int BN>
__host__ __device__ constexpr int ln_stages() {
  constexpr int bytes = LBM * LBK * 2 + BN * LBK * 2;
  constexpr int s = (200 * 1024) / bytes;
  return s > 12 ? 12 : s;
}

__device__ __forceinline__ uint32_t mapa_rank(uint32_t saddr, uint32_t rank) {
  uint32_t r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(saddr), "r"(rank));
  return r;
}
__device__ __forceinline__ float ld_dsmem(uint32_t addr) {
  float v;
  asm volatile("ld.shared::cluster.f32 %0, [%1];" : "=f"(v) : "r"(addr) : "memory");
  return v;
}
__device__ __forceinline__ void cluster_sync() {
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}

struct LnArgs {
  const void* res;   // [M, ldr] (T or fp32, io bit 0)
  int ldr;
  void* y;           // optional z output [M, ldy] (T or fp32, io bit 1)
  int ldy;
  const void* gamma;
  const void* beta;
  float eps;
  void* out;         // [M, ldo] storage dtype
  float* out32;      // optional fp32 copy of out
  int ldo;
  int io;
};

// grid (N/128, ceil(M/BN), S), cluster (N/128, 1, S), 128 threads
template <class T, int BN>
__global__ void __launch_bounds__(128, 1)
    gemm_ln_kernel(const __grid_constant__ CUtensorMap tmW, const __grid_constant__ CUtensorMap tmX, const T* bias,
                   int M, int N, int K, int nst, const LnArgs a) {
  constexpr int STAGES = ln_stages<BN>();
  constexpr uint32_t A_BYTES = LBM * LBK * 2;
  constexpr uint32_t B_BYTES = BN * LBK * 2;
  constexpr uint32_t STAGE_BYTES = A_BYTES + B_BYTES;
  constexpr uint32_t TMEM_COLS = BN < 32 ? 32 : BN;
  constexpr int PROW = BN + 1;  // fp32 tile row stride (odd: conflict-free TMEM -> smem writes)
  constexpr uint32_t IDESC = (1u << 4) | (FmtBits<T>::v << 7) | (FmtBits<T>::v << 10) | (uint32_t(BN >> 3) << 17) |
                             (uint32_t(LBM >> 4) << 24);
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  __shared__ __align__(8) uint64_t full_bar[STAGES], empty_bar[STAGES], done_bar;
  __shared__ uint32_t tmem_base_sh;
  __shared__ float sbias[LBM], sgam[LBM], sbet[LBM];
  __shared__ float psum[16][BN];     // per 8-row group partial sums (deterministic order)
  __shared__ float ssum[BN], ssq[BN];  // this CTA's per-token partials, read by every peer
  __shared__ float smean[BN], srstd[BN];

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int NX = gridDim.x, S = gridDim.z;
  const int nx = blockIdx.x, sp = blockIdx.z;
  const int n0 = nx * LBM, m0 = blockIdx.y * BN;
  const int kb_all = K / LBK;
  const int kb_lo = sp * kb_all / S;
  const int num_kb = (sp + 1) * kb_all / S - kb_lo;
  const int mcount = min(BN, M - m0);
  const int CS = NX * S;                     // cluster size; rank = nx + NX * sp
  const int RPR = LBM / S;                   // tile rows this rank owns: [sp*RPR, (sp+1)*RPR)
  const bool res32 = a.io & IO_RES_F32, y32 = a.io & IO_OUT_F32;

  if (warp == 0 && lane == 0) {
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&tmW)) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&tmX)) : "memory");
    for (int s = 0; s < STAGES; ++s) {
      mbar_init(&full_bar[s], 1);
      mbar_init(&empty_bar[s], 1);
    }
    mbar_init(&done_bar, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    // weights never depend on the previous kernel: the first ring of W tiles before the
    // grid-dependency wait (PDL)
    const int pre0 = num_kb < nst ? num_kb : nst;
    for (int kb = 0; kb < pre0; ++kb) {
      mbar_expect_tx(&full_bar[kb], STAGE_BYTES);
      tma_load_2d(&tmW, &full_bar[kb], smem + kb * STAGE_BYTES, (kb_lo + kb) * LBK, n0);
    }
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&tmem_base_sh)),
                 "r"(TMEM_COLS));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  // bias / gamma / beta of this tile's 128 W rows (weights: before the wait)
  sbias[threadIdx.x] = bias != nullptr ? Cvt<T>::to1(bias[n0 + threadIdx.x]) : 0.f;
  sgam[threadIdx.x] = Cvt<T>::to1(static_cast<const T*>(a.gamma)[n0 + threadIdx.x]);
  sbet[threadIdx.x] = Cvt<T>::to1(static_cast<const T*>(a.beta)[n0 + threadIdx.x]);
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tmem_d = tmem_base_sh;
  pdl_trigger();
  // every CTA's barriers initialised before any DSMEM access (arrive now, wait later)
  asm volatile("barrier.cluster.arrive.relaxed.aligned;" ::: "memory");
  pdl_wait();

  // epilogue units: (8 consecutive owned rows, token) pairs; thread t takes units t + 128 k
  // (RPR/8 * BN <= 16 * BN units, KU = BN / 8 per thread).  Their residuals are fetched now,
  // under the mainloop.
  constexpr int KU = BN / 8;
  const int G8 = RPR / 8;
  const int units = G8 * mcount;
  float rz[KU][8];
#pragma unroll
  for (int k = 0; k < KU; ++k) {
    const int u = threadIdx.x + 128 * k;
    if (u < units) {
      const int g = u / mcount, ml = u - g * mcount;
      const int row = sp * RPR + 8 * g;
      if (a.res != nullptr) load8<T>(a.res, (size_t)(m0 + ml) * a.ldr + n0 + row, rz[k], res32);
      else
#pragma unroll
        for (int e = 0; e < 8; ++e) rz[k][e] = 0.f;
    }
  }

  if (warp == 0 && lane == 0) {
    const int pre = num_kb < nst ? num_kb : nst;
    for (int kb = 0; kb < num_kb; ++kb) {
      const int s = kb % nst;
      uint8_t* A = smem + s * STAGE_BYTES;
      if (kb >= pre) {
        mbar_wait(&empty_bar[s], ((kb / nst) - 1) & 1);
        mbar_expect_tx(&full_bar[s], STAGE_BYTES);
        tma_load_2d(&tmW, &full_bar[s], A, (kb_lo + kb) * LBK, n0);
      }
      tma_load_2d(&tmX, &full_bar[s], A + A_BYTES, (kb_lo + kb) * LBK, m0);
    }
  } else if (warp == 1 && lane == 0) {
    for (int kb = 0; kb < num_kb; ++kb) {
      const int s = kb % nst;
      mbar_wait(&full_bar[s], (kb / nst) & 1);
      asm volatile("tcgen05.fence::after_thread_sync;");
      const uint8_t* A = smem + s * STAGE_BYTES;
      const uint64_t da = sw128_desc(A), db = sw128_desc(A + A_BYTES);
#pragma unroll
      for (int kk = 0; kk < LBK / 16; ++kk) umma_f16(tmem_d, da + 2 * kk, db + 2 * kk, IDESC, (kb | kk) != 0);
      umma_commit(&empty_bar[s]);
    }
    umma_commit(&done_bar);
  }
  __syncwarp();
  mbar_wait(&done_bar, 0);
  asm volatile("tcgen05.fence::after_thread_sync;");

  // 1) accumulator -> fp32 tile [128 W rows][BN] in shared memory (the ring is free)
  float* tile = reinterpret_cast<float*>(smem);
  {
    const int row = warp * 32 + lane;
#pragma unroll 1
    for (int c0 = 0; c0 < BN; c0 += 16) {
      uint32_t v[16];
      tmem_ld16(tmem_d + (uint32_t(warp * 32) << 16) + c0, v);
#pragma unroll
      for (int j = 0; j < 16; ++j) tile[row * PROW + c0 + j] = __uint_as_float(v[j]);
    }
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("barrier.cluster.wait.aligned;" ::: "memory");  // (matches the early arrive)
  // 2) split partials: every split rank's tile is staged before any owner sums them
  if (S > 1) cluster_sync();
  const uint32_t tile_s = smem_u32(tile);
  float z[KU][8];
#pragma unroll
  for (int k = 0; k < KU; ++k) {
    const int u = threadIdx.x + 128 * k;
    if (u < units) {
      const int g = u / mcount, ml = u - g * mcount;
      const int row = sp * RPR + 8 * g;
#pragma unroll
      for (int e = 0; e < 8; ++e) {
        float acc;
        if (S == 1) {
          acc = tile[(row + e) * PROW + ml];
        } else {
          acc = 0.f;
          for (int q = 0; q < S; ++q)  // split order 0..S-1 (deterministic)
            acc += ld_dsmem(mapa_rank(tile_s + uint32_t(((row + e) * PROW + ml) * 4), uint32_t(nx + NX * q)));
        }
        z[k][e] = acc + sbias[row + e] + rz[k][e];
      }
      if (a.y != nullptr) store8<T>(a.y, (size_t)(m0 + ml) * a.ldy + n0 + row, z[k], y32);
    }
  }
  // 3) per-token partial sums over this rank's rows -> ssum; cluster-wide mean
  for (int i = threadIdx.x; i < 16 * BN; i += 128) (&psum[0][0])[i] = 0.f;
  __syncthreads();
#pragma unroll
  for (int k = 0; k < KU; ++k) {
    const int u = threadIdx.x + 128 * k;
    if (u < units) {
      const int g = u / mcount, ml = u - g * mcount;
      float s = 0.f;
#pragma unroll
      for (int e = 0; e < 8; ++e) s += z[k][e];
      psum[g][ml] = s;
    }
  }
  __syncthreads();
  if (threadIdx.x < BN) {
    float s = 0.f;
    for (int g = 0; g < G8; ++g) s += psum[g][threadIdx.x];
    ssum[threadIdx.x] = s;
  }
  cluster_sync();  // every rank's ssum published (and every DSMEM read of the split tiles done)
  const float inv_n = 1.f / (float)N;
  if (threadIdx.x < BN) {
    float s = 0.f;
    const uint32_t base = smem_u32(&ssum[threadIdx.x]);
    for (int r = 0; r < CS; ++r) s += ld_dsmem(mapa_rank(base, (uint32_t)r));  // rank order
    smean[threadIdx.x] = s * inv_n;
  }
  __syncthreads();
  // 4) squared deviations -> rstd (two-pass variance)
#pragma unroll
  for (int k = 0; k < KU; ++k) {
    const int u = threadIdx.x + 128 * k;
    if (u < units) {
      const int g = u / mcount, ml = u - g * mcount;
      const float mu = smean[ml];
      float s = 0.f;
#pragma unroll
      for (int e = 0; e < 8; ++e) {
        const float d = z[k][e] - mu;
        s += d * d;
      }
      psum[g][ml] = s;
    }
  }
  __syncthreads();
  if (threadIdx.x < BN) {
    float s = 0.f;
    for (int g = 0; g < G8; ++g) s += psum[g][threadIdx.x];
    ssq[threadIdx.x] = s;
  }
  cluster_sync();
  if (threadIdx.x < BN) {
    float s = 0.f;
    const uint32_t base = smem_u32(&ssq[threadIdx.x]);
    for (int r = 0; r < CS; ++r) s += ld_dsmem(mapa_rank(base, (uint32_t)r));
    srstd[threadIdx.x] = rsqrtf(s * inv_n + a.eps);
  }
  __syncthreads();
  // 5) normalise the owned elements; 16-byte stores (8 consecutive columns of one token)
#pragma unroll
  for (int k = 0; k < KU; ++k) {
    const int u = threadIdx.x + 128 * k;
    if (u < units) {
      const int g = u / mcount, ml = u - g * mcount;
      const int row = sp * RPR + 8 * g;
      const float mu = smean[ml], rs = srstd[ml];
      float o[8];
#pragma unroll
      for (int e = 0; e < 8; ++e) o[e] = (z[k][e] - mu) * rs * sgam[row + e] + sbet[row + e];
      const size_t off = (size_t)(m0 + ml) * a.ldo + n0 + row;
      store8<T>(a.out, off, o, 0);
      if (a.out32 != nullptr) store8<T>(a.out32, off, o, 1);
    }
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (warp == 1) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem_d), "r"(TMEM_COLS));
  // no CTA leaves while a peer may still read its ssq (relaxed: only orders the DSMEM reads)
  asm volatile("barrier.cluster.arrive.relaxed.aligned;\n\tbarrier.cluster.wait.aligned;" ::: "memory");
}

template <class T, int BN>
void run_ln(const void* x, int ldx, const void* w, const void* bias, int M, int N, int K, int S, const LnArgs& a,
            cudaStream_t s) {
  constexpr int STAGES = ln_stages<BN>();
  constexpr size_t STAGE_BYTES = LBM * LBK * 2 + BN * LBK * 2;
  constexpr size_t smem_max = size_t(STAGES) * STAGE_BYTES + 1024;
  static_assert(size_t(LBM) * (BN + 1) * 4 + 1024 <= smem_max, "fp32 tile must fit the ring");
  static std::atomic<unsigned> attr{0};
  if (first_on_device(attr)) {
    DP_CUDA(cudaFuncSetAttribute(gemm_ln_kernel<T, BN>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem_max));
    DP_CUDA(cudaFuncSetAttribute(gemm_ln_kernel<T, BN>, cudaFuncAttributeNonPortableClusterSizeAllowed, 1));
  }
  const int dtype = std::is_same<T, __half>::value ? DP_FP16 : DP_BF16;
  const CUtensorMap mw = make_kmajor_map(w, dtype, N, K, K, LBM);
  const CUtensorMap mx = make_kmajor_map(x, dtype, M, K, ldx, BN);
  const int nx = N / LBM, mt = (M + BN - 1) / BN;
  launch_kernel_cluster(gemm_ln_kernel<T, BN>, dim3(nx, mt, S), dim3(128), smem_max, dim3(nx, 1, S), s, mw, mx,
                        (const T*)bias, M, N, K, STAGES, a);
}

// (BN, S): the slower of a CTA's ingest (~100 GB/s per SM) and the grid's aggregate L2 traffic
// (~5.5 TB/s; every token tile re-reads the whole W), + ~2 us of LN exchange, + ~4 us when the
// split partials cross DSMEM.  The B200 sweep (BERT-Base S=128 warm forward, K2+K4)
// measured BN=16/S=1 0.640 ms, 32/2 0.673, 32/1 0.771, 16/2 0.799 -- the model picks 16/1.
// DP_GEMM_LN_BN / DP_GEMM_LN_SPLIT override (sweeps).
struct LnCfg {
  int bn, s;
};
LnCfg pick_ln_cfg(int M, int N, int K) {
  static const int env_bn = getenv("DP_GEMM_LN_BN") ? atoi(getenv("DP_GEMM_LN_BN")) : 0;
  static const int env_s = getenv("DP_GEMM_LN_SPLIT") ? atoi(getenv("DP_GEMM_LN_SPLIT")) : 0;
  const int nx = N / LBM;
  LnCfg best{16, 1};
  double bt = 1e30;
  for (int bn : {16, 32}) {
    if (env_bn && bn != env_bn) continue;
    for (int s : {1, 2}) {
      if (env_s && s != env_s) continue;
      if (nx * s > 16 || (K / LBK) < 2 * s) continue;
      const int mt = (M + bn - 1) / bn;
      const int ctas = mt * nx * s, waves = (ctas + 147) / 148;
      const double per_cta = double(K) / s * (LBM + bn) * 2;
      const double t = std::max(waves * per_cta / 1e5, ctas * per_cta / 5.5e6) + 2.0 + (s > 1 ? 4.0 : 0.0);
      if (t < bt - 1e-9) bt = t, best = {bn, s};
    }
  }
  return best;
}

}  // namespace

bool gemm_ln_supported(int N) { return N % LBM == 0 && N / LBM >= 1 && N / LBM <= 8; }

void launch_gemm_ln(int dtype, const void* x, int ldx, const void* w, const void* bias, const void* res, int ldr,
                    void* y, int ldy, int M, int N, int K, int io, const void* gamma, const void* beta, float eps,
                    void* out, int ldo, void* out32, cudaStream_t s) {
  DP_CHECK(gemm_ln_supported(N) && K % LBK == 0, DP_ERR_UNSUPPORTED, "fused GEMM+LayerNorm: N = 128..1024, K % 64");
  DP_CHECK(gamma && beta && out && ldo % 8 == 0 && (!res || ldr % 8 == 0) && (!y || ldy % 8 == 0), DP_ERR_INVALID,
           "fused GEMM+LayerNorm: bad arguments");
  DP_CHECK(ldx % 8 == 0 && ((uintptr_t)x % 16) == 0 && ((uintptr_t)w % 16) == 0, DP_ERR_INVALID,
           "fused GEMM+LayerNorm: 16-byte alignment");
  if (M <= 0) return;
  const LnCfg c = pick_ln_cfg(M, N, K);
  const LnArgs a{res, ldr, y, ldy, gamma, beta, eps, out, static_cast<float*>(out32), ldo, io};
#define DP_LN_RUN(T)                                                       \
  switch (c.bn) {                                                          \
    case 16: run_ln<T, 16>(x, ldx, w, bias, M, N, K, c.s, a, s); break;   \
    default: run_ln<T, 32>(x, ldx, w, bias, M, N, K, c.s, a, s); break;   \
  }
  if (dtype == DP_BF16) {
    DP_LN_RUN(__nv_bfloat16)
  } else {
    DP_LN_RUN(__half)
  }
#undef DP_LN_RUN
}

}  // namespace dp
