// CUDA-core kernels of the hot path: DHA embedding (K1), LayerNorm (K4), DHA skinny
// linear (K3), attention core (K5, legacy mma.sync tensor path).  sm_100a.
//
// Direct-host-access (§2.2, §3.1): a kernel reads weights that
// live in cudaHostAlloc-mapped host memory in place, over PCIe.  Table 1 shows
// why the access pattern decides the cost: an embedding touches only the used rows, a
// V100 FC layer re-read its weights ~12x.  These kernels therefore (a) read host memory only
// with 16-byte vector loads that cover whole 128-byte lines, (b) stage anything reused
// (LN gamma/beta, the token-type row, a linear layer's weight rows) in shared memory so
// every host byte crosses the link once per CTA, and (c) keep many loads in flight.
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdlib>
#include <type_traits>

#include "common.h"
#include "dtype.cuh"
#include "kernels.h"
#include "launch.cuh"
#include "ln.cuh"
#include "attn.cuh"

namespace dp {

PdlState& pdl_state() {
  static thread_local PdlState s;
  return s;
}

// -------------------------------------------------------------------------------------
// K1: embedding gather + LayerNorm.  One warp per token (TPW tokens per warp, all of their host
// reads issued before any is used); VPL 16-byte vectors per lane.  The rows every token needs
// (token type 0, LN gamma / beta) are staged in shared memory: by every CTA, or -- CL = true,
// when they are host-mapped (DHA) -- by rank 0 of each cluster and broadcast over DSMEM, so they
// cross the host link once per cluster (one cluster up to 512 tokens) instead of once per CTA.
// The arithmetic per token is the same in every variant (bit-identical outputs).
// -------------------------------------------------------------------------------------
template <class T, int VPL, int TPW, bool CL>
__global__ void __launch_bounds__(256) embed_kernel(const int32_t* __restrict__ ids, int ntok, int seq, int pos_off,
                                                    const T* word, const T* pos, const T* type, const T* g,
                                                    const T* b, int H, float eps, void* __restrict__ out_,
                                                    int out_f32, float* __restrict__ out32, int vocab) {
  extern __shared__ uint4 sm[];  // [type0 | gamma | beta] as 16-byte vectors
  pdl_trigger();
  const int nv = H / 8;
  const bool has_type = type != nullptr, has_ln = g != nullptr;
  const bool stager = !CL || cta_cluster_rank() == 0;
  // the shared rows go into registers first; their host round trip overlaps the word/position
  // gathers below (one PCIe latency per CTA, not two)
  constexpr int SPT = 3;  // 3*nv <= 3*192 vectors over 256 threads
  uint4 stage[SPT];
#pragma unroll
  for (int k = 0; k < SPT; ++k) {
    const int i = threadIdx.x + k * 256;
    if (stager && i < 3 * nv) {
      const int which = i / nv, c = i - which * nv;
      const T* src = which == 0 ? type : (which == 1 ? g : b);
      if (src) stage[k] = ldg16(src + 8 * c);
    }
  }
  pdl_wait();
  const int lane = threadIdx.x & 31;
  const int gw = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5), nw = gridDim.x * (blockDim.x >> 5);
  uint4 wv[TPW][VPL], pv[TPW][VPL];
#pragma unroll
  for (int j = 0; j < TPW; ++j) {  // issue every host read of this warp's rows before using any
    const int t = gw + j * nw;
    const bool live = t < ntok;
    // ids outside [0, vocab) are clamped: a bad id must never make a DHA gather read past the
    // table in the pinned arena (vocab <= 0: unchecked, the caller's tables)
    int id = live ? ids[t] : 0;
    if (vocab > 0) id = min(max(id, 0), vocab - 1);
    const int p = pos_off + (live ? t % seq : 0);
#pragma unroll
    for (int v = 0; v < VPL; ++v) {
      const int c = lane + 32 * v;
      if (live && c < nv) {
        wv[j][v] = ldg16(word + (size_t)id * H + 8 * c);
        pv[j][v] = ldg16(pos + (size_t)p * H + 8 * c);
      }
    }
  }
#pragma unroll
  for (int k = 0; k < SPT; ++k) {
    const int i = threadIdx.x + k * 256;
    if (stager && i < 3 * nv) {
      const int which = i / nv;
      const T* src = which == 0 ? type : (which == 1 ? g : b);
      if (src) sm[i] = stage[k];
    }
  }
  if (CL)
    cluster_bcast_from_rank0(sm, 3 * nv);
  else
    __syncthreads();
#pragma unroll
  for (int j = 0; j < TPW; ++j) {
    const int t = gw + j * nw;
    if (t >= ntok) break;
    float x[VPL][8];
    float sum = 0.f;
#pragma unroll
    for (int v = 0; v < VPL; ++v) {
      const int c = lane + 32 * v;
      if (c < nv) {
        float a[8], q[8];
        unpack8<T>(wv[j][v], a);
        unpack8<T>(pv[j][v], q);
        if (has_type) {
          float y[8];
          unpack8<T>(sm[c], y);
#pragma unroll
          for (int e = 0; e < 8; ++e) x[v][e] = a[e] + q[e] + y[e];
        } else {
#pragma unroll
          for (int e = 0; e < 8; ++e) x[v][e] = a[e] + q[e];
        }
#pragma unroll
        for (int e = 0; e < 8; ++e) sum += x[v][e];
      }
    }
    if (!has_ln) {
#pragma unroll
      for (int v = 0; v < VPL; ++v) {
        const int c = lane + 32 * v;
        if (c < nv) store8<T>(out_, (size_t)t * H + 8 * c, x[v], out_f32);
      }
      continue;
    }
    const float mean = warp_sum(sum) / H;
    float sq = 0.f;
#pragma unroll
    for (int v = 0; v < VPL; ++v) {
      const int c = lane + 32 * v;
      if (c < nv) {
#pragma unroll
        for (int e = 0; e < 8; ++e) {
          const float d = x[v][e] - mean;
          sq += d * d;
        }
      }
    }
    const float rstd = rsqrtf(warp_sum(sq) / H + eps);
#pragma unroll
    for (int v = 0; v < VPL; ++v) {
      const int c = lane + 32 * v;
      if (c < nv) {
        float gg[8], bb[8], y[8];
        unpack8<T>(sm[nv + c], gg);
        unpack8<T>(sm[2 * nv + c], bb);
#pragma unroll
        for (int e = 0; e < 8; ++e) y[e] = (x[v][e] - mean) * rstd * gg[e] + bb[e];
        store8<T>(out_, (size_t)t * H + 8 * c, y, out_f32);
        if (out32 != nullptr) store8<T>(out32, (size_t)t * H + 8 * c, y, 1);  // fp32 residual-stream copy
      }
    }
  }
}

template <class T, int V, int TPW, bool CL>
static void embed_launch(int grid, int cluster, size_t sm, cudaStream_t s, const int32_t* ids, int ntok, int seq,
                         int pos_off, const void* word, const void* pos, const void* type, const void* g,
                         const void* b, int H, float eps, void* out, bool out_f32, float* out32, int vocab) {
  if (CL) {
    static std::atomic<unsigned> attr{0};
    if (first_on_device(attr))
      DP_CUDA(cudaFuncSetAttribute(embed_kernel<T, V, TPW, CL>, cudaFuncAttributeNonPortableClusterSizeAllowed, 1));
  }
  launch_kernel_cluster(embed_kernel<T, V, TPW, CL>, dim3(grid), dim3(256), sm, dim3(cluster), s, ids, ntok, seq,
                        pos_off, (const T*)word, (const T*)pos, (const T*)type, (const T*)g, (const T*)b, H, eps, out,
                        (int)out_f32, out32, vocab);
}

template <class T, int V>
static void embed_v(bool shared_host, int ntok, int grid_one, size_t sm, cudaStream_t s, const int32_t* ids, int seq,
                    int pos_off, const void* word, const void* pos, const void* type, const void* g, const void* b,
                    int H, float eps, void* out, bool out_f32, float* out32, int vocab) {
  if (!shared_host) {  // one token per warp, every CTA stages the shared rows (HBM / L2)
    embed_launch<T, V, 1, false>(grid_one, 1, sm, s, ids, ntok, seq, pos_off, word, pos, type, g, b, H, eps, out,
                                 out_f32, out32, vocab);
    return;
  }
  // host-mapped shared rows: clusters of 16 CTAs (128 warps), up to 4 tokens per warp
  const int tpw = ntok <= 128 ? 1 : ntok <= 256 ? 2 : 4;
  int grid = (ntok + 8 * tpw - 1) / (8 * tpw);
  const int cluster = std::min(16, grid);
  grid = (grid + cluster - 1) / cluster * cluster;
#define DP_EMB_T(P) embed_launch<T, V, P, true>(grid, cluster, sm, s, ids, ntok, seq, pos_off, word, pos, type, g, b, H, \
                                               eps, out, out_f32, out32, vocab)
  if (tpw == 1) DP_EMB_T(1);
  else if (tpw == 2) DP_EMB_T(2);
  else DP_EMB_T(4);
#undef DP_EMB_T
}

template <class T>
static void embed_t(const int32_t* ids, int ntok, int seq, int pos_off, const void* word, const void* pos,
                    const void* type, const void* g, const void* b, int H, float eps, void* out, bool out_f32,
                    float* out32, int vocab, bool shared_host, cudaStream_t s) {
  const int warps = 8;
  const int grid = (ntok + warps - 1) / warps;
  const size_t sm = size_t(3) * (H / 8) * 16;
  const int vpl = (H / 8 + 31) / 32;
  shared_host = shared_host && (type != nullptr || g != nullptr);  // GPT-2 has no shared rows
#define DP_EMB(V)                                                                                                   \
  embed_v<T, V>(shared_host, ntok, grid, sm, s, ids, seq, pos_off, word, pos, type, g, b, H, eps, out, out_f32, out32, \
                vocab)
  switch (vpl) {
    case 1: DP_EMB(1); break;
    case 2: DP_EMB(2); break;
    case 3: DP_EMB(3); break;
    case 4: DP_EMB(4); break;
    case 5: DP_EMB(5); break;
    case 6: DP_EMB(6); break;
    default: fail(DP_ERR_UNSUPPORTED, "embedding hidden size > 1536");
  }
#undef DP_EMB
  DP_CUDA(cudaGetLastError());
}

void launch_embed(int dtype, const int32_t* ids, int ntok, int seq, int pos_off, const void* word, const void* pos,
                  const void* type, const void* g, const void* b, int H, float eps, void* out, bool out_f32,
                  cudaStream_t s, void* out32, int vocab, bool shared_host) {
  DP_CHECK(H % 8 == 0 && H > 0, DP_ERR_INVALID, "hidden must be a multiple of 8");
  DP_CHECK(seq > 0 && ntok >= 0, DP_ERR_INVALID, "bad token counts");
  if (ntok == 0) return;
  if (dtype == DP_FP32) {
    launch_embed_f32(ids, ntok, seq, pos_off, word, pos, type, g, b, H, eps, out, out32, vocab, s);
    return;
  }
  if (dtype == DP_BF16)
    embed_t<__nv_bfloat16>(ids, ntok, seq, pos_off, word, pos, type, g, b, H, eps, out, out_f32,
                           static_cast<float*>(out32), vocab, shared_host, s);
  else
    embed_t<__half>(ids, ntok, seq, pos_off, word, pos, type, g, b, H, eps, out, out_f32, static_cast<float*>(out32),
                    vocab, shared_host, s);
}

// -------------------------------------------------------------------------------------
// K4: LayerNorm (+ residual).  gamma/beta staged in shared memory: by every CTA when they are in
// HBM, or -- when they are host-mapped (DHA), CL = true -- by rank 0 of a single cluster of <= 16
// CTAs and broadcast over DSMEM, so the host link carries them exactly once per launch.
// -------------------------------------------------------------------------------------
// MODE: the forward's two LayerNorm forms as compile-time variants (fp32 input, no residual;
// 1 = with the fp32 copy of the output -- BERT's residual stream --, 2 = without -- GPT-2), 0 =
// any (the test hooks, DHA gamma / beta).  A variant carries only its own load / store code: a
// CTA runs its code once and cold instruction fetch is on its critical path (K2 round 2).
template <class T, int VPL, bool CL, int MODE>
__global__ void __launch_bounds__(256) layernorm_kernel(const void* __restrict__ x, const void* __restrict__ r,
                                                        const T* g, const T* b, T* __restrict__ y, int rows,
                                                        int n, float eps, int in_f32, float* __restrict__ y32) {
  extern __shared__ uint4 sm[];  // [gamma | beta]
  pdl_trigger();
  const int nv = n / 8;
  if (!CL || cta_cluster_rank() == 0)
    for (int i = threadIdx.x; i < 2 * nv; i += blockDim.x) sm[i] = ldg16(i < nv ? g + 8 * i : b + 8 * (i - nv));
  pdl_wait();
  if (CL)
    cluster_bcast_from_rank0(sm, 2 * nv);
  else
    __syncthreads();
  const int lane = threadIdx.x & 31;
  const int nwarps = gridDim.x * (blockDim.x >> 5);
  for (int row = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); row < rows; row += nwarps)
    if constexpr (MODE == 1)
      ln_row_warp<T, VPL, 0>(x, nullptr, (size_t)row * n, n, eps, 1, sm, y, (size_t)row * n, y32);
    else if constexpr (MODE == 2)
      ln_row_warp<T, VPL, 0>(x, nullptr, (size_t)row * n, n, eps, 1, sm, y, (size_t)row * n, nullptr);
    else
      ln_row_warp<T, VPL, 0>(x, r, (size_t)row * n, n, eps, in_f32, sm, y, (size_t)row * n, y32);
}

// rows (warps) per LayerNorm CTA: 4 up to 128 rows (32 CTAs: BERT-Base S128 warm 0.3465 ->
// 0.343 ms), else 8 (4 measured slower at 256-1024 rows; profiles/r02_warm_ab_ln_warps.jsonl).
// DP_LN_WARPS overrides it in instrumented builds (A/B only).
static int ln_warps(int rows) {
  static const int w = experiment_env("DP_LN_WARPS", 0);
  return w > 0 ? w : rows <= 128 ? 4 : 8;
}

template <class T, int V, bool CL, int MODE>
static void layernorm_launch_m(int grid, size_t sm, cudaStream_t s, const void* x, const void* r, const void* g,
                               const void* b, void* y, int rows, int n, float eps, bool in_f32, float* y32) {
  if (CL) {
    static std::atomic<unsigned> attr{0};
    if (first_on_device(attr))
      DP_CUDA(cudaFuncSetAttribute(layernorm_kernel<T, V, CL, MODE>, cudaFuncAttributeNonPortableClusterSizeAllowed,
                                   1));
  }
  launch_kernel_cluster(layernorm_kernel<T, V, CL, MODE>, dim3(grid), dim3(32 * ln_warps(rows)), sm, dim3(CL ? grid : 1), s, x, r,
                        (const T*)g, (const T*)b, (T*)y, rows, n, eps, (int)in_f32, y32);
}

template <class T, int V, bool CL>
static void layernorm_launch(int grid, size_t sm, cudaStream_t s, const void* x, const void* r, const void* g,
                             const void* b, void* y, int rows, int n, float eps, bool in_f32, float* y32) {
  if constexpr (!CL) {
    if (in_f32 && r == nullptr) {
      if (y32 != nullptr)
        layernorm_launch_m<T, V, CL, 1>(grid, sm, s, x, r, g, b, y, rows, n, eps, in_f32, y32);
      else
        layernorm_launch_m<T, V, CL, 2>(grid, sm, s, x, r, g, b, y, rows, n, eps, in_f32, y32);
      return;
    }
  }
  layernorm_launch_m<T, V, CL, 0>(grid, sm, s, x, r, g, b, y, rows, n, eps, in_f32, y32);
}

template <class T>
static void layernorm_t(const void* x, const void* r, const void* g, const void* b, void* y, int rows, int n,
                        float eps, bool in_f32, float* y32, bool gb_host, cudaStream_t s) {
  // one row per warp (latency: every row's loads in flight at once).  gamma/beta in HBM: every
  // CTA stages them (L2 hits); host-mapped (DHA): ONE cluster of <= 16 CTAs (up to 128 warps,
  // several rows each beyond 128 rows) reads them once and shares them over DSMEM, so the host
  // link carries exactly 2 x n elements (the algorithmic bytes)
  const int warps = ln_warps(rows);
  int grid = (rows + warps - 1) / warps;
  if (grid > 148 * 8) grid = 148 * 8;
  if (gb_host && grid > 16) grid = 16;
  if (grid < 1) grid = 1;
  const size_t sm = size_t(2) * (n / 8) * 16;
  const int vpl = (n / 8 + 31) / 32;
#define DP_LN(V)                                                                                               \
  (gb_host ? layernorm_launch<T, V, true>(grid, sm, s, x, r, g, b, y, rows, n, eps, in_f32, y32)               \
           : layernorm_launch<T, V, false>(grid, sm, s, x, r, g, b, y, rows, n, eps, in_f32, y32))
  switch (vpl) {
    case 1: DP_LN(1); break;
    case 2: DP_LN(2); break;
    case 3: DP_LN(3); break;
    case 4: DP_LN(4); break;
    case 5: DP_LN(5); break;
    case 6: DP_LN(6); break;
    default: fail(DP_ERR_UNSUPPORTED, "layernorm width > 1536");
  }
#undef DP_LN
  DP_CUDA(cudaGetLastError());
}

void launch_layernorm(int dtype, const void* x, const void* r, const void* g, const void* b, void* y, int rows,
                      int n, float eps, bool in_f32, cudaStream_t s, void* y32, bool gb_host) {
  if (ablate_mask() & 2) return;
  DP_CHECK(n % 8 == 0 && n > 0, DP_ERR_INVALID, "LN width must be a multiple of 8");
  if (rows <= 0) return;
  if (dtype == DP_FP32) {
    launch_layernorm_f32(x, r, g, b, y, rows, n, eps, s, y32);
    return;
  }
  if (dtype == DP_BF16)
    layernorm_t<__nv_bfloat16>(x, r, g, b, y, rows, n, eps, in_f32, static_cast<float*>(y32), gb_host, s);
  else
    layernorm_t<__half>(x, r, g, b, y, rows, n, eps, in_f32, static_cast<float*>(y32), gb_host, s);
}

// -------------------------------------------------------------------------------------
// K3: skinny linear for direct-host-access.  Each CTA owns R consecutive rows of W
// ([N,K] row-major, so its slice is one contiguous R*K*2-byte block): it streams the
// slice from (host) memory ONCE with coalesced 16-byte loads into shared memory, then
// every warp computes whole-K dot products for its tokens against the staged rows and
// reduces them with warp shuffles.  Host-link bytes = N*K*2 + N*2 exactly (Table 1's
// 12x re-read of a stock FC layer under DHA, is what this avoids).
// -------------------------------------------------------------------------------------
template <class T, int R>
__global__ void __launch_bounds__(256) skinny_linear_kernel(const T* __restrict__ X, int ldx, const T* W,
                                                            const T* bias, const void* res, int ldr,
                                                            void* Y, int ldy, int M, int N, int K,
                                                            int act, int io) {
  extern __shared__ float4 swf[];  // R rows x K as fp32 (converted once), 2 float4 per 8 elements
  pdl_trigger();
  const int kv = K / 8;
  const int n0 = blockIdx.x * R;
  const int rows = min(R, N - n0);
  const int total = rows * kv;
  const uint4* src = reinterpret_cast<const uint4*>(W + (size_t)n0 * K);
  // weights never depend on the previous kernel: stream them (host or HBM) before the
  // grid-dependency wait, up to 8 independent 16-byte loads in flight per thread
  for (int base = threadIdx.x; base < total; base += 8 * 256) {
    uint4 r[8];
#pragma unroll
    for (int j = 0; j < 8; ++j)
      if (base + j * 256 < total) r[j] = ldg16(src + base + j * 256);
#pragma unroll
    for (int j = 0; j < 8; ++j)
      if (base + j * 256 < total) {
        float f[8];
        unpack8<T>(r[j], f);
        swf[2 * (base + j * 256)] = make_float4(f[0], f[1], f[2], f[3]);
        swf[2 * (base + j * 256) + 1] = make_float4(f[4], f[5], f[6], f[7]);
      }
  }
  __shared__ float sbias[R];
  if (threadIdx.x < rows) sbias[threadIdx.x] = bias ? Cvt<T>::to1(bias[n0 + threadIdx.x]) : 0.f;
  pdl_wait();
  __syncthreads();
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  // two tokens per warp iteration: every staged weight read feeds two FMAs
  for (int m = 2 * warp; m < M; m += 16) {
    const bool two = m + 1 < M;
    float acc[2][R];
#pragma unroll
    for (int r = 0; r < R; ++r) acc[0][r] = acc[1][r] = 0.f;
    const T* x0 = X + (size_t)m * ldx;
    const T* x1 = two ? x0 + ldx : x0;
    for (int c = lane; c < kv; c += 32) {
      float a[8], b[8];
      unpack8<T>(*reinterpret_cast<const uint4*>(x0 + 8 * c), a);
      unpack8<T>(*reinterpret_cast<const uint4*>(x1 + 8 * c), b);
#pragma unroll
      for (int r = 0; r < R; ++r) {
        if (r < rows) {
          const float4 w0 = swf[2 * (r * kv + c)], w1 = swf[2 * (r * kv + c) + 1];
          const float wf[8] = {w0.x, w0.y, w0.z, w0.w, w1.x, w1.y, w1.z, w1.w};
#pragma unroll
          for (int e = 0; e < 8; ++e) {
            acc[0][r] = fmaf(a[e], wf[e], acc[0][r]);
            acc[1][r] = fmaf(b[e], wf[e], acc[1][r]);
          }
        }
      }
    }
#pragma unroll
    for (int t = 0; t < 2; ++t) {
#pragma unroll
      for (int r = 0; r < R; ++r) acc[t][r] = warp_sum(acc[t][r]);
      float mine = 0.f;
#pragma unroll
      for (int r = 0; r < R; ++r)
        if (lane == r) mine = acc[t][r];
      if (lane < rows && (t == 0 || two)) {
        const int n = n0 + lane, mm = m + t;
        float v = apply_act(mine + sbias[lane], act);
        if (res) v += load1<T>(res, (size_t)mm * ldr + n, io & IO_RES_F32);
        store1<T>(Y, (size_t)mm * ldy + n, v, io & IO_OUT_F32);
      }
    }
  }
}

// K3 variant for M <= 8 rows and K = 256 * VPL <= 1024 (the pooler, GPT-2's LM head): a
// streaming GEMV.  One warp per output column n (a W row), two rows per iteration: every lane
// issues its 2 x VPL 16-byte loads of the two rows before any FMA, so ~2 x K x 2 bytes per warp
// are in flight; X sits in shared memory as fp32.  W is read exactly once (host-mapped or HBM),
// no shared-memory staging of W (the skinny kernel above stages W as fp32 for reuse across
// many tokens, which a 1..4-row GEMV does not need).
template <class T, int MR, int VPL>
__global__ void __launch_bounds__(256) gemv_kernel(const T* __restrict__ X, int ldx, const T* W, const T* bias,
                                                   const void* res, int ldr, void* Y, int ldy, int M, int N,
                                                   int act, int io) {
  constexpr int K = 256 * VPL;
  extern __shared__ float xs[];  // [MR][K]
  pdl_trigger();
  const int lane = threadIdx.x & 31;
  const int gw = blockIdx.x * 8 + (threadIdx.x >> 5), nw = gridDim.x * 8;
  // weights never depend on the previous kernel: the first two rows are in flight before the
  // grid-dependency wait
  uint4 wa[VPL], wb[VPL];
  int n = gw;
  auto fetch = [&](uint4* dst, int row) {
#pragma unroll
    for (int v = 0; v < VPL; ++v)
      if (row < N) dst[v] = ldg16(W + (size_t)row * K + 8 * (lane + 32 * v));
  };
  fetch(wa, n);
  fetch(wb, n + nw);
  pdl_wait();
  for (int i = threadIdx.x; i < MR * K / 8; i += 256) {
    const int m = i / (K / 8), c = i - m * (K / 8);
    float f[8] = {0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f};
    if (m < M) unpack8<T>(ldg16(X + (size_t)m * ldx + 8 * c), f);
#pragma unroll
    for (int e = 0; e < 8; ++e) xs[m * K + 8 * c + e] = f[e];
  }
  __syncthreads();
  for (; n < N; n += 2 * nw) {
    float acc[2][MR];
#pragma unroll
    for (int t = 0; t < 2; ++t)
#pragma unroll
      for (int m = 0; m < MR; ++m) acc[t][m] = 0.f;
#pragma unroll
    for (int v = 0; v < VPL; ++v) {
      float a[8], b[8];
      unpack8<T>(wa[v], a);
      unpack8<T>(wb[v], b);
#pragma unroll
      for (int m = 0; m < MR; ++m) {
        const float4* xp = reinterpret_cast<const float4*>(xs + m * K + 8 * (lane + 32 * v));
        const float4 x0 = xp[0], x1 = xp[1];
        const float xv[8] = {x0.x, x0.y, x0.z, x0.w, x1.x, x1.y, x1.z, x1.w};
#pragma unroll
        for (int e = 0; e < 8; ++e) {
          acc[0][m] = fmaf(xv[e], a[e], acc[0][m]);
          acc[1][m] = fmaf(xv[e], b[e], acc[1][m]);
        }
      }
    }
    const int n0 = n, n1 = n + nw;
    fetch(wa, n + 2 * nw);  // the next two rows stream while this pair is reduced and stored
    fetch(wb, n + 3 * nw);
#pragma unroll
    for (int t = 0; t < 2; ++t) {
      const int row = t == 0 ? n0 : n1;
#pragma unroll
      for (int m = 0; m < MR; ++m) acc[t][m] = warp_sum(acc[t][m]);
      if (lane == 0 && row < N) {
        const float bz = bias ? Cvt<T>::to1(bias[row]) : 0.f;
#pragma unroll
        for (int m = 0; m < MR; ++m) {
          if (m < M) {
            float v = apply_act(acc[t][m] + bz, act);
            if (res) v += load1<T>(res, (size_t)m * ldr + row, io & IO_RES_F32);
            store1<T>(Y, (size_t)m * ldy + row, v, io & IO_OUT_F32);
          }
        }
      }
    }
  }
}

template <class T, int MR>
static void gemv_mr(const void* x, int ldx, const void* w, const void* bias, const void* res, int ldr, void* y,
                    int ldy, int M, int N, int K, int act, int io, cudaStream_t s) {
  const size_t sm = size_t(MR) * K * 4;
  int grid = (N + 15) / 16;  // 8 warps x 2 rows per CTA per pass
  if (grid > 148 * 8) grid = 148 * 8;
#define DP_GEMV(V)                                                                                           \
  launch_kernel(gemv_kernel<T, MR, V>, dim3(grid), dim3(256), sm, s, (const T*)x, ldx, (const T*)w, (const T*)bias, \
                res, ldr, y, ldy, M, N, act, io)
  switch (K / 256) {
    case 1: DP_GEMV(1); break;
    case 2: DP_GEMV(2); break;
    case 3: DP_GEMV(3); break;
    case 4: DP_GEMV(4); break;
    default: fail(DP_ERR_UNSUPPORTED, "gemv: K must be 256..1024");
  }
#undef DP_GEMV
}

bool gemv_supported(int M, int K, int ldx, const void* x) {
  return M >= 1 && M <= 8 && K % 256 == 0 && K <= 1024 && ldx % 8 == 0 && ((uintptr_t)x % 16) == 0;
}

template <class T>
static void gemv_t(const void* x, int ldx, const void* w, const void* bias, const void* res, int ldr, void* y, int ldy,
                   int M, int N, int K, int act, int io, cudaStream_t s) {
  if (M == 1) gemv_mr<T, 1>(x, ldx, w, bias, res, ldr, y, ldy, M, N, K, act, io, s);
  else if (M == 2) gemv_mr<T, 2>(x, ldx, w, bias, res, ldr, y, ldy, M, N, K, act, io, s);
  else if (M <= 4) gemv_mr<T, 4>(x, ldx, w, bias, res, ldr, y, ldy, M, N, K, act, io, s);
  else gemv_mr<T, 8>(x, ldx, w, bias, res, ldr, y, ldy, M, N, K, act, io, s);
}

template <class T>
static void skinny_t(const void* x, int ldx, const void* w, const void* bias, const void* res, int ldr, void* y,
                     int ldy, int M, int N, int K, int act, int io, cudaStream_t s) {
  constexpr int R = 8;
  const size_t sm = size_t(R) * K * sizeof(float);
  static std::atomic<unsigned> attr_set{0};  // one per template instantiation
  if (first_on_device(attr_set))
    DP_CUDA(cudaFuncSetAttribute(skinny_linear_kernel<T, R>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024));
  launch_kernel(skinny_linear_kernel<T, R>, dim3((N + R - 1) / R), dim3(256), sm, s, (const T*)x, ldx, (const T*)w,
                (const T*)bias, res, ldr, y, ldy, M, N, K, act, io);
}

template <class T>
void skinny_mma_t(const void* x, int ldx, const void* w, const void* bias, const void* res, int ldr, void* y, int ldy,
                  int M, int N, int K, int act, int io, cudaStream_t s);
int skinny_cluster(int K);

// M <= 16 tokens (e.g. the pooler): warp-shuffle dot products; more tokens: the same one-pass
// weight staging with the per-CTA products on mma.sync (the link stays the bound).
void launch_skinny_linear(int dtype, const void* x, int ldx, const void* w, const void* bias, const void* res,
                          int ldr, void* y, int ldy, int M, int N, int K, int act, int io, cudaStream_t s) {
  if (ablate_mask() & 8) return;
  DP_CHECK(K % 8 == 0 && K > 0 && N > 0, DP_ERR_INVALID, "skinny linear needs K % 8 == 0");
  if (M <= 0) return;
  if (dtype == DP_FP32) {  // W read once, as below; fp32 in / out (io flags are implied)
    launch_linear_f32(x, ldx, w, bias, res, ldr, y, ldy, M, N, K, act, s);
    return;
  }
  const bool mma = M > 16 && N % 16 == 0 && K % 16 == 0 && ldx % 8 == 0 && ((uintptr_t)x % 16) == 0 &&
                   skinny_cluster(K) > 0;
  if (mma) {
    if (dtype == DP_BF16)
      skinny_mma_t<__nv_bfloat16>(x, ldx, w, bias, res, ldr, y, ldy, M, N, K, act, io, s);
    else
      skinny_mma_t<__half>(x, ldx, w, bias, res, ldr, y, ldy, M, N, K, act, io, s);
    return;
  }
  if (gemv_supported(M, K, ldx, x)) {
    if (dtype == DP_BF16)
      gemv_t<__nv_bfloat16>(x, ldx, w, bias, res, ldr, y, ldy, M, N, K, act, io, s);
    else
      gemv_t<__half>(x, ldx, w, bias, res, ldr, y, ldy, M, N, K, act, io, s);
    return;
  }
  DP_CHECK(size_t(8) * K * 4 <= 200 * 1024, DP_ERR_UNSUPPORTED, "skinny linear: K too large");
  if (dtype == DP_BF16)
    skinny_t<__nv_bfloat16>(x, ldx, w, bias, res, ldr, y, ldy, M, N, K, act, io, s);
  else
    skinny_t<__half>(x, ldx, w, bias, res, ldr, y, ldy, M, N, K, act, io, s);
}

// -------------------------------------------------------------------------------------
// K5: attention core (the tile body lives in attn.cuh, shared with the persistent kernel)
// -------------------------------------------------------------------------------------
template <class T>
__global__ void __launch_bounds__(128) attention_kernel(const T* __restrict__ qkv, int ldqkv, T* __restrict__ ctx,
                                                        int seq, int H, int causal, float scale_log2) {
  __shared__ __align__(16) T sq[ATT_BQ * ATT_LD];
  __shared__ __align__(16) T sk[2 * ATT_BK * ATT_LD];
  __shared__ __align__(16) T sv[2 * ATT_BK * ATT_LD];
  pdl_trigger();
  pdl_wait();  // q, k, v come from the previous kernels
  attention_tile<T>(qkv, ldqkv, ctx, seq, H, causal, scale_log2, blockIdx.x, blockIdx.y, blockIdx.z, sq, sk, sv,
                    threadIdx.x, [] { __syncthreads(); });
}

// K5b: the same tile on 8 warps in two groups that split the key tiles (group g takes tiles
// g, g+2, ...) for the same 64 query rows, each with its own 2-deep K/V ring; the two partial
// online-softmax states (running max, sum, unnormalised O) are merged through shared memory at
// the end.  Halves the dependent chain of key tiles per query tile (the causal S = 1024 tiles
// near the diagonal walk 16 of them) and doubles the warps feeding the SM's tensor pipes.
// Q + 2 stages x G groups x (K, V)
template <int G>
constexpr int att_groups_smem() { return (ATT_BQ * ATT_LD + 4 * G * ATT_BK * ATT_LD) * 2; }

template <class T, int G>
__global__ void __launch_bounds__(128 * G) attention2_kernel(const T* __restrict__ qkv, int ldqkv, T* __restrict__ ctx,
                                                             int seq, int H, int causal, float scale_log2) {
  extern __shared__ __align__(16) uint8_t att2_smem[];
  T* sq = reinterpret_cast<T*>(att2_smem);
  T* kv = sq + ATT_BQ * ATT_LD;
  auto ktile = [&](int stage, int g) { return kv + ((stage * G + g) * 2 + 0) * ATT_BK * ATT_LD; };
  auto vtile = [&](int stage, int g) { return kv + ((stage * G + g) * 2 + 1) * ATT_BK * ATT_LD; };
  constexpr int NT = 128 * G;
  pdl_trigger();
  pdl_wait();  // q, k, v come from the previous kernels
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5, grp = warp >> 2, wq = warp & 3;
  // grid (heads, query tiles, batch): CTAs start in linear order, so with causal masking the
  // query tiles are visited last-first -- the longest key chains go out in the first wave and
  // the short ones fill in behind them (longest-processing-time-first)
  const int head = blockIdx.x, bidx = blockIdx.z;
  const int qt = causal > 1 ? (int)gridDim.y - 1 - (int)blockIdx.y : (int)blockIdx.y;
  const size_t tok0 = (size_t)bidx * seq;
  const int q0 = qt * ATT_BQ;
  const T* qbase = qkv + tok0 * ldqkv + head * ATT_D;
  const T* kbase = qbase + H;
  const T* vbase = qbase + 2 * H;
  int nkt = (seq + ATT_BK - 1) / ATT_BK;
  if (causal) nkt = min(nkt, (q0 + ATT_BQ - 1) / ATT_BK + 1);
  const int npair = (nkt + G - 1) / G;
  auto load_pair = [&](int j) {  // key tiles G*j + g (group g) into stage j & 1
    for (int i = tid; i < G * ATT_BK * 8; i += NT) {
      const int g = i / (ATT_BK * 8), r = (i >> 3) & (ATT_BK - 1), c = i & 7;
      const int kt = G * j + g;
      if (kt >= nkt) continue;
      const int k0 = kt * ATT_BK;
      const bool ok = k0 + r < seq;
      const size_t off = (size_t)(ok ? k0 + r : 0) * ldqkv + c * 8;
      cp_async16_zfill(&ktile(j & 1, g)[r * ATT_LD + c * 8], kbase + off, ok);
      cp_async16_zfill(&vtile(j & 1, g)[r * ATT_LD + c * 8], vbase + off, ok);
    }
  };
  for (int i = tid; i < ATT_BQ * 8; i += NT) {
    const int r = i >> 3, c = i & 7;
    const bool ok = q0 + r < seq;
    cp_async16_zfill(&sq[r * ATT_LD + c * 8], qbase + (size_t)(ok ? q0 + r : 0) * ldqkv + c * 8, ok);
  }
  load_pair(0);
  cp_async_commit();
  if (npair > 1) load_pair(1);
  cp_async_commit();
  cp_async_wait<1>();
  __syncthreads();
  uint32_t qa[4][4];
  {
    const int r = wq * 16 + (lane & 7) + ((lane >> 3) & 1) * 8;
#pragma unroll
    for (int kk = 0; kk < 4; ++kk) ldsm_x4(qa[kk], &sq[r * ATT_LD + kk * 16 + (lane >> 4) * 8]);
  }
  float o[8][4];
#pragma unroll
  for (int i = 0; i < 8; ++i) o[i][0] = o[i][1] = o[i][2] = o[i][3] = 0.f;
  float mrow[2] = {-INFINITY, -INFINITY}, lrow[2] = {0.f, 0.f};
  const int qrow0 = q0 + wq * 16 + (lane >> 2);
  for (int j = 0; j < npair; ++j) {
    if (j > 0) {
      cp_async_wait<1>();
      __syncthreads();
    }
    const int kt = G * j + grp;
    if (kt < nkt)
      attention_key_tile<T>(ktile(j & 1, grp), vtile(j & 1, grp), qa, o, mrow, lrow, kt * ATT_BK, qrow0, seq, causal,
                            scale_log2, lane);
    if (j + 2 < npair) {
      __syncthreads();  // both groups are done with stage j & 1
      load_pair(j + 2);
    }
    cp_async_commit();
  }
#pragma unroll
  for (int h = 0; h < 2; ++h) {  // full row sums across the 4 lanes of a row
    lrow[h] += __shfl_xor_sync(0xffffffffu, lrow[h], 1);
    lrow[h] += __shfl_xor_sync(0xffffffffu, lrow[h], 2);
  }
  // merge: group 1 publishes its state per (warp, lane) -- the same fragment elements as the
  // group-0 lane that merges it
  cp_async_wait<0>();
  __syncthreads();
  float* xs = reinterpret_cast<float*>(kv);  // [G-1 groups][4 warps][32 lanes][36]
  if (grp > 0) {
    float* mine = xs + (((grp - 1) * 4 + wq) * 32 + lane) * 36;
#pragma unroll
    for (int db = 0; db < 8; ++db)
#pragma unroll
      for (int e = 0; e < 4; ++e) mine[db * 4 + e] = o[db][e];
    mine[32] = mrow[0], mine[33] = mrow[1], mine[34] = lrow[0], mine[35] = lrow[1];
  }
  __syncthreads();
  if (grp > 0) return;
  // group 0 merges the groups in order 1..G-1 (deterministic)
  float inv[2];
#pragma unroll
  for (int g = 1; g < G; ++g) {
    const float* ot = xs + (((g - 1) * 4 + wq) * 32 + lane) * 36;
#pragma unroll
    for (int h = 0; h < 2; ++h) {
      const float m1 = ot[32 + h], l1 = ot[34 + h];
      const float m = fmaxf(mrow[h], m1);
      const float a0 = (mrow[h] == -INFINITY) ? 0.f : exp2f(mrow[h] - m);
      const float a1 = (m1 == -INFINITY) ? 0.f : exp2f(m1 - m);
      lrow[h] = lrow[h] * a0 + l1 * a1;
      mrow[h] = m;
#pragma unroll
      for (int db = 0; db < 8; ++db) {
        o[db][2 * h] = o[db][2 * h] * a0 + ot[db * 4 + 2 * h] * a1;
        o[db][2 * h + 1] = o[db][2 * h + 1] * a0 + ot[db * 4 + 2 * h + 1] * a1;
      }
    }
  }
#pragma unroll
  for (int h = 0; h < 2; ++h) inv[h] = lrow[h] > 0.f ? 1.f / lrow[h] : 0.f;
  T* cbase = ctx + tok0 * H + head * ATT_D;
#pragma unroll
  for (int db = 0; db < 8; ++db) {
    const int col = db * 8 + (lane & 3) * 2;
    float v[4];
#pragma unroll
    for (int e = 0; e < 4; ++e) v[e] = o[db][e] * inv[e >> 1];
    if (qrow0 < seq) *reinterpret_cast<uint32_t*>(cbase + (size_t)qrow0 * H + col) = Cvt<T>::from2(v[0], v[1]);
    if (qrow0 + 8 < seq)
      *reinterpret_cast<uint32_t*>(cbase + (size_t)(qrow0 + 8) * H + col) = Cvt<T>::from2(v[2], v[3]);
  }
}

void launch_attention(int dtype, const void* qkv, int ldqkv, void* ctx, int batch, int seq, int H, int heads,
                      bool causal, cudaStream_t s, int tc_mode) {
  if (ablate_mask() & 1) return;
  DP_CHECK(heads > 0 && H % heads == 0 && H / heads == ATT_D, DP_ERR_UNSUPPORTED, "attention needs head dim 64");
  DP_CHECK(ldqkv % 8 == 0, DP_ERR_INVALID, "ldqkv must be a multiple of 8");
  if (batch <= 0 || seq <= 0) return;
  if (dtype == DP_FP32) {
    launch_attention_f32(qkv, ldqkv, ctx, batch, seq, H, heads, causal, s);
    return;
  }
  // K5t (tcgen05, attn_tc.cu) from 384 tokens (tc_mode 0) or when forced (1).  Warm forwards, K5t
  // vs K5 / K5b: GPT-2 Medium S1024 1.82 vs 2.01 ms, BERT-Large S384 1.347 vs 1.362, GPT-2 S512
  // 0.631 vs 0.652; below 384 tokens the mma.sync kernels win (GPT-2 S256 0.550 vs 0.505, BERT-Base
  // S128 0.475 vs 0.465; profiles/r02_warm_attention_tc.jsonl)
  const bool use_tc = tc_mode == 1 || (tc_mode == 0 && seq >= 384);
  if (use_tc && attention_tc_supported(ldqkv, H, heads, qkv)) {
    launch_attention_tc(dtype, qkv, ldqkv, ctx, batch, seq, H, heads, causal, s);
    return;
  }
  dim3 grid((seq + ATT_BQ - 1) / ATT_BQ, heads, batch);
  const float scale_log2 = 1.4426950408889634f / sqrtf((float)ATT_D);
  static const int env_att = experiment_env("DP_ATT_GROUPS", 0);  // experiments
  // >= 3 key tiles: 2 or 4 key-tile groups per query tile (K5b).  At 2 tiles (BERT-Base
  // S = 128) the merge and the larger footprint cost more than the shorter chain saves (warm
  // forward 0.480 vs 0.472 ms); with 2 groups BERT-Large S = 384 1.78 -> 1.58 ms, GPT-2 Medium
  // S = 1024 2.81 -> 2.47 ms
  auto run_groups = [&](auto gtag) {
    constexpr int G = decltype(gtag)::value;
    constexpr int smem = att_groups_smem<G>();
    static std::atomic<unsigned> attr{0};
    if (first_on_device(attr)) {
      DP_CUDA(cudaFuncSetAttribute(attention2_kernel<__half, G>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
      DP_CUDA(cudaFuncSetAttribute(attention2_kernel<__nv_bfloat16, G>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                   smem));
    }
    const dim3 g2(heads, grid.x, batch);
    static const int env_lpt = experiment_env("DP_ATT_LPT", 1);  // experiments
    const int cmode = causal ? (env_lpt ? 2 : 1) : 0;  // 2: causal, longest query tiles first
    if (dtype == DP_BF16)
      launch_kernel(attention2_kernel<__nv_bfloat16, G>, g2, dim3(128 * G), smem, s, (const __nv_bfloat16*)qkv,
                    ldqkv, (__nv_bfloat16*)ctx, seq, H, cmode, scale_log2);
    else
      launch_kernel(attention2_kernel<__half, G>, g2, dim3(128 * G), smem, s, (const __half*)qkv, ldqkv,
                    (__half*)ctx, seq, H, cmode, scale_log2);
  };
  // groups by key tiles (DP_ATT_GROUPS forces 1 / 2 / 4 for experiments): >= 4 tiles -> 4
  // groups (BERT-Large S384 warm 1.58 -> 1.48 ms; GPT-2 Medium S1024 unchanged), 3 -> 2
  const int nkt = (seq + ATT_BK - 1) / ATT_BK;
  // causal: 2 groups (2 CTAs per SM fit; GPT-2 S256 0.542 vs 0.554 ms with 4, S1024 equal)
  const int groups = env_att > 0 ? env_att : causal ? (nkt >= 3 ? 2 : 1) : (nkt >= 4 ? 4 : nkt == 3 ? 2 : 1);
  if (groups == 4 && nkt >= 3) {
    run_groups(std::integral_constant<int, 4>{});
    return;
  }
  if (groups == 2 && nkt >= 3) {
    run_groups(std::integral_constant<int, 2>{});
    return;
  }
  if (dtype == DP_BF16)
    launch_kernel(attention_kernel<__nv_bfloat16>, grid, dim3(128), 0, s, (const __nv_bfloat16*)qkv, ldqkv,
                  (__nv_bfloat16*)ctx, seq, H, causal ? 1 : 0, scale_log2);
  else
    launch_kernel(attention_kernel<__half>, grid, dim3(128), 0, s, (const __half*)qkv, ldqkv, (__half*)ctx, seq, H,
                  causal ? 1 : 0, scale_log2);
}

// -------------------------------------------------------------------------------------
// K3 (M > 16 tokens): the DHA skinny linear with its products on mma.sync.
//
// The cost is set by the host link: one host round trip (~7 us measured on this box,
// profiles/r01_linkprobe.json zc_gather) plus W bytes at ~51 GB/s.  Everything else must
// hide under that.  Each CTA owns 16 W rows x a K slice KS = K / cs (cs = cluster size,
// chosen so KS <= 768):
//   1. its whole W slice (<= 6 x 16-byte loads per thread, coalesced) is issued into
//      registers before the grid-dependency wait -- weights never depend on the previous
//      kernel, so under PDL these host reads overlap the predecessor's tail;
//   2. right after the wait, the first X chunks ([128 tokens][64 k], from L2) go into a
//      4-stage cp.async ring, so X staging overlaps the W round trip;
//   3. the registers land in padded shared memory ([16][KS+8], conflict-free ldmatrix);
//   4. per chunk: ldmatrix A = W rows, B = X rows, two m16n8k16 per warp (16 tokens).
//   5. cs > 1: the fp32 partial tiles are summed across the cluster through distributed
//      shared memory in rank order 0..cs-1 (deterministic; each rank finishes a share of
//      the tokens), then bias / activation / residual.
// Host-link bytes = N*K*2 + N*2 exactly; the kernel is the same whether W lives in host or
// device memory, so DHA and loaded execution of a layer are bit-identical.
// -------------------------------------------------------------------------------------
constexpr int SK_TOK = 128;  // tokens per block (8 warps x 16)
constexpr int SK_KCH = 64;   // K elements per X chunk
constexpr int SK_STG = 4;    // cp.async ring depth
constexpr int SK_XP = SK_KCH + 8;
constexpr int SK_WREG = 6;   // W vectors per thread: 16 rows x 768 / 8 / 256

__device__ __forceinline__ uint32_t cluster_rank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
__device__ __forceinline__ void cluster_sync_all() {
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
__device__ __forceinline__ void cluster_sync_relaxed() {  // exit barrier: no release fence needed
  asm volatile("barrier.cluster.arrive.relaxed.aligned;\n\tbarrier.cluster.wait.aligned;" ::: "memory");
}
__device__ __forceinline__ float ld_dsmem_f32(const float* p, uint32_t rank) {
  uint32_t a = static_cast<uint32_t>(__cvta_generic_to_shared(p)), ra;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(ra) : "r"(a), "r"(rank));
  float v;
  asm volatile("ld.shared::cluster.f32 %0, [%1];" : "=f"(v) : "r"(ra) : "memory");
  return v;
}

template <class T>
__global__ void __launch_bounds__(256) skinny_mma_kernel(const T* __restrict__ X, int ldx, const T* W,
                                                         const T* bias, const void* res, int ldr, void* Y, int ldy,
                                                         int M, int N, int K, int KS, int cs, int act, int io) {
  extern __shared__ __align__(16) uint8_t smem_sk[];
  const int KP = KS + 8;
  T* sw = reinterpret_cast<T*>(smem_sk);  // W slice [16][KS + 8]
  T* sx = sw + 16 * KP;                   // X ring [SK_STG][SK_TOK][SK_XP]
  float* red = reinterpret_cast<float*>(sx);  // cs > 1: partial tile [SK_TOK][16], aliases the ring
  pdl_trigger();
  const int rank = cs > 1 ? (int)cluster_rank() : 0;
  const int n0 = (blockIdx.x / cs) * 16;
  const int k0 = rank * KS;
  const int kv = KS / 8;
  // (1) the W slice, all in flight at once
  uint4 wr[SK_WREG];
#pragma unroll
  for (int j = 0; j < SK_WREG; ++j) {
    const int i = threadIdx.x + j * 256;
    if (i < 16 * kv) wr[j] = ldg16(W + (size_t)(n0 + i / kv) * K + k0 + (i % kv) * 8);
  }
  float breg = 0.f;
  if (bias && threadIdx.x < 16) breg = Cvt<T>::to1(bias[n0 + threadIdx.x]);
  __shared__ float sbias[16];
  pdl_wait();
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int g = lane >> 2, t4 = lane & 3;
  const int nch = KS / SK_KCH + (KS % SK_KCH ? 1 : 0);
  auto stage = [&](int t0, int nt, int c) {  // X chunk c of token block t0 -> ring slot c % SK_STG
    T* dst = sx + (c % SK_STG) * SK_TOK * SK_XP;
    const int kc = k0 + c * SK_KCH, kw = min(SK_KCH, KS - c * SK_KCH);
    for (int i = threadIdx.x; i < SK_TOK * (SK_KCH / 8); i += 256) {
      const int r = i / (SK_KCH / 8), q = i % (SK_KCH / 8);
      if (r < nt && q * 8 < kw) cp_async16(dst + r * SK_XP + q * 8, X + (size_t)(t0 + r) * ldx + kc + q * 8);
    }
  };
  const T* arow = &sw[(lane & 15) * KP + (lane >> 4) * 8];
  const int brow_off = (16 * warp + (lane & 7) + ((lane >> 4) << 3)) * SK_XP + ((lane >> 3) & 1) * 8;
  for (int t0 = 0; t0 < M; t0 += SK_TOK) {
    const int nt = min(SK_TOK, M - t0);
    // (2) prefetch the first chunks
#pragma unroll
    for (int c = 0; c < SK_STG - 1; ++c) {
      if (c < nch) stage(t0, nt, c);
      cp_async_commit();
    }
    if (t0 == 0) {  // (3) W registers -> shared (waits for the host round trip)
#pragma unroll
      for (int j = 0; j < SK_WREG; ++j) {
        const int i = threadIdx.x + j * 256;
        if (i < 16 * kv) *reinterpret_cast<uint4*>(&sw[(i / kv) * KP + (i % kv) * 8]) = wr[j];
      }
      if (threadIdx.x < 16) sbias[threadIdx.x] = breg;
    }
    float acc[2][4] = {{0.f, 0.f, 0.f, 0.f}, {0.f, 0.f, 0.f, 0.f}};
    // (4) the ring
    for (int c = 0; c < nch; ++c) {
      cp_async_wait<SK_STG - 2>();
      __syncthreads();  // chunk c visible to all; slot (c-1) % SK_STG free
      if (c + SK_STG - 1 < nch) stage(t0, nt, c + SK_STG - 1);
      cp_async_commit();
      if (16 * warp < nt) {
        const T* xs = sx + (c % SK_STG) * SK_TOK * SK_XP + brow_off;
        const int kw = min(SK_KCH, KS - c * SK_KCH);
#pragma unroll
        for (int ks = 0; ks < SK_KCH; ks += 16) {
          if (ks < kw) {
            uint32_t a[4], b[4];
            ldsm_x4(a, arow + c * SK_KCH + ks);
            ldsm_x4(b, xs + ks);
            MmaOp<T>::mma(acc[0], a, b);
            MmaOp<T>::mma(acc[1], a, b + 2);
          }
        }
      }
    }
    cp_async_wait<0>();
    __syncthreads();  // every warp is done with the ring (it is reused below / next block)
    // acc[q]: c0,c1 -> W row g, tokens 2*t4, 2*t4+1 of group q; c2,c3 -> W row g+8
    if (cs == 1) {
#pragma unroll
      for (int q = 0; q < 2; ++q) {
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          const int r = g + (e >> 1) * 8;
          const int m = t0 + 16 * warp + 8 * q + 2 * t4 + (e & 1);
          if (m < M) {
            const int n = n0 + r;
            float v = apply_act(acc[q][e] + sbias[r], act);
            if (res) v += load1<T>(res, (size_t)m * ldr + n, io & IO_RES_F32);
            store1<T>(Y, (size_t)m * ldy + n, v, io & IO_OUT_F32);
          }
        }
      }
    } else {
      // (5) deterministic cluster reduction over distributed shared memory
#pragma unroll
      for (int q = 0; q < 2; ++q)
#pragma unroll
        for (int e = 0; e < 4; ++e)
          red[(16 * warp + 8 * q + 2 * t4 + (e & 1)) * 16 + g + (e >> 1) * 8] = acc[q][e];
      cluster_sync_all();
      const int per = ((SK_TOK + cs - 1) / cs) * 16;  // elements (token-major, 16 rows each) per rank
      const int lo = rank * per, hi = min(SK_TOK * 16, lo + per);
      for (int i = lo + threadIdx.x; i < hi; i += 256) {
        const int tok = i >> 4, r = i & 15, m = t0 + tok;
        if (m >= M) continue;
        float v = 0.f;
        for (int s = 0; s < cs; ++s) v += ld_dsmem_f32(red + i, (uint32_t)s);
        const int n = n0 + r;
        v = apply_act(v + sbias[r], act);
        if (res) v += load1<T>(res, (size_t)m * ldr + n, io & IO_RES_F32);
        store1<T>(Y, (size_t)m * ldy + n, v, io & IO_OUT_F32);
      }
      cluster_sync_relaxed();  // peers have read this CTA's partials before the ring is reused / exit
    }
  }
}

// the K-slice split: smallest cluster size with a slice of at most 768 elements
int skinny_cluster(int K) {
  for (int cs = 1; cs <= 8; ++cs)
    if (K % (16 * cs) == 0 && K / cs <= 768) return cs;
  return 0;
}

template <class T>
void skinny_mma_t(const void* x, int ldx, const void* w, const void* bias, const void* res, int ldr, void* y, int ldy,
                  int M, int N, int K, int act, int io, cudaStream_t s) {
  const int cs = skinny_cluster(K);
  DP_CHECK(cs > 0, DP_ERR_UNSUPPORTED, "skinny linear: K must split into <= 8 slices of <= 768 (multiples of 16)");
  const int KS = K / cs;
  const size_t sm = (size_t(16) * (KS + 8) + size_t(SK_STG) * SK_TOK * SK_XP) * sizeof(T);
  static std::atomic<unsigned> attr_set{0};  // one per template instantiation
  if (first_on_device(attr_set)) {
    DP_CUDA(cudaFuncSetAttribute(skinny_mma_kernel<T>, cudaFuncAttributeMaxDynamicSharedMemorySize, 160 * 1024));
    DP_CUDA(cudaFuncSetAttribute(skinny_mma_kernel<T>, cudaFuncAttributeNonPortableClusterSizeAllowed, 1));
  }
  launch_kernel_cluster(skinny_mma_kernel<T>, dim3((N / 16) * cs), dim3(256), sm, dim3(cs, 1, 1), s, (const T*)x, ldx,
                        (const T*)w, (const T*)bias, res, ldr, y, ldy, M, N, K, KS, cs, act, io);
}

// -------------------------------------------------------------------------------------
// L2 flush for profiling (Exe(DHA) measured with cold caches, SURVEY hard part 6)
// -------------------------------------------------------------------------------------
__global__ void l2_flush_kernel(uint4* buf, size_t n16) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n16; i += (size_t)gridDim.x * blockDim.x)
    buf[i] = make_uint4((uint32_t)i, 0, 0, 0);
}

void launch_l2_flush(void* buf, size_t bytes, cudaStream_t s) {
  l2_flush_kernel<<<148 * 4, 512, 0, s>>>((uint4*)buf, bytes / 16);
  DP_CUDA(cudaGetLastError());
}

// Fault injection (tests): occupy a stream for `cycles` SM cycles.
__global__ void spin_kernel(long long cycles) {
  const long long t0 = clock64();
  while (clock64() - t0 < cycles) {
  }
}

__global__ void timestamp_kernel(uint64_t* slot) {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  *slot = t;
}

void launch_timestamp(uint64_t* slot, cudaStream_t s) {
  timestamp_kernel<<<1, 1, 0, s>>>(slot);
  DP_CUDA(cudaGetLastError());
}

void launch_spin(long long cycles, cudaStream_t s) {
  spin_kernel<<<1, 1, 0, s>>>(cycles);
  DP_CUDA(cudaGetLastError());
}

}  // namespace dp
