// K6: persistent layer-program kernel -- every transformer layer of a forward pass in ONE
// launch (SURVEY §8(a) a12-a14 on the warm / resident path).
//
// Why: at the hot path's token counts (B*S = 128..384) each resident layer is ~14 MB of
// weights and ~2 GFLOP, i.e. ~2 us of HBM time on B200, but the per-kernel chain (7 launches a
// layer, each paying launch, prologue, first-TMA latency and a drained tail) costs ~40 us a
// layer.  Here one CTA per SM (grid = #SMs, cooperative launch => co-resident) walks a
// host-built program of ops separated by grid barriers, and the weight tiles of the next GEMM
// op stream into shared memory while the current op (a reduction, the attention core) runs.
//
// Ops (built by build_persist_program from the model's units; K6):
//   GEMM    part[split][M][g*N + n] = X[M, krange] . W_g[n, krange]^T     (fp32 partials)
//           swap-AB tcgen05 tiles as in K2: W rows on the MMA's M = 128 TMEM lanes, tokens on
//           N = bn; items = groups x N/128 x ceil(M/bn) x splits, round-robin over the CTAs.
//   REDUCE  z = sum_s part[s] (or a plain input) + bias (+ residual); then either act(z) or
//           LayerNorm(z) (one warp per row, fp32 two-pass statistics) -> storage dtype;
//           optionally z itself (GPT-2's fp32 residual stream).
//   ATTN    the K5 flash-attention tile (attn.cuh) on the 4 compute warps.
// Warp roles (192 threads): warp 4 lane 0 = TMA producer, warp 5 lane 0 = MMA issuer (both
// walk the GEMM ops of the program independently, ahead of the compute warps), warps 0-3 =
// TMEM epilogue / reductions / attention / the grid barrier.  Pipelines: smem full/empty
// (TMA <-> MMA), TMEM full/empty (MMA <-> epilogue, two 128-column accumulators), and the
// per-op epoch (compute warps -> producer: an op's activations may be read only after the
// grid barrier that ends the previous op).  Every wait is bounded: a stuck pipeline traps
// (a launch error) instead of hanging the GPU.
#include <cuda.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <memory>
#include <vector>

#include "attn.cuh"
#include "common.h"
#include "dtype.cuh"
#include "engine.h"
#include "kernels.h"
#include "launch.cuh"
#include "persist.h"
#include "tc.cuh"

namespace dp {

namespace {

constexpr int PBM = 128;                    // W rows per tile (MMA M, TMEM lanes)
constexpr int PBK = 64;                     // K per stage (one 128-byte swizzle row)
constexpr int PBN_MAX = 64;                 // token tile (MMA N) at most
constexpr int P_STAGES = 6;                 // smem ring depth
constexpr uint32_t P_A_BYTES = PBM * PBK * 2;        // 16 KB W tile
constexpr uint32_t P_B_MAX = PBN_MAX * PBK * 2;      // 8 KB X tile (bn <= 64)
constexpr uint32_t P_STAGE = P_A_BYTES + P_B_MAX;    // 24 KB
constexpr uint32_t P_ATT_ELEMS = (ATT_BQ + 4 * ATT_BK) * ATT_LD;  // sq | sk[2] | sv[2]
constexpr uint32_t P_TMEM_COLS = 2 * PBN_MAX;        // two accumulators
constexpr int P_THREADS = 192;

enum { POP_GEMM = 0, POP_REDUCE = 1, POP_ATTN = 2 };
enum { PG_PARTIAL = 0, PG_FINAL = 1 };  // GEMM epilogue: fp32 split partials | bias+act -> storage dtype

}  // namespace

// One op of the program (device memory; read by every CTA).
struct POp {
  int type;
  // GEMM
  int wmap, xmap, groups;  // W maps wmap .. wmap+groups-1 share X
  int M, N, K, splits, bn, mtiles, ntiles, items;
  int mode, omap;          // PG_PARTIAL: TMA store into part [splits][M][groups*N] (3D fp32 map);
                           // PG_FINAL (splits 1): act(acc + bias) -> out (2D map), bias/act below
  float* part;
  // REDUCE
  int rows, cols, rsplits, act, in_f32, res_f32, zout_f32, out_final, bias_w;
  const float* rpart;      // [rsplits][rows][cols]; rsplits == 0: z = in
  const void* in;
  const void* bias0;       // column c uses bias{c / bias_w}[c % bias_w]
  const void* bias1;
  const void* bias2;
  const void* res;         // [rows][cols] or nullptr
  const void* gamma;       // LayerNorm when non-null (cols <= 1024)
  const void* beta;
  float eps;
  void* zout;              // optional z (pre-LN) [rows][cols]
  float* out32;            // optional fp32 copy of the LayerNorm output (BERT residual stream)
  void* out;               // [rows][cols] storage dtype (out_final: the kernel's `final_out`)
  // ATTN
  const void* qkv;
  void* ctx;
  int batch, seq, H, heads, causal;
  float scale_log2;
};

namespace {

__device__ __forceinline__ unsigned long long gtime() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

#ifdef DP_PERSIST_TRACE
// per CTA, per op: [0] op start (compute warps), [1] work done (before the grid barrier),
// [2] GEMM: first accumulator ready (X landed + MMAs done), [3] work issued (before the fences)
constexpr int P_TR_OPS = 512;
__device__ unsigned long long g_persist_trace[160][P_TR_OPS][8];
#define PTRACE(o, i)                                                             \
  do {                                                                           \
    if (threadIdx.x == 0 && (o) < P_TR_OPS) g_persist_trace[blockIdx.x][o][i] = gtime(); \
  } while (0)
#else
#define PTRACE(o, i) \
  do {               \
  } while (0)
#endif

// Bounded mbarrier wait: ~2 s without progress is a bug (trap => launch error, not a hang).
__device__ __forceinline__ void mbar_wait_bounded(uint64_t* bar, uint32_t phase) {
  const uint32_t a = smem_u32(bar);
  uint32_t ok = 0;
  unsigned long long t0 = 0;
  for (int it = 0;; ++it) {
    asm volatile(
        "{\n"
        ".reg .pred P1;\n"
        "mbarrier.try_wait.parity.shared::cta.b64 P1, [%1], %2;\n"
        "selp.u32 %0, 1, 0, P1;\n"
        "}\n"
        : "=r"(ok)
        : "r"(a), "r"(phase)
        : "memory");
    if (ok) return;
    if ((it & 1023) == 1023) {
      const unsigned long long t = gtime();
      if (t0 == 0) t0 = t;
      else if (t - t0 > 2000000000ull) __trap();
    }
  }
}

__device__ __forceinline__ void named_sync(int id, int n) {
  asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(n) : "memory");
}

__device__ __forceinline__ unsigned ld_acquire_gpu(const unsigned* p) {
  unsigned v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}

__device__ __forceinline__ void fence_proxy_async_global() {
  asm volatile("fence.proxy.async.global;" ::: "memory");
}

struct ItemCoord {
  int g, nt, mt, sp, kb_lo, kb_n;
};

// item -> (group, n-tile, m-tile, split) and its K-block range
__device__ __forceinline__ ItemCoord decode_item(const POp& op, int item) {
  ItemCoord c;
  c.sp = item % op.splits;
  int r = item / op.splits;
  c.mt = r % op.mtiles;
  r /= op.mtiles;
  c.nt = r % op.ntiles;
  c.g = r / op.ntiles;
  const int kb_all = op.K / PBK;
  c.kb_lo = c.sp * kb_all / op.splits;
  c.kb_n = (c.sp + 1) * kb_all / op.splits - c.kb_lo;
  return c;
}

// element i of a storage-dtype / fp32 array written earlier in this grid: through L2 (a line
// this SM cached in L1 during an earlier op may be stale)
template <class T>
__device__ __forceinline__ float ld1_cg(const void* base, size_t i, int f32) {
  if (f32) return __ldcg(static_cast<const float*>(base) + i);
  const unsigned short u = __ldcg(reinterpret_cast<const unsigned short*>(static_cast<const T*>(base) + i));
  T v;
  memcpy(&v, &u, 2);
  return Cvt<T>::to1(v);
}

// bias element c of a REDUCE op (weights: never written inside the grid)
template <class T>
__device__ __forceinline__ float bias_at(const POp& op, int c) {
  const int g = c / op.bias_w;
  const void* b = g == 0 ? op.bias0 : (g == 1 ? op.bias1 : op.bias2);
  return Cvt<T>::to1(static_cast<const T*>(b)[c - g * op.bias_w]);
}

// z for row r at the V columns c0 + 128*e (e < V) of the calling thread: the split partials
// (or the plain input) + bias (+ residual).  All loads of a group of 4 splits are issued
// before any is summed (the reduction is latency-bound: ~V*S independent L2 reads per
// thread); the sum order is split 0, 1, ..., S-1 regardless (deterministic).
template <class T, int V>
__device__ __forceinline__ void reduce_cols(const POp& op, int r, int c0, float* z) {
  const size_t row = (size_t)r * op.cols;
  if (op.rsplits > 0) {
    const size_t slice = (size_t)op.rows * op.cols;
    const float* p = op.rpart + row + c0;
#pragma unroll
    for (int e = 0; e < V; ++e) z[e] = 0.f;
    int s = 0;
    for (; s + 4 <= op.rsplits; s += 4) {
      float v[4][V];
#pragma unroll
      for (int j = 0; j < 4; ++j)
#pragma unroll
        for (int e = 0; e < V; ++e) v[j][e] = __ldcg(p + (s + j) * slice + 128 * e);
#pragma unroll
      for (int j = 0; j < 4; ++j)
#pragma unroll
        for (int e = 0; e < V; ++e) z[e] += v[j][e];
    }
    for (; s < op.rsplits; ++s)
#pragma unroll
      for (int e = 0; e < V; ++e) z[e] += __ldcg(p + s * slice + 128 * e);
  } else {
#pragma unroll
    for (int e = 0; e < V; ++e) z[e] = load1<T>(op.in, row + c0 + 128 * e, op.in_f32);
  }
  if (op.bias0 != nullptr) {
#pragma unroll
    for (int e = 0; e < V; ++e) z[e] += bias_at<T>(op, c0 + 128 * e);
  }
  if (op.res != nullptr) {
#pragma unroll
    for (int e = 0; e < V; ++e) {
      const size_t i = row + c0 + 128 * e;
      z[e] += ld1_cg<T>(op.res, i, op.res_f32);
    }
  }
}

// LayerNorm rows: one CTA (the 128 compute threads) per row, thread t owns columns
// t + 128*e; fp32 two-pass statistics (mean, then the mean squared deviation) through shared
// memory.  V = cols / 128.
template <class T, int V>
__device__ __forceinline__ void reduce_ln_rows(const POp& op, int b, int G, void* out, float* red, int o) {
  const int t = threadIdx.x, lane = t & 31, warp = t >> 5;
  const float inv_n = 1.f / (float)op.cols;
  for (int r = b; r < op.rows; r += G) {
    float z[V];
    reduce_cols<T, V>(op, r, t, z);
#ifdef DP_PERSIST_TRACE
    if (r == b && t == 0) g_persist_trace[blockIdx.x][o][4] = gtime();
#endif
    const size_t row = (size_t)r * op.cols;
    if (op.zout != nullptr) {
#pragma unroll
      for (int e = 0; e < V; ++e) store1<T>(op.zout, row + t + 128 * e, z[e], op.zout_f32);
    }
    float sum = 0.f;
#pragma unroll
    for (int e = 0; e < V; ++e) sum += z[e];
    sum = warp_sum(sum);
    if (lane == 0) red[warp] = sum;
    named_sync(1, 128);
    const float mean = ((red[0] + red[1]) + (red[2] + red[3])) * inv_n;
    float sq = 0.f;
#pragma unroll
    for (int e = 0; e < V; ++e) {
      const float d = z[e] - mean;
      sq += d * d;
    }
    sq = warp_sum(sq);
    named_sync(1, 128);  // everyone has read red[] (the sums)
    if (lane == 0) red[warp] = sq;
    named_sync(1, 128);
    const float rstd = rsqrtf(((red[0] + red[1]) + (red[2] + red[3])) * inv_n + op.eps);
#pragma unroll
    for (int e = 0; e < V; ++e) {
      const int c = t + 128 * e;
      const float g = Cvt<T>::to1(static_cast<const T*>(op.gamma)[c]);
      const float be = Cvt<T>::to1(static_cast<const T*>(op.beta)[c]);
      const float y = (z[e] - mean) * rstd * g + be;
      static_cast<T*>(out)[row + c] = Cvt<T>::from1(y);
      if (op.out32 != nullptr) op.out32[row + c] = y;
    }
    named_sync(1, 128);  // red[] free for the next row
  }
}

// element-wise REDUCE (no LayerNorm): one warp per (row, 32*VEC-column chunk); a lane owns
// VEC consecutive columns (float4 partial loads, one 8/16-byte store); all loads of a group
// of 4 splits in flight before they are summed in split order.
template <class T, int VEC>
__device__ __forceinline__ void reduce_elementwise(const POp& op, int b, int G, void* out) {
  const int lane = threadIdx.x & 31;
  const int gw = b * 4 + (threadIdx.x >> 5), nw = G * 4;
  const int chunks = op.cols / (32 * VEC);
  const int total = op.rows * chunks;
  const size_t slice = (size_t)op.rows * op.cols;
  for (int i = gw; i < total; i += nw) {
    const int r = i / chunks;
    const int c = (i - r * chunks) * (32 * VEC) + lane * VEC;
    const size_t off = (size_t)r * op.cols + c;
    float z[VEC];
    if (op.rsplits > 0) {
#pragma unroll
      for (int e = 0; e < VEC; ++e) z[e] = 0.f;
      const float4* p = reinterpret_cast<const float4*>(op.rpart + off);
      const size_t sl4 = slice / 4;
      int s = 0;
      for (; s + 4 <= op.rsplits; s += 4) {
        float4 v[4][VEC / 4];
#pragma unroll
        for (int j = 0; j < 4; ++j)
#pragma unroll
          for (int q = 0; q < VEC / 4; ++q) v[j][q] = __ldcg(p + (s + j) * sl4 + q);
#pragma unroll
        for (int j = 0; j < 4; ++j)
#pragma unroll
          for (int q = 0; q < VEC / 4; ++q) {
            z[4 * q] += v[j][q].x, z[4 * q + 1] += v[j][q].y, z[4 * q + 2] += v[j][q].z, z[4 * q + 3] += v[j][q].w;
          }
      }
      for (; s < op.rsplits; ++s)
#pragma unroll
        for (int q = 0; q < VEC / 4; ++q) {
          const float4 v = __ldcg(p + s * sl4 + q);
          z[4 * q] += v.x, z[4 * q + 1] += v.y, z[4 * q + 2] += v.z, z[4 * q + 3] += v.w;
        }
    } else {
#pragma unroll
      for (int e = 0; e < VEC; ++e) z[e] = load1<T>(op.in, off + e, op.in_f32);
    }
    uint32_t packed[VEC / 2];
#pragma unroll
    for (int e = 0; e < VEC; e += 2) {
      float v0 = z[e], v1 = z[e + 1];
      if (op.bias0 != nullptr) v0 += bias_at<T>(op, c + e), v1 += bias_at<T>(op, c + e + 1);
      if (op.res != nullptr) v0 += ld1_cg<T>(op.res, off + e, op.res_f32), v1 += ld1_cg<T>(op.res, off + e + 1, op.res_f32);
      packed[e / 2] = Cvt<T>::from2(apply_act(v0, op.act), apply_act(v1, op.act));
    }
    if constexpr (VEC == 8)
      *reinterpret_cast<uint4*>(static_cast<T*>(out) + off) = make_uint4(packed[0], packed[1], packed[2], packed[3]);
    else
      *reinterpret_cast<uint2*>(static_cast<T*>(out) + off) = make_uint2(packed[0], packed[1]);
  }
}

template <class T>
__device__ __forceinline__ void run_reduce(const POp& op, int b, int G, void* final_out, float* red, int o) {
  void* out = op.out_final ? final_out : op.out;
  if (op.gamma != nullptr) {
    switch (op.cols / 128) {
      case 1: reduce_ln_rows<T, 1>(op, b, G, out, red, o); break;
      case 2: reduce_ln_rows<T, 2>(op, b, G, out, red, o); break;
      case 4: reduce_ln_rows<T, 4>(op, b, G, out, red, o); break;
      case 6: reduce_ln_rows<T, 6>(op, b, G, out, red, o); break;
      case 8: reduce_ln_rows<T, 8>(op, b, G, out, red, o); break;
      default: __trap();  // rejected on the host (persist_supported)
    }
    return;
  }
  if (op.cols % 256 == 0) reduce_elementwise<T, 8>(op, b, G, out);
  else reduce_elementwise<T, 4>(op, b, G, out);
}

template <class T>
__global__ void __launch_bounds__(P_THREADS, 1)
    persist_kernel(const POp* __restrict__ ops, int nops, const CUtensorMap* __restrict__ maps, unsigned* gbar,
                   void* final_out, int flags) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  uint8_t* ring = smem;
  T* att = reinterpret_cast<T*>(smem + P_STAGES * P_STAGE);
  __shared__ __align__(8) uint64_t full_bar[P_STAGES], empty_bar[P_STAGES], tfull[2], tempty[2];
  __shared__ uint32_t tmem_base_sh;
  __shared__ volatile int epoch;
  __shared__ float red[4];  // LayerNorm row statistics (compute warps)

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int G = gridDim.x, b = blockIdx.x;
  if (threadIdx.x == 0) {
    for (int s = 0; s < P_STAGES; ++s) {
      mbar_init(&full_bar[s], 1);
      mbar_init(&empty_bar[s], 1);
    }
    for (int i = 0; i < 2; ++i) {
      mbar_init(&tfull[i], 1);
      mbar_init(&tempty[i], 4);  // one arrival per epilogue warp
    }
    epoch = 0;
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&tmem_base_sh)),
                 "r"(P_TMEM_COLS));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tmem = tmem_base_sh;

  if (warp == 4) {
    // ===== TMA producer =====
    if (lane == 0) {
      uint32_t t = 0;  // ring task counter (one task = one K block of one item)
      auto issue_w = [&](const POp& op, const ItemCoord& c, int kb, uint32_t task) {
        const int s = task % P_STAGES;
        if (task >= (uint32_t)P_STAGES) mbar_wait_bounded(&empty_bar[s], ((task / P_STAGES) - 1) & 1);
        mbar_expect_tx(&full_bar[s], P_A_BYTES + uint32_t(op.bn) * PBK * 2);
        tma_load_2d(maps + op.wmap + c.g, &full_bar[s], ring + s * P_STAGE, (c.kb_lo + kb) * PBK, c.nt * PBM);
      };
      for (int o = 0; o < nops; ++o) {
        const POp op = ops[o];  // by value: fields live in registers (asm memory clobbers would force reloads)
        if (op.type != POP_GEMM) continue;
        asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(maps + op.xmap)) : "memory");
        // pass A: weights never depend on earlier ops.  Every W tile of this CTA's items is
        // prefetched into L2 now (HBM latency hidden under the ops still running), and the
        // first ring's worth is loaded into shared memory
        for (int item = b; item < op.items; item += G) {
          const ItemCoord c = decode_item(op, item);
          for (int kb = 0; kb < c.kb_n; ++kb)
            tma_prefetch_l2_2d(maps + op.wmap + c.g, (c.kb_lo + kb) * PBK, c.nt * PBM);
        }
        uint32_t tw = t;
        {
          int item = b, kb = 0;
          while (item < op.items && tw - t < (uint32_t)P_STAGES) {
            const ItemCoord c = decode_item(op, item);
            issue_w(op, c, kb, tw++);
            if (++kb == c.kb_n) kb = 0, item += G;
          }
        }
        // pass B: activations only after the grid barrier that ends op o-1
        {
          unsigned long long t0 = 0;
          for (int it = 0; epoch < o; ++it) {
            __nanosleep(64);  // a hot spin would steal issue slots from compute warp 0 (same SMSP)
            if ((it & 1023) == 1023) {
              const unsigned long long tt = gtime();
              if (t0 == 0) t0 = tt;
              else if (tt - t0 > 2000000000ull) __trap();
            }
          }
        }
        __threadfence();
        fence_proxy_async_global();
        int item = b, kb = 0;
        while (item < op.items) {
          const ItemCoord c = decode_item(op, item);
          if (t == tw) issue_w(op, c, kb, tw++);
          const int s = t % P_STAGES;
          tma_load_2d(maps + op.xmap, &full_bar[s], ring + s * P_STAGE + P_A_BYTES, (c.kb_lo + kb) * PBK,
                      c.mt * op.bn);
          ++t;
          if (++kb == c.kb_n) kb = 0, item += G;
        }
      }
    }
  } else if (warp == 5) {
    // ===== MMA issuer =====
    if (lane == 0) {
      uint32_t t = 0, it = 0;
      for (int o = 0; o < nops; ++o) {
        const POp op = ops[o];  // by value: fields live in registers (asm memory clobbers would force reloads)
        if (op.type != POP_GEMM) continue;
        const uint32_t idesc = (1u << 4) | (FmtBits<T>::v << 7) | (FmtBits<T>::v << 10) |
                               (uint32_t(op.bn >> 3) << 17) | (uint32_t(PBM >> 4) << 24);
        for (int item = b; item < op.items; item += G, ++it) {
          const ItemCoord c = decode_item(op, item);
          const int buf = it & 1;
          if (it >= 2) mbar_wait_bounded(&tempty[buf], ((it >> 1) - 1) & 1);
          asm volatile("tcgen05.fence::after_thread_sync;");
          const uint32_t d = tmem + buf * PBN_MAX;
          for (int kb = 0; kb < c.kb_n; ++kb, ++t) {
            const int s = t % P_STAGES;
            mbar_wait_bounded(&full_bar[s], (t / P_STAGES) & 1);
            asm volatile("tcgen05.fence::after_thread_sync;");
            const uint64_t da = sw128_desc(ring + s * P_STAGE), db = sw128_desc(ring + s * P_STAGE + P_A_BYTES);
#pragma unroll
            for (int kk = 0; kk < PBK / 16; ++kk) umma_f16(d, da + 2 * kk, db + 2 * kk, idesc, (kb | kk) != 0);
            umma_commit(&empty_bar[s]);
          }
          umma_commit(&tfull[buf]);
        }
      }
    }
  } else {
    // ===== compute warps 0-3: epilogue, reductions, attention, grid barrier =====
    uint32_t eit = 0;
    unsigned target = 0;
    for (int o = 0; o < nops; ++o) {
      const POp op = ops[o];  // by value: fields live in registers (asm memory clobbers would force reloads)
      PTRACE(o, 0);
      if (o + 1 < nops) {
        // the next op's bias / gamma / beta (weights: independent of this op) into L2 now
        const POp& nx = ops[o + 1];
        const int n = nx.type == POP_REDUCE ? nx.cols : (nx.type == POP_GEMM ? nx.bias_w : 0);
        const int lines = (n * 2 + 127) / 128;
        const void* vec[5] = {nx.bias0, nx.bias1, nx.bias2, nx.gamma, nx.beta};
        for (int i = threadIdx.x + b * 128; i < 5 * lines; i += 128 * G) {
          const void* base = vec[i / lines];
          if (base != nullptr)
            asm volatile("prefetch.global.L2 [%0];" ::"l"(static_cast<const char*>(base) + (i % lines) * 128));
        }
      }
      if (op.type == POP_GEMM) {
        // TMEM -> registers (+ bias, act) -> staging tile in shared memory [bn][128] -> one TMA
        // bulk store per item (coalesced, asynchronous; the staging tile is the attention
        // scratch, free during GEMM ops)
        bool pending = false;
        const bool fin = op.mode == PG_FINAL;
        for (int item = b; item < op.items; item += G, ++eit) {
          const ItemCoord c = decode_item(op, item);
          const int buf = eit & 1;
          const int nl = warp * 32 + lane;  // this lane's W row within the tile
          float bz = 0.f;                   // FINAL: bias of this output column (prefetched)
          if (fin && op.bias0 != nullptr) bz = bias_at<T>(op, c.g * op.bias_w + c.nt * PBM + nl);
          mbar_wait_bounded(&tfull[buf], (eit >> 1) & 1);
          asm volatile("tcgen05.fence::after_thread_sync;");
          if (item == b) PTRACE(o, 2);
          if (pending) {  // the previous item's store has read the staging tile
            if (threadIdx.x == 0) bulk_wait_read0();
            named_sync(1, 128);
          }
#pragma unroll 1
          for (int c0 = 0; c0 < op.bn; c0 += 16) {
            uint32_t v[16];
            tmem_ld16(tmem + (uint32_t(warp * 32) << 16) + buf * PBN_MAX + c0, v);
            if (item == b && c0 == 0) PTRACE(o, 4);
            if (fin) {
              T* st = reinterpret_cast<T*>(att) + c0 * PBM + nl;
#pragma unroll
              for (int j = 0; j < 16; ++j) st[j * PBM] = Cvt<T>::from1(apply_act(__uint_as_float(v[j]) + bz, op.act));
            } else {
              float* st = reinterpret_cast<float*>(att) + c0 * PBM + nl;
#pragma unroll
              for (int j = 0; j < 16; ++j) st[j * PBM] = __uint_as_float(v[j]);
            }
          }
          if (item == b) PTRACE(o, 5);
          asm volatile("tcgen05.fence::before_thread_sync;");
          __syncwarp();
          if (lane == 0) mbar_arrive(&tempty[buf]);  // TMEM buffer free for the item after next
          asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // staging -> async proxy
          named_sync(1, 128);
          if (threadIdx.x == 0) {
            const int col = c.g * op.N + c.nt * PBM, row = c.mt * op.bn;
            if (fin) tma_store_2d(maps + op.omap, att, col, row);
            else tma_store_3d(maps + op.omap, att, col, row, c.sp);
            bulk_commit();
          }
          pending = true;
        }
        if (pending && threadIdx.x == 0) bulk_wait0();  // stores complete before the grid barrier
      } else if (op.type == POP_REDUCE) {
        run_reduce<T>(op, b, G, final_out, red, o);
      } else {  // POP_ATTN
        const int qtiles = (op.seq + ATT_BQ - 1) / ATT_BQ;
        const int items = qtiles * op.heads * op.batch;
        for (int item = b; item < items; item += G) {
          const int qt = item % qtiles, r = item / qtiles;
          attention_tile<T>(static_cast<const T*>(op.qkv), 3 * op.H, static_cast<T*>(op.ctx), op.seq, op.H,
                            op.causal, op.scale_log2, qt, r % op.heads, r / op.heads, att, att + ATT_BQ * ATT_LD,
                            att + (ATT_BQ + 2 * ATT_BK) * ATT_LD, threadIdx.x, [] { named_sync(1, 128); });
        }
      }
      PTRACE(o, 3);
      if (o + 1 < nops) {
        // grid barrier: this op's stores -> every CTA's next op (generic and TMA readers)
        if (!(flags & 1)) fence_proxy_async_global();
        named_sync(1, 128);
        PTRACE(o, 1);
        if (threadIdx.x == 0) {
          target += G;
          __threadfence();
          atomicAdd(gbar, 1u);
          unsigned long long t0 = 0;
          for (int it = 0; ld_acquire_gpu(gbar) < target; ++it) {
            if ((it & 255) == 255) {
              const unsigned long long tt = gtime();
              if (t0 == 0) t0 = tt;
              else if (tt - t0 > 2000000000ull) __trap();
            }
          }
          __threadfence();
          epoch = o + 1;
        }
        named_sync(1, 128);
      }
    }
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (warp == 0)
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(P_TMEM_COLS));
}

size_t persist_smem_bytes() { return size_t(P_STAGES) * P_STAGE + P_ATT_ELEMS * 2 + 1024; }

// (bn, splits) for a GEMM op from a per-CTA cost model (us): a CTA ingests its W + X tiles at
// ~100 GB/s and writes its fp32 partial tile at ~200 GB/s; the reduction reads every partial
// once, spread over all CTAs.  Single wave preferred.
struct PCfg {
  int bn, splits;
};
// (bn, splits) for a GEMM op from a per-CTA cost model (us): a CTA ingests its W + X tiles at
// ~100 GB/s (TMA, traced), an item costs ~0.5 us of first-load latency + epilogue, and a
// PARTIAL op's LayerNorm reduction pays ~0.7 us per group of 4 splits it sums (L2 round
// trips).  FINAL ops (bias/act in the epilogue, no reduction) run unsplit.  Single wave
// preferred.  DP_PERSIST_BN / DP_PERSIST_SPLIT override (sweeps).
PCfg pick_persist_cfg(int M, int Ntot, int K, int G, bool final_mode) {
  static const int env_bn = getenv("DP_PERSIST_BN") ? atoi(getenv("DP_PERSIST_BN")) : 0;
  static const int env_sp = getenv("DP_PERSIST_SPLIT") ? atoi(getenv("DP_PERSIST_SPLIT")) : 0;
  const int kb = K / PBK, ntile = Ntot / PBM;
  PCfg best{32, 1};
  double best_t = 1e30;
  for (int bn : {16, 32, 64}) {
    if (env_bn > 0 && bn != env_bn) continue;
    if (bn > 16 && M <= bn / 2) continue;
    const int mt = (M + bn - 1) / bn;
    for (int sp = 1; sp <= (final_mode ? 1 : kb); ++sp) {
      if (!final_mode && env_sp > 0 && sp != env_sp) continue;
      const int items = ntile * mt * sp;
      const int waves = (items + G - 1) / G;
      const double kbper = double(kb) / sp;
      const double t_item = kbper * (P_A_BYTES + bn * PBK * 2) / 1e5 + 0.5;
      const double t_red = final_mode ? 0.0 : 0.7 * ((sp + 3) / 4);
      const double t = waves * t_item + t_red;
      if (t < best_t - 1e-9) {
        best_t = t;
        best = {bn, sp};
      }
    }
  }
  return best;
}

}  // namespace

struct PersistProgram {
  int dev = -1, dtype = 0, G = 0, nops = 0;
  POp* d_ops = nullptr;
  CUtensorMap* d_maps = nullptr;
  float* d_part = nullptr;
  unsigned* d_bar = nullptr;
  ~PersistProgram() {
    cudaFree(d_ops);
    cudaFree(d_maps);
    cudaFree(d_part);
    cudaFree(d_bar);
  }
};

bool persist_supported(const dp_model* m, const int8_t* method, int T) {
  const auto& c = m->cfg;
  if (T <= 16 || c.layers <= 0) return false;
  if (c.hidden % 128 || c.ffn % 128 || c.hidden > 1024 || c.hidden / c.heads != ATT_D) return false;
  for (const auto& u : m->units) {
    if (u.layer < 0) continue;  // embeddings / pooler run outside the program
    if (method[&u - m->units.data()] != DP_LOAD) return false;  // every layer unit resident
  }
  return true;
}

std::shared_ptr<PersistProgram> build_persist_program(dp_model* m, int dev, int batch, int seq) {
  const auto& c = m->cfg;
  const int T = batch * seq, H = c.hidden, F = c.ffn, L = c.layers;
  const bool gpt2 = c.family == DP_FAMILY_GPT2;
  ensure_workspace(m, dev, T);
  Workspace& ws = m->dev[dev].ws;
  auto prog = std::make_shared<PersistProgram>();
  prog->dev = dev;
  prog->dtype = c.dtype;
  int nsm = 0;
  DP_CUDA(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev));
  prog->G = nsm;
  const int G = nsm;

  std::vector<POp> ops;
  std::vector<CUtensorMap> maps;
  size_t part_floats = 0;
  auto W = [&](int u) -> const void* { return m->device(dev, u); };
  auto second = [&](int u) -> const void* {
    return static_cast<const uint8_t*>(W(u)) + m->params[m->units[u].first_param].bytes;
  };
  // PARTIAL ops' output maps point into the partial buffer, allocated once its size is known
  struct PartFix {
    int map, splits, ntot, bn;
  };
  std::vector<PartFix> part_fix;
  auto gemm = [&](const void* x, int ldx, std::vector<int> wu, int N, int K, bool final_mode,
                  std::vector<const void*> bias, int act, void* out, int ldo) {
    const int ntot = N * (int)wu.size();
    const PCfg cfg = pick_persist_cfg(T, ntot, K, G, final_mode);
    POp op;
    std::memset(&op, 0, sizeof(op));
    op.type = POP_GEMM;
    op.wmap = (int)maps.size();
    for (int u : wu) maps.push_back(make_kmajor_map(W(u), c.dtype, N, K, K, PBM));
    op.xmap = (int)maps.size();
    maps.push_back(make_kmajor_map(x, c.dtype, T, K, ldx, cfg.bn));
    op.groups = (int)wu.size();
    op.M = T, op.N = N, op.K = K, op.splits = cfg.splits, op.bn = cfg.bn;
    op.mtiles = (T + cfg.bn - 1) / cfg.bn;
    op.ntiles = N / PBM;
    op.items = op.groups * op.ntiles * op.mtiles * op.splits;
    op.mode = final_mode ? PG_FINAL : PG_PARTIAL;
    op.omap = (int)maps.size();
    if (final_mode) {
      // out [T rows][ldo] (storage dtype): columns g*N + n
      const uint64_t dims[2] = {(uint64_t)ntot, (uint64_t)T};
      const uint64_t str[1] = {(uint64_t)ldo * 2};
      const uint32_t box[2] = {(uint32_t)PBM, (uint32_t)cfg.bn};
      maps.push_back(make_plain_map(out, c.dtype == DP_BF16 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16
                                                             : CU_TENSOR_MAP_DATA_TYPE_FLOAT16,
                                    2, dims, str, box));
      op.act = act;
      op.bias_w = N;
      op.bias0 = bias.size() > 0 ? bias[0] : nullptr;
      op.bias1 = bias.size() > 1 ? bias[1] : nullptr;
      op.bias2 = bias.size() > 2 ? bias[2] : nullptr;
    } else {
      maps.emplace_back();
      part_fix.push_back({op.omap, cfg.splits, ntot, cfg.bn});
      part_floats = std::max(part_floats, size_t(op.splits) * T * ntot);
    }
    if (getenv("DP_PERSIST_VERBOSE"))
      fprintf(stderr, "[persist] op %zu GEMM %s M=%d N=%dx%d K=%d bn=%d splits=%d items=%d\n", ops.size(),
              final_mode ? "final" : "partial", T, N, op.groups, K, op.bn, op.splits, op.items);
    ops.push_back(op);
    return op.splits;
  };
  auto reduce = [&](int splits, int cols, std::vector<const void*> bias, int act, const void* res, int res_f32,
                    int ln_unit, void* zout, int zout_f32, void* out, bool out_final) {
    POp op;
    std::memset(&op, 0, sizeof(op));
    op.type = POP_REDUCE;
    op.rows = T, op.cols = cols, op.rsplits = splits, op.act = act;
    op.bias_w = bias.empty() ? cols : cols / (int)bias.size();
    op.bias0 = bias.size() > 0 ? bias[0] : nullptr;
    op.bias1 = bias.size() > 1 ? bias[1] : nullptr;
    op.bias2 = bias.size() > 2 ? bias[2] : nullptr;
    op.res = res, op.res_f32 = res_f32;
    if (ln_unit >= 0) op.gamma = W(ln_unit), op.beta = second(ln_unit), op.eps = (float)c.ln_eps;
    op.zout = zout, op.zout_f32 = zout_f32;
    op.out = out, op.out_final = out_final ? 1 : 0;
    ops.push_back(op);
    return (int)ops.size() - 1;
  };
  auto attn = [&](bool causal) {
    POp op;
    std::memset(&op, 0, sizeof(op));
    op.type = POP_ATTN;
    op.qkv = ws.qkv, op.ctx = ws.ctx, op.batch = batch, op.seq = seq, op.H = H, op.heads = c.heads;
    op.causal = causal ? 1 : 0;
    op.scale_log2 = 1.4426950408889634f / sqrtf((float)ATT_D);
    ops.push_back(op);
  };

  if (!gpt2) {
    int u = 4;  // word, pos, type, emb_ln precede layer 0
    for (int l = 0; l < L; ++l) {
      const int q = u++, k = u++, v = u++, ao = u++, ln1 = u++, fc1 = u++, fc2 = u++, ln2 = u++;
      gemm(ws.x, H, {q, k, v}, H, H, true, {second(q), second(k), second(v)}, ACT_NONE, ws.qkv, 3 * H);
      attn(false);
      int sp = gemm(ws.ctx, H, {ao}, H, H, false, {}, 0, nullptr, 0);
      // fp32 residual stream (xr / x1r), as in the per-kernel path (R21)
      ops[reduce(sp, H, {second(ao)}, ACT_NONE, ws.xr, 1, ln1, nullptr, 0, ws.x1, false)].out32 =
          static_cast<float*>(ws.x1r);
      gemm(ws.x1, H, {fc1}, F, H, true, {second(fc1)}, ACT_GELU_ERF, ws.h, F);
      sp = gemm(ws.h, F, {fc2}, H, F, false, {}, 0, nullptr, 0);
      ops[reduce(sp, H, {second(fc2)}, ACT_NONE, ws.x1r, 1, ln2, nullptr, 0, ws.x, l == L - 1)].out32 =
          l == L - 1 ? nullptr : static_cast<float*>(ws.xr);
    }
  } else {
    const int first_ln = 2;  // wte, wpe, then ln_1 of block 0
    // x (fp32 residual stream, written by the embedding kernel) -> x1 = ln_1(x)
    {
      const int i = reduce(0, H, {}, ACT_NONE, nullptr, 0, first_ln, nullptr, 0, ws.x1, false);
      ops[i].in = ws.x, ops[i].in_f32 = 1;
    }
    for (int l = 0; l < L; ++l) {
      int u = first_ln + 6 * l + 1;
      const int at = u++, pr = u++, ln_2 = u++, fc = u++, pr2 = u++, ln_next = u;
      gemm(ws.x1, H, {at}, 3 * H, H, true, {second(at)}, ACT_NONE, ws.qkv, 3 * H);
      attn(true);
      int sp = gemm(ws.ctx, H, {pr}, H, H, false, {}, 0, nullptr, 0);
      reduce(sp, H, {second(pr)}, ACT_NONE, ws.x, 1, ln_2, ws.x, 1, ws.x1, false);
      gemm(ws.x1, H, {fc}, F, H, true, {second(fc)}, ACT_GELU_TANH, ws.h, F);
      sp = gemm(ws.h, F, {pr2}, H, F, false, {}, 0, nullptr, 0);
      reduce(sp, H, {second(pr2)}, ACT_NONE, ws.x, 1, ln_next, ws.x, 1, ws.x1, l == L - 1);
    }
  }
  DP_CUDA(cudaSetDevice(dev));
  DP_CUDA(cudaMalloc(&prog->d_part, std::max<size_t>(part_floats, 4) * sizeof(float)));
  for (const auto& f : part_fix) {  // [splits][T][ntot] fp32, box {128, bn, 1}
    const uint64_t dims[3] = {(uint64_t)f.ntot, (uint64_t)T, (uint64_t)f.splits};
    const uint64_t str[2] = {(uint64_t)f.ntot * 4, (uint64_t)T * f.ntot * 4};
    const uint32_t box[3] = {(uint32_t)PBM, (uint32_t)f.bn, 1u};
    maps[f.map] = make_plain_map(prog->d_part, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 3, dims, str, box);
  }
  for (auto& op : ops) {
    if (op.type == POP_GEMM) op.part = prog->d_part;
    if (op.type == POP_REDUCE && op.rsplits > 0) op.rpart = prog->d_part;
  }
  prog->nops = (int)ops.size();
  DP_CUDA(cudaMalloc(&prog->d_ops, ops.size() * sizeof(POp)));
  DP_CUDA(cudaMemcpy(prog->d_ops, ops.data(), ops.size() * sizeof(POp), cudaMemcpyHostToDevice));
  DP_CUDA(cudaMalloc(&prog->d_maps, std::max<size_t>(maps.size(), 1) * sizeof(CUtensorMap)));
  DP_CUDA(cudaMemcpy(prog->d_maps, maps.data(), maps.size() * sizeof(CUtensorMap), cudaMemcpyHostToDevice));
  DP_CUDA(cudaMalloc(&prog->d_bar, 256));
  return prog;
}

int persist_num_ops(const PersistProgram& p) { return p.nops; }

void launch_persist(const PersistProgram& p, void* final_out, cudaStream_t s) {
  const size_t smem = persist_smem_bytes();
  static std::atomic<unsigned> attr[2];
  const bool bf = p.dtype == DP_BF16;
  auto kern = bf ? persist_kernel<__nv_bfloat16> : persist_kernel<__half>;
  if (first_on_device(attr[bf]))
    DP_CUDA(cudaFuncSetAttribute(reinterpret_cast<const void*>(kern), cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 (int)smem));
  DP_CUDA(cudaMemsetAsync(p.d_bar, 0, sizeof(unsigned), s));
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(p.G);
  cfg.blockDim = dim3(P_THREADS);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeCooperative;  // all CTAs co-resident (the grid barrier needs it)
  at[0].val.cooperative = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  const POp* ops = p.d_ops;
  const CUtensorMap* maps = p.d_maps;
  static const int flags = getenv("DP_PERSIST_FLAGS") ? atoi(getenv("DP_PERSIST_FLAGS")) : 0;
  DP_CUDA(cudaLaunchKernelEx(&cfg, kern, ops, p.nops, maps, p.d_bar, final_out, flags));
}

}  // namespace dp

#ifdef DP_PERSIST_TRACE
extern "C" __attribute__((visibility("default"))) int dp_debug_persist_trace(void* host, int nblocks, int nops) {
  if (nblocks > 160) nblocks = 160;
  std::vector<unsigned long long> all(size_t(160) * dp::P_TR_OPS * 8);
  int r = (int)cudaMemcpyFromSymbol(all.data(), dp::g_persist_trace, all.size() * 8);
  unsigned long long* h = static_cast<unsigned long long*>(host);
  for (int b = 0; b < nblocks; ++b)
    for (int o = 0; o < nops && o < dp::P_TR_OPS; ++o)
      for (int i = 0; i < 8; ++i) h[(size_t(b) * nops + o) * 8 + i] = all[(size_t(b) * dp::P_TR_OPS + o) * 8 + i];
  return r;
}
#endif
