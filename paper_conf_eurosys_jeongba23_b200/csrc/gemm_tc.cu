// K2: resident-weight GEMM on the 5th-generation tensor cores (tcgen05 + TMEM + TMA).
//
//   Y[M, N] = act(X[M, K] . W[N, K]^T + bias[N]) (+ R[M, N])
//
// Used only for layers whose weights are already in HBM: loaded layers
// are true dense contractions.  Shapes on the hot path are skinny in M (tokens: 32..1024)
// and wide in N (768..4096), so the kernel is "swap-AB": the MMA's M axis (128 lanes of
// TMEM) runs over W's rows (N) and the MMA's N axis over tokens (BN = 32..256 columns).
//
// Per CTA (128 threads, one 128 x BN output tile, a K range):
//   warp 0 / lane 0  : TMA producer -- W tile [128 x 64] and X tile [BN x 64] per stage,
//                      both K-major with the 128-byte swizzle, into a STAGES-deep ring; the
//                      first ring of W tiles is issued BEFORE the grid-dependency wait (PDL):
//                      weights never depend on the previous kernel;
//   warp 1 / lane 0  : MMA issuer  -- 4 x tcgen05.mma (K = 16 each) per stage, fp32
//                      accumulator in TMEM; tcgen05.commit releases the smem stage;
//   warp 1           : TMEM allocate / free (BN columns);
//   all 4 warps      : epilogue -- tcgen05.ld 32 lanes x 16 columns into a shared-memory
//                      fp32 tile, then + bias, activation, + residual and 16-byte stores.
// blockIdx.z selects one of up to 3 weight matrices sharing X (BERT q/k/v in one launch).
// Explored and measured slower on B200 (profiles/r01_gemm_sweep_v1.txt): split-K over a
// thread-block cluster with a DSMEM reduction (cluster-barrier waits dominated).
// Descriptor encodings follow the sm_100 UMMA descriptor layout (start>>4, LBO, SBO = 1024 B
// for 8-row swizzle atoms, version 1, layout SWIZZLE_128B = 2).
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <cstring>
#include <cstdlib>
#include <algorithm>
#include <mutex>

#include "common.h"
#include "dtype.cuh"
#include "kernels.h"
#include "launch.cuh"

namespace dp {

namespace {

constexpr int BM = 128;  // W rows per tile (MMA M)
constexpr int BK = 64;   // K per stage: 64 x 2 B = one 128-byte swizzle row

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}

__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
               : "memory");
}

__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t phase) {
  const uint32_t a = smem_u32(bar);
  asm volatile(
      "{\n"
      ".reg .pred P1;\n"
      "WAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
      "@!P1 bra WAIT_%=;\n"
      "}\n" ::"r"(a),
      "r"(phase)
      : "memory");
}

__device__ __forceinline__ void tma_load_2d(const CUtensorMap* map, uint64_t* bar, void* dst, int c0, int c1) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];" ::"r"(
          smem_u32(dst)),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(c0), "r"(c1), "r"(smem_u32(bar))
      : "memory");
}

__device__ __forceinline__ uint64_t sw128_desc(const void* smem_tile) {
  const uint64_t addr = smem_u32(smem_tile);
  uint64_t d = 0;
  d |= (addr & 0x3FFFFull) >> 4;  // start address
  d |= uint64_t(1) << 16;          // LBO (unused for swizzled K-major)
  d |= uint64_t(1024 >> 4) << 32;  // SBO: 8 rows x 128 B
  d |= uint64_t(1) << 46;          // descriptor version (sm_100)
  d |= uint64_t(2) << 61;          // SWIZZLE_128B
  return d;
}

__device__ __forceinline__ void umma_f16(uint32_t tmem_d, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "setp.ne.b32 p, %4, 0;\n"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n"
      "}\n" ::"r"(tmem_d),
      "l"(a), "l"(b), "r"(idesc), "r"(acc));
}

__device__ __forceinline__ void umma_commit(uint64_t* bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(bar))
               : "memory");
}

__device__ __forceinline__ void tmem_ld16(uint32_t taddr, uint32_t* v) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
      : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
        "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15])
      : "r"(taddr));
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}




template <class T>
struct FmtBits;
template <>
struct FmtBits<__half> {
  static constexpr uint32_t v = 0;
};
template <>
struct FmtBits<__nv_bfloat16> {
  static constexpr uint32_t v = 1;
};

// Ring depth per tile width: as many stages as ~224 KB of shared memory holds (<= 12), so a
// K = 768 layer (12 k-blocks) has its whole weight slice in flight at once.
template <int BN>
__host__ __device__ constexpr int stages_for() {
  constexpr int bytes = BM * BK * 2 + BN * BK * 2;
  constexpr int s = (224 * 1024) / bytes;
  return s > 12 ? 12 : s;
}

// Up to 3 independent weight matrices sharing X, M, N, K (BERT's q/k/v): blockIdx.z selects
// the weight, its bias and the output column offset, so the three projections are one launch.
struct GemmGroup {
  CUtensorMap w[3];
  const void* bias[3];
  long long ycol[3];
};

#ifdef DP_GEMM_TRACE
// phase timestamps (globaltimer, ns) per CTA: entry, setup done, after grid-dependency wait,
// first stage landed (MMA issuer), all MMAs done, partial/tile in smem, end; [7] = SM id
__device__ unsigned long long g_gemm_trace[4096][8];
__device__ __forceinline__ unsigned long long gtime() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
#define TRACE(i)                                                                                  \
  do {                                                                                            \
    const int b_ = (blockIdx.z * gridDim.y + blockIdx.y) * gridDim.x + blockIdx.x;                \
    if (b_ < 4096) g_gemm_trace[b_][i] = gtime();                                                 \
  } while (0)
#else
#define TRACE(i) \
  do {           \
  } while (0)
#endif

// Split-K: blockIdx.z = group * splits + split; each split accumulates its K range in TMEM,
// writes the fp32 tile to a workspace slot and bumps the tile's counter; the LAST split to
// arrive sums the slots in split order 0..splits-1 (deterministic whichever CTA is last),
// resets the counter and runs the epilogue.  Spreads a weight tile's bytes over `splits`
// SMs: at the hot path's 128-token shapes a CTA's time is set by the bytes it ingests.
template <class T, int BN>
__global__ void __launch_bounds__(128, 1)
    gemm_tc_kernel(const __grid_constant__ GemmGroup grp, const __grid_constant__ CUtensorMap tmX,
                   const void* res, int ldr, void* Y, int ldy, int M, int N, int K, int act, int io, int splits,
                   float* __restrict__ ws, int* __restrict__ cnt) {
  constexpr int STAGES = stages_for<BN>();
  constexpr uint32_t A_BYTES = BM * BK * 2;  // 16 KB
  constexpr uint32_t B_BYTES = BN * BK * 2;
  constexpr uint32_t STAGE_BYTES = A_BYTES + B_BYTES;
  constexpr uint32_t TMEM_COLS = BN < 32 ? 32 : BN;
  constexpr int PROW = BN + 1;  // fp32 tile row stride (odd: conflict-free TMEM->smem writes)
  // kind::f16, fp32 accumulate, A/B K-major, M = 128, N = BN
  constexpr uint32_t IDESC = (1u << 4) | (FmtBits<T>::v << 7) | (FmtBits<T>::v << 10) | (uint32_t(BN >> 3) << 17) |
                             (uint32_t(BM >> 4) << 24);

  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  __shared__ __align__(8) uint64_t full_bar[STAGES], empty_bar[STAGES], done_bar;
  __shared__ uint32_t tmem_base_sh;

  TRACE(0);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int n0 = blockIdx.x * BM, m0 = blockIdx.y * BN;
  const int grp_i = blockIdx.z / splits, sp = blockIdx.z - grp_i * splits;
  const CUtensorMap* tmW = &grp.w[grp_i];
  const T* bias = static_cast<const T*>(grp.bias[grp_i]);
  const long long ycol = grp.ycol[grp_i];
  const int kb_all = K / BK;
  const int kb_lo = sp * kb_all / splits;
  const int num_kb = (sp + 1) * kb_all / splits - kb_lo;  // >= 1 (splits <= kb_all)

  if (warp == 0 && lane == 0) {
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(tmW)) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&tmX)) : "memory");
    for (int s = 0; s < STAGES; ++s) {
      mbar_init(&full_bar[s], 1);
      mbar_init(&empty_bar[s], 1);
    }
    mbar_init(&done_bar, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&tmem_base_sh)),
                 "r"(TMEM_COLS));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tmem_d = tmem_base_sh;
  pdl_trigger();

  // Weights never depend on the previous kernel: the producer puts the first ring's worth
  // of W tiles in flight BEFORE the grid-dependency wait (PDL), so their HBM latency
  // overlaps the predecessor's tail.  Activations (X, residual) and every store come after.
  const int pre = num_kb < STAGES ? num_kb : STAGES;
  if (warp == 0 && lane == 0) {
    for (int kb = 0; kb < pre; ++kb) {
      mbar_expect_tx(&full_bar[kb], STAGE_BYTES);
      tma_load_2d(tmW, &full_bar[kb], smem + kb * STAGE_BYTES, (kb_lo + kb) * BK, n0);
    }
  }
  TRACE(1);
  pdl_wait();
  TRACE(2);

  if (warp == 0 && lane == 0) {
    // TMA producer
    for (int kb = 0; kb < num_kb; ++kb) {
      const int s = kb % STAGES;
      uint8_t* a = smem + s * STAGE_BYTES;
      uint8_t* b = a + A_BYTES;
      if (kb >= pre) {
        mbar_wait(&empty_bar[s], ((kb / STAGES) - 1) & 1);
        mbar_expect_tx(&full_bar[s], STAGE_BYTES);
        tma_load_2d(tmW, &full_bar[s], a, (kb_lo + kb) * BK, n0);
      }
      tma_load_2d(&tmX, &full_bar[s], b, (kb_lo + kb) * BK, m0);
    }
  } else if (warp == 1 && lane == 0) {
    // MMA issuer
    for (int kb = 0; kb < num_kb; ++kb) {
      const int s = kb % STAGES;
      mbar_wait(&full_bar[s], (kb / STAGES) & 1);
      if (kb == 0) TRACE(3);
      asm volatile("tcgen05.fence::after_thread_sync;");
      const uint8_t* a = smem + s * STAGE_BYTES;
      const uint8_t* b = a + A_BYTES;
      const uint64_t da = sw128_desc(a), db = sw128_desc(b);
#pragma unroll
      for (int kk = 0; kk < BK / 16; ++kk)  // advance 16 elements = 32 B = 2 in descriptor units
        umma_f16(tmem_d, da + 2 * kk, db + 2 * kk, IDESC, (kb | kk) != 0);
      umma_commit(&empty_bar[s]);
    }
    umma_commit(&done_bar);
  }
  __syncwarp();

  mbar_wait(&done_bar, 0);
  if (threadIdx.x == 0) TRACE(4);
  asm volatile("tcgen05.fence::after_thread_sync;");
  // 1) TMEM -> shared memory (the ring is free once the MMAs are done): the fp32 tile,
  //    [128 W rows][BN tokens] with an odd row stride
  const int row = warp * 32 + lane;  // TMEM lane = W row within the tile
  float* tile = reinterpret_cast<float*>(smem);
#pragma unroll 1
  for (int c0 = 0; c0 < BN; c0 += 16) {
    uint32_t v[16];
    tmem_ld16(tmem_d + (uint32_t(warp * 32) << 16) + c0, v);
#pragma unroll
    for (int j = 0; j < 16; ++j) tile[row * PROW + c0 + j] = __uint_as_float(v[j]);
  }
  __syncthreads();
  if (splits > 1) {
    // 1b) split-K fixup (see above): publish this split's tile, count arrivals
    __shared__ int last_sh;
    const int tile_id = (grp_i * gridDim.y + blockIdx.y) * gridDim.x + blockIdx.x;
    float* slots = ws + (size_t)tile_id * splits * (BM * BN);
    float* mine = slots + (size_t)sp * (BM * BN);
    for (int i = threadIdx.x; i < BM * BN / 4; i += 128) {
      const int r = (4 * i) / BN, c = (4 * i) % BN;
      reinterpret_cast<float4*>(mine)[i] =
          make_float4(tile[r * PROW + c], tile[r * PROW + c + 1], tile[r * PROW + c + 2], tile[r * PROW + c + 3]);
    }
    __threadfence();
    __syncthreads();
    if (threadIdx.x == 0) last_sh = atomicAdd(&cnt[tile_id], 1) == splits - 1;
    __syncthreads();
    if (!last_sh) {
      if (threadIdx.x == 0) {
        TRACE(5);
        TRACE(6);
      }
      asm volatile("tcgen05.fence::before_thread_sync;");
      __syncthreads();
      if (warp == 1) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem_d), "r"(TMEM_COLS));
      return;
    }
    __threadfence();
    for (int i = threadIdx.x; i < BM * BN / 4; i += 128) {
      float4 a = __ldcg(reinterpret_cast<const float4*>(slots) + i);
      for (int p = 1; p < splits; ++p) {
        const float4 b = __ldcg(reinterpret_cast<const float4*>(slots + (size_t)p * (BM * BN)) + i);
        a.x += b.x, a.y += b.y, a.z += b.z, a.w += b.w;
      }
      const int r = (4 * i) / BN, c = (4 * i) % BN;
      tile[r * PROW + c] = a.x, tile[r * PROW + c + 1] = a.y, tile[r * PROW + c + 2] = a.z, tile[r * PROW + c + 3] = a.w;
    }
    if (threadIdx.x == 0) cnt[tile_id] = 0;  // ready for the next launch
    __syncthreads();
  }
  if (threadIdx.x == 0) TRACE(5);
  // 2) out[m][n0 .. n0+127] for every token m: thread t owns 8 consecutive W rows
  //    (n = n0 + 8*(t%16) ..+7) of token m = t/16 + 8*pass -> one 16-byte store (and one
  //    16-byte residual load) per 8 outputs
  {
    const int t = threadIdx.x;
    const int nl = 8 * (t & 15);
    const int n = n0 + nl;
    const bool nok = n < N;  // N % 128 == 0, so all 8 rows are valid together
    float bv[8];
#pragma unroll
    for (int e = 0; e < 8; ++e) bv[e] = (bias != nullptr && nok) ? Cvt<T>::to1(bias[n + e]) : 0.f;
    const int mcount = min(BN, M - m0);
    const bool res32 = io & IO_RES_F32, out32 = io & IO_OUT_F32;
#pragma unroll 1
    for (int ml = t >> 4; ml < mcount && nok; ml += 8) {
      float acc[8];
#pragma unroll
      for (int e = 0; e < 8; ++e) acc[e] = apply_act(tile[(nl + e) * PROW + ml] + bv[e], act);
      const size_t m = (size_t)(m0 + ml);
      if (res) {
        float r8[8];
        load8<T>(res, m * ldr + n, r8, res32);
#pragma unroll
        for (int e = 0; e < 8; ++e) acc[e] += r8[e];
      }
      store8<T>(Y, m * ldy + n + ycol, acc, out32);
    }
  }
#ifdef DP_GEMM_TRACE
  if (threadIdx.x == 0) {
    TRACE(6);
    unsigned smid;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
    const int b_ = (blockIdx.z * gridDim.y + blockIdx.y) * gridDim.x + blockIdx.x;
    if (b_ < 4096) g_gemm_trace[b_][7] = smid;
  }
#endif
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (warp == 1) {
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem_d), "r"(TMEM_COLS));
  }
}

PFN_cuTensorMapEncodeTiled_v12000 get_encode() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
  });
  DP_CHECK(fn != nullptr, DP_ERR_CUDA, "cuTensorMapEncodeTiled unavailable");
  return fn;
}

// 2D K-major tile map: rows x K elements with row stride ld (elements), box {64, box_rows}.
CUtensorMap make_map(const void* base, int dtype, int rows, int K, int ld, int box_rows) {
  CUtensorMap m;
  std::memset(&m, 0, sizeof(m));
  cuuint64_t dims[2] = {(cuuint64_t)K, (cuuint64_t)rows};
  cuuint64_t strides[1] = {(cuuint64_t)ld * 2};
  cuuint32_t box[2] = {(cuuint32_t)BK, (cuuint32_t)box_rows};
  cuuint32_t estr[2] = {1, 1};
  CUresult r = get_encode()(&m, dtype == DP_BF16 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT16,
                            2, const_cast<void*>(base), dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                            CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                            CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  DP_CHECK(r == CUDA_SUCCESS, DP_ERR_CUDA, "cuTensorMapEncodeTiled failed (" + std::to_string((int)r) + ")");
  return m;
}

// Split-K workspace, one per device: fp32 tile slots + per-tile arrival counters (zeroed
// once; the last split of every tile resets its counter).  Kernels on one device use it in
// stream order (the engine runs a forward's kernels on one stream; PDL successors touch it
// only after griddepcontrol.wait, i.e. after the previous GEMM completed).
constexpr size_t SPLIT_WS_BYTES = size_t(32) << 20;
constexpr int SPLIT_MAX_TILES = 16384;
struct SplitWs {
  float* ws = nullptr;
  int* cnt = nullptr;
};
SplitWs& split_ws(int dev) {
  static SplitWs w[64];
  return w[dev];
}
std::mutex split_mu;

SplitWs& split_ws_ready(cudaStream_t s) {
  int dev;
  DP_CUDA(cudaGetDevice(&dev));
  SplitWs& w = split_ws(dev);
  if (w.ws) return w;
  cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
  DP_CUDA(cudaStreamIsCapturing(s, &cs));
  DP_CHECK(cs == cudaStreamCaptureStatusNone, DP_ERR_STATE, "split-K workspace must be prepared before capture");
  gemm_prepare(dev);
  return w;
}

template <class T, int BN>
void run(const void* x, int ldx, int ngroups, const void* const* w, const void* const* bias, const long long* ycol,
         const void* res, int ldr, void* y, int ldy, int M, int N, int K, int act, int io, int splits,
         cudaStream_t s) {
  constexpr size_t smem = size_t(stages_for<BN>()) * (BM * BK * 2 + BN * BK * 2) + 1024;
  static_assert(size_t(BM) * (BN + 1) * 4 + 1024 <= smem, "fp32 tile must fit the ring");
  static bool attr = false;
  if (!attr) {
    DP_CUDA(cudaFuncSetAttribute(gemm_tc_kernel<T, BN>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    attr = true;
  }
  const int dtype = std::is_same<T, __half>::value ? DP_FP16 : DP_BF16;
  GemmGroup g;
  std::memset(&g, 0, sizeof(g));
  for (int i = 0; i < ngroups; ++i) {
    g.w[i] = make_map(w[i], dtype, N, K, K, BM);
    g.bias[i] = bias ? bias[i] : nullptr;
    g.ycol[i] = ycol ? ycol[i] : 0;
  }
  CUtensorMap mx = make_map(x, dtype, M, K, ldx, BN);
  const int mt = (M + BN - 1) / BN;
  float* ws = nullptr;
  int* cnt = nullptr;
  if (splits > 1) {
    const size_t tiles = size_t(N / BM) * mt * ngroups;
    if (tiles * splits * BM * BN * 4 > SPLIT_WS_BYTES || tiles > (size_t)SPLIT_MAX_TILES) splits = 1;
  }
  if (splits > 1) {
    SplitWs& sw = split_ws_ready(s);
    ws = sw.ws;
    cnt = sw.cnt;
  }
  launch_kernel(gemm_tc_kernel<T, BN>, dim3(N / BM, mt, ngroups * splits), dim3(128), smem, s, g, mx, res, ldr, y,
                ldy, M, N, K, act, io, splits, ws, cnt);
}

template <class T>
void dispatch(int bn, const void* x, int ldx, int ngroups, const void* const* w, const void* const* bias,
              const long long* ycol, const void* res, int ldr, void* y, int ldy, int M, int N, int K, int act, int io,
              int sp, cudaStream_t s) {
  switch (bn) {
    case 32: run<T, 32>(x, ldx, ngroups, w, bias, ycol, res, ldr, y, ldy, M, N, K, act, io, sp, s); break;
    case 64: run<T, 64>(x, ldx, ngroups, w, bias, ycol, res, ldr, y, ldy, M, N, K, act, io, sp, s); break;
    case 128: run<T, 128>(x, ldx, ngroups, w, bias, ycol, res, ldr, y, ldy, M, N, K, act, io, sp, s); break;
    case 256: run<T, 256>(x, ldx, ngroups, w, bias, ycol, res, ldr, y, ldy, M, N, K, act, io, sp, s); break;
    default: fail(DP_ERR_INVALID, "gemm: BN must be 32/64/128/256");
  }
}

}  // namespace

void gemm_prepare(int dev) {
  std::lock_guard<std::mutex> lk(split_mu);
  SplitWs& w = split_ws(dev);
  if (w.ws) return;
  int cur;
  DP_CUDA(cudaGetDevice(&cur));
  DP_CUDA(cudaSetDevice(dev));
  void *a = nullptr, *b = nullptr;
  if (cudaMalloc(&a, SPLIT_WS_BYTES) != cudaSuccess || cudaMalloc(&b, SPLIT_MAX_TILES * sizeof(int)) != cudaSuccess)
    fail(DP_ERR_OOM, "split-K workspace cudaMalloc failed");
  DP_CUDA(cudaMemset(b, 0, SPLIT_MAX_TILES * sizeof(int)));
  DP_CUDA(cudaDeviceSynchronize());
  w.ws = static_cast<float*>(a);
  w.cnt = static_cast<int*>(b);
  DP_CUDA(cudaSetDevice(cur));
}

bool gemm_tc_supported(int N, int K) { return N > 0 && K > 0 && N % BM == 0 && K % BK == 0; }

// Tile width over tokens: the widest BN that still gives >= 96 CTAs (~2/3 of the SMs), else
// 32.  Chosen from the B200 sweep in profiles/r01_gemm_sweep_v2.txt: it picks the fastest
// measured BN at every hot-path shape (M = 128 / 384 / 1024; N, K in 768..4096).
static int pick_bn(int M, int N) {
  const int ntile = N / BM;
  for (int bn : {256, 128, 64}) {
    if (M >= bn && ntile * ((M + bn - 1) / bn) >= 96) return bn;
  }
  return 32;
}

// Split-K factor: enough K splits to put ~one CTA on every SM, each with >= 2 k-blocks.
static int pick_split(int M, int N, int K, int bn) {
  const int tiles = (N / BM) * ((M + bn - 1) / bn);
  int sp = 148 / std::max(1, tiles);
  sp = std::min(sp, (K / BK) / 2);
  return std::max(1, sp);
}

void launch_gemm_tc_group(int dtype, const void* x, int ldx, int ngroups, const void* const* w,
                          const void* const* bias, const long long* ycol, const void* res, int ldr, void* y, int ldy,
                          int M, int N, int K, int act, int io, int bn_hint, cudaStream_t s) {
  DP_CHECK(gemm_tc_supported(N, K), DP_ERR_UNSUPPORTED, "tcgen05 GEMM needs N % 128 == 0 and K % 64 == 0");
  DP_CHECK(ngroups >= 1 && ngroups <= 3, DP_ERR_INVALID, "gemm: 1..3 weight groups");
  DP_CHECK(ldx % 8 == 0 && ((uintptr_t)x % 16) == 0, DP_ERR_INVALID, "GEMM activations must be 16-byte aligned");
  for (int i = 0; i < ngroups; ++i)
    DP_CHECK(((uintptr_t)w[i] % 16) == 0 && (!ycol || ycol[i] % 8 == 0), DP_ERR_INVALID,
             "GEMM weights / output columns must be 16-byte aligned");
  DP_CHECK(ldy % 8 == 0 && (!res || ldr % 8 == 0), DP_ERR_INVALID, "GEMM output rows must be 16-byte aligned");
  if (M <= 0) return;
  // tuning override for experiments (DP_GEMM_BN), read once
  static const int env_bn = getenv("DP_GEMM_BN") ? atoi(getenv("DP_GEMM_BN")) : 0;
  const int bn = bn_hint > 0 ? bn_hint : (env_bn > 0 ? env_bn : pick_bn(M, N * ngroups));
  static const int env_sp = getenv("DP_GEMM_SPLIT") ? atoi(getenv("DP_GEMM_SPLIT")) : 0;
  int sp = env_sp > 0 ? env_sp : pick_split(M, N * ngroups, K, bn);
  sp = std::max(1, std::min(sp, K / BK));
  if (dtype == DP_BF16)
    dispatch<__nv_bfloat16>(bn, x, ldx, ngroups, w, bias, ycol, res, ldr, y, ldy, M, N, K, act, io, sp, s);
  else
    dispatch<__half>(bn, x, ldx, ngroups, w, bias, ycol, res, ldr, y, ldy, M, N, K, act, io, sp, s);
}

void launch_gemm_tc(int dtype, const void* x, int ldx, const void* w, const void* bias, const void* res, int ldr,
                    void* y, int ldy, int M, int N, int K, int act, int io, int bn_hint, cudaStream_t s) {
  launch_gemm_tc_group(dtype, x, ldx, 1, &w, &bias, nullptr, res, ldr, y, ldy, M, N, K, act, io, bn_hint, s);
}

}  // namespace dp

#ifdef DP_GEMM_TRACE
extern "C" __attribute__((visibility("default"))) int dp_debug_gemm_trace(void* host, int nblocks) {
  if (nblocks > 4096) nblocks = 4096;
  return (int)cudaMemcpyFromSymbol(host, dp::g_gemm_trace, size_t(nblocks) * 8 * sizeof(unsigned long long));
}
#endif
