// K2: resident-weight GEMM on the 5th-generation tensor cores (tcgen05 + TMEM + TMA).
//
//   Y[M, N] = act(X[M, K] . W[N, K]^T + bias[N]) (+ R[M, N])
//
// Used only for layers whose weights are already in HBM: loaded layers
// are true dense contractions.  Shapes on the hot path are skinny in M (tokens: 32..1024)
// and wide in N (768..4096), so the kernel is "swap-AB": the MMA's M axis (128 lanes of
// TMEM) runs over W's rows (N) and the MMA's N axis over tokens (BN = 32..256 columns).
//
// Per CTA (256 threads, one 128 x BN output tile, a K range):
//   warp 0 / lane 0  : TMA producer -- W tile [128 x 64 KS] and X tile [BN x 64 KS] per stage
//                      (KS = ks_for<BN>() 64-deep chunks, one 3D box each when KS > 1),
//                      both K-major with the 128-byte swizzle, into a STAGES-deep ring; the
//                      first ring of W tiles is issued BEFORE the grid-dependency wait (PDL):
//                      weights never depend on the previous kernel;
//   warp 1 / lane 0  : MMA issuer  -- 4 x tcgen05.mma (K = 16 each) per stage, fp32
//                      accumulator in TMEM; tcgen05.commit releases the smem stage;
//   warp 1           : TMEM allocate / free (BN columns);
//   all 8 warps      : epilogue -- tcgen05.ld 32 lanes x 16 columns (warp w: lane quarter w%4,
//                      column half w/4) into a shared-memory fp32 tile, then + bias,
//                      activation, + residual and 16-byte stores (8 warps: the epilogue is
//                      latency-bound, 39% of a 1024-token tile with 4 warps).
// blockIdx.z selects one of up to 3 weight matrices sharing X (BERT q/k/v in one launch).
// Explored and measured slower on B200 (profiles/r01_gemm_sweep_v1.txt): split-K over a
// thread-block cluster with a DSMEM reduction (cluster-barrier waits dominated).
// Descriptor encodings follow the sm_100 UMMA descriptor layout (start>>4, LBO, SBO = 1024 B
// for 8-row swizzle atoms, version 1, layout SWIZZLE_128B = 2).
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>
#include <cstring>
#include <cstdlib>
#include <algorithm>
#include <mutex>

#include "common.h"
#include "dtype.cuh"
#include "kernels.h"
#include "launch.cuh"
#include "ln.cuh"
#include "tc.cuh"

namespace dp {

static PFN_cuTensorMapEncodeTiled_v12000 get_encode() {
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

CUtensorMap make_kmajor_map(const void* base, int dtype, int rows, int K, int ld, int box_rows) {
  CUtensorMap m;
  std::memset(&m, 0, sizeof(m));
  cuuint64_t dims[2] = {(cuuint64_t)K, (cuuint64_t)rows};
  cuuint64_t strides[1] = {(cuuint64_t)ld * 2};
  cuuint32_t box[2] = {64u, (cuuint32_t)box_rows};  // 64 elements = one 128-byte swizzle row
  cuuint32_t estr[2] = {1, 1};
  CUresult r = get_encode()(&m, dtype == DP_BF16 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT16,
                            2, const_cast<void*>(base), dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                            CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                            CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  DP_CHECK(r == CUDA_SUCCESS, DP_ERR_CUDA, "cuTensorMapEncodeTiled failed (" + std::to_string((int)r) + ")");
  return m;
}

// K-major tile map whose box spans `kch` consecutive 64-element K chunks: dims {64, rows, K/64}
// (the chunk dimension strides 128 B), box {64, box_rows, kch} -> shared memory [kch][box_rows]
// [128 B], i.e. kch swizzled K-major sub-tiles back to back, in ONE TMA operation.
CUtensorMap make_kmajor_map3(const void* base, int dtype, int rows, int K, int ld, int box_rows, int kch) {
  CUtensorMap m;
  std::memset(&m, 0, sizeof(m));
  cuuint64_t dims[3] = {64, (cuuint64_t)rows, (cuuint64_t)(K / 64)};
  cuuint64_t strides[2] = {(cuuint64_t)ld * 2, 128};
  cuuint32_t box[3] = {64u, (cuuint32_t)box_rows, (cuuint32_t)kch};
  cuuint32_t estr[3] = {1, 1, 1};
  CUresult r = get_encode()(&m, dtype == DP_BF16 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT16,
                            3, const_cast<void*>(base), dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                            CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                            CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  DP_CHECK(r == CUDA_SUCCESS, DP_ERR_CUDA, "cuTensorMapEncodeTiled (3d) failed (" + std::to_string((int)r) + ")");
  return m;
}

// Generic tiled map (no swizzle): rank 1..3, dims/strides in elements / bytes (strides of
// dims 1.., as cuTensorMapEncodeTiled takes them).  Used for K6's TMA stores.
CUtensorMap make_plain_map(const void* base, CUtensorMapDataType dt, int rank, const uint64_t* dims,
                           const uint64_t* strides_bytes, const uint32_t* box) {
  CUtensorMap m;
  std::memset(&m, 0, sizeof(m));
  cuuint64_t d[3], st[2];
  cuuint32_t bx[3], es[3] = {1, 1, 1};
  for (int i = 0; i < rank; ++i) d[i] = dims[i], bx[i] = box[i];
  for (int i = 0; i + 1 < rank; ++i) st[i] = strides_bytes[i];
  CUresult r = get_encode()(&m, dt, rank, const_cast<void*>(base), d, st, bx, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                            CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_NONE,
                            CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  DP_CHECK(r == CUDA_SUCCESS, DP_ERR_CUDA, "cuTensorMapEncodeTiled (plain) failed (" + std::to_string((int)r) + ")");
  return m;
}

namespace {

constexpr int BM = 128;  // W rows per tile (MMA M)
constexpr int NT = 256;  // threads per CTA: warp 0 TMA, warp 1 MMA + TMEM, all 8 warps the epilogue
constexpr int BK = 64;   // K per 128-byte swizzle row (64 x 2 B)
// 64-deep K chunks per ring stage of the single-CTA kernel: > 1 makes one 3D TMA box per
// operand span them.  The per-CTA traces put the 128-token mainloop at ~0.26 us per TMA
// box pair whatever its bytes (BN 32..128 alike; W in 64- / 32-row boxes was slower), so fewer,
// deeper boxes stream faster.  Measured in the warm forwards (profiles/r02_warm_ab_kchunks.jsonl,
// A/B of 1..4 chunks per tile width): 3 for BN <= 64, 2 for BN 96 / 128, 1 for BN 256 (deeper
// 256-wide stages leave only 2 ring stages).  BERT-Base 0.424 -> 0.365 ms, BERT-Large 1.199 ->
// 1.109, GPT-2 Medium 1.671 -> 1.577.  (Experiment overrides: -DDP_GEMM_KS_{SMALL,MID,BIG}.)
#ifndef DP_GEMM_KS_SMALL
#define DP_GEMM_KS_SMALL 3
#endif
#ifndef DP_GEMM_KS_MID
#define DP_GEMM_KS_MID 2
#endif
#ifndef DP_GEMM_KS_BIG
#define DP_GEMM_KS_BIG 1
#endif
template <int BN>
__host__ __device__ constexpr int ks_for() {
  return BN <= 64 ? DP_GEMM_KS_SMALL : BN <= 128 ? DP_GEMM_KS_MID : DP_GEMM_KS_BIG;
}

__device__ __forceinline__ void tma_load_3d(const CUtensorMap* map, uint64_t* bar, void* dst, int c0, int c1, int c2) {
  asm volatile(
      "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], [%5];" ::"r"(
          smem_u32(dst)),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(c0), "r"(c1), "r"(c2), "r"(smem_u32(bar))
      : "memory");
}
// one stage's tile (rows x KS*64 K) from a KS-chunk map (KS == 1: the 2D map)
template <int KS>
__device__ __forceinline__ void tma_load_stage(const CUtensorMap* map, uint64_t* bar, void* dst, int kblk, int row) {
  if constexpr (KS == 1)
    tma_load_2d(map, bar, dst, kblk * BK, row);
  else
    tma_load_3d(map, bar, dst, 0, row, kblk * KS);
}

// Ring depth per tile width: as many stages as ~224 KB of shared memory holds (<= 12), so a
// K = 768 layer (12 k-blocks) has its whole weight slice in flight at once.
template <int BN>
__host__ __device__ constexpr int stages_for() {
  constexpr int KS = ks_for<BN>();
  constexpr int bytes = KS * (BM * BK * 2 + BN * BK * 2);
  constexpr int s = (224 * 1024) / bytes;
  return s > 12 / KS ? 12 / KS : s;
}

// Up to 3 independent weight matrices sharing X, M, N, K (BERT's q/k/v): blockIdx.z selects
// the weight, its bias and the output column offset, so the three projections are one launch.
struct GemmGroup {
  CUtensorMap w[3];
  const void* bias[3];
  long long ycol[3];
};

#ifdef DP_GEMM_TRACE
// phase timestamps (globaltimer, ns) per CTA: 0 entry, 1 W prefetch issued, 2 setup done,
// 3 after the grid-dependency wait, 4 first stage landed, 5 MMAs done, 6 tile in smem,
// 7 tile reduced (split-K), 8 end; [15] = SM id
__device__ unsigned long long g_gemm_trace[4096][16];
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

__device__ __forceinline__ uint32_t mapa_u32(uint32_t saddr, uint32_t rank) {
  uint32_t r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(saddr), "r"(rank));
  return r;
}
__device__ __forceinline__ float ld_cluster_f32(uint32_t addr) {
  float v;
  asm volatile("ld.shared::cluster.f32 %0, [%1];" : "=f"(v) : "r"(addr) : "memory");
  return v;
}

// The epilogue's kernel parameters, copied to shared memory in the prologue: read from the
// constant bank only after the mainloop, each cold parameter line cost a constant-cache miss on
// the critical path (the compiler rematerialises a register copy from the bank, so the copy has
// to be opaque to it).
struct EpiParams {
  const void* res;
  int ldr, ycol, io, mcount;
};

// Single-split epilogue, shared by K2 and its CTA-pair variant: straight from TMEM to the
// output.  Each thread owns one W row (feature n) and walks the token columns 16 at a time:
// + bias, activation, + residual (a warp's 32 lanes read 32 consecutive features of a token:
// coalesced), and writes the value into an output tile in shared memory laid out like Y
// ([BN tokens][128 features], the output dtype) -- a warp writes 32 consecutive elements per
// token, conflict-free.  One TMA bulk tensor store then writes the tile (rows past M are
// clipped by the tensor map), replacing the fp32 round trip through shared memory and the
// per-thread 16-byte stores of round 1.  `otile` is the ring, free once the MMAs are done.
// IOT: the epilogue's I/O as a compile-time constant where the forward pass fixes it -- 1 = no
// residual, output in the storage type (q/k/v, fc1); 2 = fp32 residual, fp32 output (attn-out,
// fc2, GPT-2's projections into the fp32 residual stream); 0 = any (read from io / res at run
// time: the kernel test hooks).  Each variant carries only its own epilogue code: a CTA runs
// its code once, and cold instruction fetch is on its critical path.
template <int IOT>
struct EpiIO {
  __device__ __forceinline__ static const void* res(const void* r) { return IOT == 1 ? nullptr : r; }
  __device__ __forceinline__ static bool has_res(const void* r) { return IOT == 2 ? true : IOT == 1 ? false : r != nullptr; }
  __device__ __forceinline__ static bool res32(int io) { return IOT == 2 ? true : IOT == 1 ? false : (io & IO_RES_F32); }
  __device__ __forceinline__ static bool out32(int io) { return IOT == 2 ? true : IOT == 1 ? false : (io & IO_OUT_F32); }
};

template <class T, int BN, int ACT, int IOT>
__device__ __forceinline__ void store_tile(uint8_t* otile, uint32_t tmem_d, const float* sbias,
                                           const CUtensorMap* tmY, int n0, int m0, const EpiParams& ep) {
  if (threadIdx.x == 64) TRACE(14);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const void* res = EpiIO<IOT>::res(ep.res);
  const bool has_res = EpiIO<IOT>::has_res(res);
  const int ldr = ep.ldr, ycol = ep.ycol, mcount = ep.mcount;
  const bool res32 = EpiIO<IOT>::res32(ep.io), out32 = EpiIO<IOT>::out32(ep.io);
  // TMEM lane = W row within the tile; warp w reads its lane quarter (w % 4) for the column
  // half w / 4 of the tile
  const int row = (warp & 3) * 32 + lane;
  const int chalf = (warp >> 2) * (BN / 2);
  const int n = n0 + row;
  const float bsv = sbias[row];
#pragma unroll 1
  for (int c0 = chalf; c0 < chalf + BN / 2; c0 += 16) {
    float rv[16];
    if (has_res) {
#pragma unroll
      for (int j = 0; j < 16; ++j) {
        const int ml = c0 + j;
        rv[j] = ml < mcount ? load1<T>(res, (size_t)(m0 + ml) * ldr + n, res32) : 0.f;
      }
    }
    uint32_t v[16];
    if (threadIdx.x == 0 && c0 == 0) TRACE(9);
    tmem_ld16(tmem_d + (uint32_t((warp & 3) * 32) << 16) + c0, v);
    if (threadIdx.x == 0 && c0 == 0) TRACE(10);
#pragma unroll
    for (int j = 0; j < 16; ++j) {
      float a = apply_act_c<ACT>(__uint_as_float(v[j]) + bsv);
      if (has_res) a += rv[j];
      if (out32)
        reinterpret_cast<float*>(otile)[(c0 + j) * BM + row] = a;
      else
        reinterpret_cast<T*>(otile)[(c0 + j) * BM + row] = Cvt<T>::from1(a);
    }
  }
  if (threadIdx.x == 0) TRACE(11);
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // generic writes -> async proxy
  if (threadIdx.x == 0) TRACE(12);
  __syncthreads();
  if (threadIdx.x == 0) {
    TRACE(6);
    TRACE(7);
    tma_store_2d(tmY, otile, n0 + ycol, m0);
    bulk_commit();
    bulk_wait0();  // the tile is written (and its shared memory read) before the CTA exits
  }
}

// Split-K over a thread-block cluster: blockIdx.z = group * splits + split, and the `splits`
// CTAs of one output tile form a cluster (1 x 1 x splits).  Each accumulates its K range in
// TMEM and stages its fp32 tile in its own shared memory; after one cluster barrier rank r
// finalizes its share of the tile's 8-row groups by summing the `splits` tiles over DSMEM in
// rank order 0..splits-1 (deterministic), then runs the epilogue.  At the hot path's
// 128-token shapes a CTA's time is set by the bytes it ingests (~100 GB/s per SM measured,
// profiles/r01_gemm_trace.jsonl), so spreading a weight tile over `splits` SMs pays.
template <class T, int BN, int ACT, bool SPLIT, int IOT>
__global__ void __launch_bounds__(NT, 1)
    gemm_tc_kernel(const __grid_constant__ GemmGroup grp, const __grid_constant__ CUtensorMap tmX,
                   const __grid_constant__ CUtensorMap tmY, const void* res_, int ldr, void* Y, int ldy, int M, int N,
                   int K, int act, int io, int splits, int nst) {
  const void* res = EpiIO<IOT>::res(res_);
  const bool has_res = EpiIO<IOT>::has_res(res);
  constexpr int KS = ks_for<BN>();
  constexpr int STAGES = stages_for<BN>();
  constexpr uint32_t A_BYTES = KS * BM * BK * 2;  // KS x 16 KB
  constexpr uint32_t B_BYTES = KS * BN * BK * 2;
  constexpr uint32_t STAGE_BYTES = A_BYTES + B_BYTES;
  constexpr uint32_t TMEM_COLS = BN <= 32 ? 32 : BN <= 64 ? 64 : BN <= 128 ? 128 : 256;  // a power of 2
  constexpr int PROW = BN + 1;  // fp32 tile row stride (odd: conflict-free TMEM->smem writes)
  // kind::f16, fp32 accumulate, A/B K-major, M = 128, N = BN
  constexpr uint32_t IDESC = (1u << 4) | (FmtBits<T>::v << 7) | (FmtBits<T>::v << 10) | (uint32_t(BN >> 3) << 17) |
                             (uint32_t(BM >> 4) << 24);

  extern __shared__ uint8_t smem_raw[];
  // 1024-byte aligned for the 128-byte swizzle atoms; offset arithmetic on the __shared__ array
  // (not an integer round trip) keeps the pointer in the shared address space, so the
  // epilogue compiles to LDS/STS rather than generic loads/stores
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  __shared__ __align__(8) uint64_t full_bar[STAGES], empty_bar[STAGES], done_bar, recv_bar;
  __shared__ uint32_t tmem_base_sh;
  __shared__ float sbias[BM];
  __shared__ EpiParams ep;

  TRACE(0);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int n0 = blockIdx.x * BM, m0 = blockIdx.y * BN;
  const int grp_i = blockIdx.z / splits, sp = blockIdx.z - grp_i * splits;
  const CUtensorMap* tmW = &grp.w[grp_i];
  const T* bias = static_cast<const T*>(grp.bias[grp_i]);
  const long long ycol = grp.ycol[grp_i];
  const int kb_all = (K / BK + KS - 1) / KS;  // ring stages over the whole K (a last odd chunk: TMA zero fill)
  const int kb_lo = sp * kb_all / splits;
  const int num_kb = (sp + 1) * kb_all / splits - kb_lo;  // >= 1 (splits <= kb_all)
  const int mcount = min(BN, M - m0);
  const bool res32 = EpiIO<IOT>::res32(io), out32 = EpiIO<IOT>::out32(io);

  if (warp == 0 && lane == 0) {
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(tmW)) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&tmX)) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&tmY)) : "memory");
    ep = EpiParams{res, ldr, (int)ycol, io, mcount};
    // (rolled loops here and below: this thread runs them once, so unrolling only adds cold
    // instruction fetch in front of the first TMA)
#pragma unroll 1
    for (int s = 0; s < STAGES; ++s) {
      mbar_init(&full_bar[s], 1);
      mbar_init(&empty_bar[s], 1);
    }
    mbar_init(&done_bar, 1);
    mbar_init(&recv_bar, 1);  // split-K: the peers' partial rows land here (async-proxy pushes)
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    // Weights never depend on the previous kernel: the first ring's worth of W tiles goes in
    // flight right away -- before the TMEM allocation / CTA barrier and before the
    // grid-dependency wait (PDL) -- so its HBM latency overlaps the setup and the
    // predecessor's tail.  Activations (X, residual) and every store come after the wait.
    const int pre0 = num_kb < nst ? num_kb : nst;
#pragma unroll 1
    for (int kb = 0; kb < pre0; ++kb) {
      mbar_expect_tx(&full_bar[kb], STAGE_BYTES);
      tma_load_stage<KS>(tmW, &full_bar[kb], smem + kb * STAGE_BYTES, kb_lo + kb, n0);
    }
    TRACE(1);
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

  // nst <= STAGES: the ring depth actually used (a shallower ring leaves room on the SM for
  // the previous kernel's CTAs, so the PDL prologue overlap is not blocked on shared memory)
  const int pre = num_kb < nst ? num_kb : nst;
  // the bias never depends on the previous kernel either (128 threads = 128 rows of the tile;
  // read after the W tiles are in flight, visible to the epilogue after its barrier)
  if (threadIdx.x < BM) sbias[threadIdx.x] = bias != nullptr ? Cvt<T>::to1(bias[n0 + threadIdx.x]) : 0.f;
  if (threadIdx.x == 0) TRACE(2);
  pdl_wait();
  if (threadIdx.x == 0) TRACE(3);

  if (warp == 0 && lane == 0) {
    // TMA producer (stage s and its phase bit ph as running counters: no integer division)
    int s = 0;
    uint32_t ph = 0;
#pragma unroll 1
    for (int kb = 0; kb < num_kb; ++kb) {
      uint8_t* a = smem + s * STAGE_BYTES;
      uint8_t* b = a + A_BYTES;
      if (kb >= pre) {
        mbar_wait(&empty_bar[s], ph ^ 1u);
        mbar_expect_tx(&full_bar[s], STAGE_BYTES);
        tma_load_stage<KS>(tmW, &full_bar[s], a, kb_lo + kb, n0);
      }
      tma_load_stage<KS>(&tmX, &full_bar[s], b, kb_lo + kb, m0);
      if (++s == nst) s = 0, ph ^= 1u;
    }
  } else if (warp == 1 && lane == 0) {
    // MMA issuer
    int s = 0;
    uint32_t ph = 0;
#pragma unroll 1
    for (int kb = 0; kb < num_kb; ++kb) {
      mbar_wait(&full_bar[s], ph);
      if (kb == 0) TRACE(4);
      asm volatile("tcgen05.fence::after_thread_sync;");
      const uint8_t* a = smem + s * STAGE_BYTES;
      const uint8_t* b = a + A_BYTES;
      const uint64_t da = sw128_desc(a), db = sw128_desc(b);
#pragma unroll
      for (int kc = 0; kc < KS; ++kc)  // K chunk kc: sub-tiles BM x 128 B / BN x 128 B further on
#pragma unroll
        for (int kk = 0; kk < BK / 16; ++kk)  // advance 16 elements = 32 B = 2 in descriptor units
          umma_f16(tmem_d, da + (kc * BM * 128 >> 4) + 2 * kk, db + (kc * BN * 128 >> 4) + 2 * kk, IDESC,
                   (kb | kc | kk) != 0);
      umma_commit(&empty_bar[s]);
      if (++s == nst) s = 0, ph ^= 1u;
    }
    umma_commit(&done_bar);
  }
  __syncwarp();

  // one thread spins on the MMAs' completion and releases the CTA through its barrier (every
  // warp waiting on the mbarrier itself woke ~1 us late: try_wait suspends the waiter)
  if (threadIdx.x == 32) mbar_wait_spin(&done_bar, 0);
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (threadIdx.x == 0) TRACE(5);
  if (threadIdx.x == 64) TRACE(13);
  // split-K: announce that this CTA's MMAs are done, i.e. its TMA ring -- which the receive
  // slots below overlap -- is free.  Peers push into our receive slots only after the
  // matching wait.  (An arrive right after setup let a fast peer push while a slow CTA was
  // still streaming stages into that memory: a corrupted operand under SM contention, caught
  // by tools/stress_concurrency.py.)  Release orders our tensor-core reads of the ring before
  // the peers' async-proxy writes into it.
  if constexpr (SPLIT) asm volatile("barrier.cluster.arrive.release.aligned;" ::: "memory");
  asm volatile("tcgen05.fence::after_thread_sync;");
  // TMEM lane = W row within the tile; warp w reads its lane quarter (w % 4) for the column
  // half w / 4 of the tile
  const int row = (warp & 3) * 32 + lane;
  const int chalf = (warp >> 2) * (BN / 2);
  float* tile = reinterpret_cast<float*>(smem);
  if constexpr (!SPLIT) {
    store_tile<T, BN, ACT, IOT>(smem, tmem_d, sbias, &tmY, n0, m0, ep);
  } else {
    // 1) TMEM -> shared memory: this split's fp32 partial tile [128 W rows][BN tokens], unpadded,
    //    so each owner's rows are one contiguous block to push.  Within a row the 16-byte chunks
    //    are XOR-swizzled by (row & 7): the 32 lanes of a warp write 32 consecutive rows, BN * 4
    //    bytes apart (a multiple of 128 B), so the unswizzled float4 stores were 32-way bank
    //    conflicts -- 2-3 us per tile by the per-CTA trace (profiles/r02_gemm_trace_splitk.jsonl).
    //    Every tile and receive slot uses the same layout; the owner reads it back swizzled.
#pragma unroll 1
    for (int c0 = chalf; c0 < chalf + BN / 2; c0 += 16) {
      uint32_t v[16];
      tmem_ld16(tmem_d + (uint32_t((warp & 3) * 32) << 16) + c0, v);
#pragma unroll
      for (int j = 0; j < 16; j += 4)
        *reinterpret_cast<float4*>(&tile[row * BN + ((((c0 + j) >> 2) ^ (row & 7)) << 2)]) =
            make_float4(__uint_as_float(v[j]), __uint_as_float(v[j + 1]), __uint_as_float(v[j + 2]),
                        __uint_as_float(v[j + 3]));
    }
    // 2) + bias, activation, + residual; one 16-byte store per 8 outputs (8 W rows of a token)
    auto finish = [&](int nl, int ml, float* acc, const float* rpre = nullptr) {
      const size_t m = (size_t)(m0 + ml);
      const int nn = n0 + nl;
#pragma unroll
      for (int e = 0; e < 8; ++e) acc[e] = apply_act_c<ACT>(acc[e] + sbias[nl + e]);
      if (has_res) {
        float r8[8];
        if (rpre != nullptr) {
#pragma unroll
          for (int e = 0; e < 8; ++e) r8[e] = rpre[e];
        } else {
          load8<T>(res, m * ldr + nn, r8, res32);
        }
#pragma unroll
        for (int e = 0; e < 8; ++e) acc[e] += r8[e];
      }
      store8<T>(Y, m * ldy + nn + ycol, acc, out32);
    };
    // 1b) cluster split-K reduction: rank r owns tile rows [r*RPR, (r+1)*RPR).  Every CTA pushes
    //     the rows each peer owns from its send buffer into that peer's receive slot with a
    //     bulk async copy (cp.async.bulk shared::cta -> shared::cluster) that completes on the
    //     peer's recv_bar -- no cluster-wide barrier with a release fence, no latency-bound
    //     remote loads.  The owner sums the slots in rank order 0..splits-1 (deterministic).
    const int RPR = BM / splits;                     // rows per owner (splits is a power of 2)
    const uint32_t slot_bytes = uint32_t(RPR) * BN * 4;
    float* recv = tile + BM * BN;                    // [splits][RPR][BN]
    if (threadIdx.x == 0) {
      TRACE(6);
      // this CTA expects splits-1 slots; the arrival keeps the phase open until then
      asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(&recv_bar)),
                   "r"(slot_bytes * (splits - 1))
                   : "memory");
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // send buffer -> async proxy
    __syncthreads();
    asm volatile("barrier.cluster.wait.acquire.aligned;" ::: "memory");  // peers' rings free, recv_bar ready
    if (threadIdx.x == 0) {
      for (int r = 0; r < splits; ++r) {
        if (r == sp) continue;
        const uint32_t src = smem_u32(tile + r * RPR * BN);
        const uint32_t dst = mapa_u32(smem_u32(recv + sp * RPR * BN), (uint32_t)r);
        const uint32_t bar = mapa_u32(smem_u32(&recv_bar), (uint32_t)r);
        asm volatile(
            "cp.async.bulk.shared::cluster.shared::cta.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst),
            "r"(src), "r"(slot_bytes), "r"(bar)
            : "memory");
      }
      asm volatile("cp.async.bulk.commit_group;" ::: "memory");
    }
    mbar_wait(&recv_bar, 0);
    if (threadIdx.x == 0) TRACE(7);
    const int units = (RPR / 8) * mcount;
    if (!has_res) {
      for (int u = threadIdx.x; u < units; u += NT) {
        const int gi = u / mcount, ml = u - gi * mcount;  // 8-row group within the owned rows
        float acc[8] = {0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f};
        for (int p = 0; p < splits; ++p) {
          const float* sl = p == sp ? tile + sp * RPR * BN : recv + p * RPR * BN;
#pragma unroll
          for (int e = 0; e < 8; ++e) acc[e] += sl[(8 * gi + e) * BN + ((((ml >> 2) ^ e) << 2) | (ml & 3))];
        }
        finish(sp * RPR + 8 * gi, ml, acc);
      }
    } else {
      // with a residual: the residual loads of two units are issued before either is finished
      // (one latency per pair instead of one per unit; the 1024-token shapes finalise 2-4 units
      // per thread, the 128-token ones 1)
      for (int u0 = threadIdx.x; u0 < units; u0 += 2 * NT) {
        float r8[2][8];
#pragma unroll
        for (int b = 0; b < 2; ++b) {
          const int u = u0 + b * NT;
          if (u < units) {
            const int gi = u / mcount, ml = u - gi * mcount;
            load8<T>(res, (size_t)(m0 + ml) * ldr + n0 + sp * RPR + 8 * gi, r8[b], res32);
          }
        }
#pragma unroll
        for (int b = 0; b < 2; ++b) {
          const int u = u0 + b * NT;
          if (u >= units) break;
          const int gi = u / mcount, ml = u - gi * mcount;
          float acc[8] = {0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f};
          for (int p = 0; p < splits; ++p) {
            const float* sl = p == sp ? tile + sp * RPR * BN : recv + p * RPR * BN;
#pragma unroll
            for (int e = 0; e < 8; ++e) acc[e] += sl[(8 * gi + e) * BN + ((((ml >> 2) ^ e) << 2) | (ml & 3))];
          }
          finish(sp * RPR + 8 * gi, ml, acc, r8[b]);
        }
      }
    }
    // the pushes must have read this CTA's send buffer before it exits
    if (threadIdx.x == 0) asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
  }
#ifdef DP_GEMM_TRACE
  if (threadIdx.x == 0) {
    TRACE(8);
    unsigned smid;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
    const int b_ = (blockIdx.z * gridDim.y + blockIdx.y) * gridDim.x + blockIdx.x;
    if (b_ < 4096) g_gemm_trace[b_][15] = smid;
  }
#endif
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (warp == 1) {
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem_d), "r"(TMEM_COLS));
  }
}

// ---------------------------------------------------------------------------------------------
// K2p: the CTA-pair variant (tcgen05 cta_group::2).  Two CTAs of a (2 x 1 x 1) cluster -- one
// TPC -- compute a 256 x BN output tile with M = 256 MMAs issued by the even CTA (the leader):
// each CTA stages its own 128 W rows (the MMA's A halves) and HALF of the tile's BN tokens
// (the B halves), and the tensor cores read the peer's B half over the pair's shared-memory
// path.  Per CTA the ingest drops from 128 + BN to 128 + BN / 2 rows per k-block at the same
// MMA work; at the large models' shapes (M = 384 / 1024 tokens) the single-CTA mainloop was
// bound by what an SM can pull from L2 (~110 GB/s per SM, profiles/r02_gemm_trace.jsonl), not
// by the tensor pipe.  Each CTA's TMEM holds its own 128 W rows x all BN tokens, so the
// epilogue is K2's, per CTA.
//   * both CTAs' TMA loads complete on the LEADER's full barrier (the leader arms it with the
//     pair's bytes); the leader's MMA commits multicast to both CTAs' empty / done barriers;
//   * TMEM is allocated / freed by warp 1 of both CTAs (cta_group::2), and a cluster barrier
//     separates barrier init / allocation from the first TMA and the epilogue from the free.
template <int BN>
__host__ __device__ constexpr int stages_for_pair() {
  constexpr int bytes = BM * BK * 2 + (BN / 2) * BK * 2;
  constexpr int s = (224 * 1024) / bytes;
  return s > 12 ? 12 : s;
}

__device__ __forceinline__ void tma_load_2d_pair(const CUtensorMap* map, uint32_t bar_cluster, void* dst, int c0,
                                                 int c1) {
  asm volatile(
      "cp.async.bulk.tensor.2d.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, "
      "%3}], [%4];" ::"r"(smem_u32(dst)),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(c0), "r"(c1), "r"(bar_cluster)
      : "memory");
}
__device__ __forceinline__ void umma_f16_pair(uint32_t tmem_d, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "setp.ne.b32 p, %4, 0;\n"
      "tcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;\n"
      "}\n" ::"r"(tmem_d),
      "l"(a), "l"(b), "r"(idesc), "r"(acc));
}
// arrive on the barrier at this shared::cta offset in both CTAs of the pair when the MMAs
// issued so far complete
__device__ __forceinline__ void umma_commit_pair(uint64_t* bar) {
  asm volatile(
      "tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(
          smem_u32(bar)),
      "h"((unsigned short)3)
      : "memory");
}
__device__ __forceinline__ void cluster_sync_all() {
  asm volatile("barrier.cluster.arrive.release.aligned;\nbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}

template <class T, int BN, int ACT>
__global__ void __launch_bounds__(NT, 1)
    gemm_tc_pair_kernel(const __grid_constant__ GemmGroup grp, const __grid_constant__ CUtensorMap tmX,
                        const __grid_constant__ CUtensorMap tmY, const void* res, int ldr, int M, int K, int io,
                        int nst) {
  constexpr int HB = BN / 2;                 // tokens staged by each CTA
  constexpr uint32_t A_BYTES = BM * BK * 2;  // 16 KB
  constexpr uint32_t B_BYTES = HB * BK * 2;
  constexpr uint32_t STAGE_BYTES = A_BYTES + B_BYTES;
  constexpr int STAGES = stages_for_pair<BN>();
  constexpr uint32_t TMEM_COLS = BN <= 32 ? 32 : BN <= 64 ? 64 : BN <= 128 ? 128 : 256;
  // kind::f16, fp32 accumulate, A/B K-major, M = 256 (the pair), N = BN
  constexpr uint32_t IDESC = (1u << 4) | (FmtBits<T>::v << 7) | (FmtBits<T>::v << 10) | (uint32_t(BN >> 3) << 17) |
                             (uint32_t((2 * BM) >> 4) << 24);
  static_assert(BN % 32 == 0 && BN >= 64 && BN <= 256, "pair tile: BN in 64..256, a multiple of 32");

  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  __shared__ __align__(8) uint64_t full_bar[STAGES], empty_bar[STAGES], done_bar;
  __shared__ uint32_t tmem_base_sh;
  __shared__ float sbias[BM];
  __shared__ EpiParams ep;

  TRACE(0);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t rank = cta_cluster_rank();  // = blockIdx.x & 1
  const int n0 = blockIdx.x * BM, m0 = blockIdx.y * BN;
  const int xrow = m0 + int(rank) * HB;
  const CUtensorMap* tmW = &grp.w[blockIdx.z];
  const T* bias = static_cast<const T*>(grp.bias[blockIdx.z]);
  const int ycol = (int)grp.ycol[blockIdx.z];
  const int num_kb = K / BK;
  const int mcount = min(BN, M - m0);
  const bool res32 = io & IO_RES_F32, out32 = io & IO_OUT_F32;

  if (warp == 0 && lane == 0) {
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(tmW)) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&tmX)) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&tmY)) : "memory");
    ep = EpiParams{res, ldr, ycol, io, mcount};
    for (int s = 0; s < STAGES; ++s) {
      mbar_init(&full_bar[s], 1);
      mbar_init(&empty_bar[s], 1);
    }
    mbar_init(&done_bar, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&tmem_base_sh)),
                 "r"(TMEM_COLS));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  // the leader's barriers are initialised (the peer's loads complete on them) and both CTAs'
  // TMEM is allocated before anything is issued
  cluster_sync_all();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tmem_d = tmem_base_sh;
  const bool leader = rank == 0;
  // the leader's full barrier of stage s, as a shared::cluster address
  const uint32_t full0 = mapa_u32(smem_u32(&full_bar[0]), 0);
  const int pre = num_kb < nst ? num_kb : nst;
  if (warp == 0 && lane == 0) {
    // weights never depend on the previous kernel: the first ring of W tiles before the PDL wait
    for (int kb = 0; kb < pre; ++kb) {
      if (leader) mbar_expect_tx(&full_bar[kb], 2 * STAGE_BYTES);
      tma_load_2d_pair(tmW, full0 + kb * 8, smem + kb * STAGE_BYTES, kb * BK, n0);
    }
    TRACE(1);
  }
  pdl_trigger();
  if (threadIdx.x < BM) sbias[threadIdx.x] = bias != nullptr ? Cvt<T>::to1(bias[n0 + threadIdx.x]) : 0.f;
  if (threadIdx.x == 0) TRACE(2);
  pdl_wait();
  if (threadIdx.x == 0) TRACE(3);

  if (warp == 0 && lane == 0) {
    // TMA producer (both CTAs: own W rows, own half of the tokens)
    for (int kb = 0; kb < num_kb; ++kb) {
      const int s = kb % nst;
      uint8_t* a = smem + s * STAGE_BYTES;
      if (kb >= pre) {
        mbar_wait(&empty_bar[s], ((kb / nst) - 1) & 1);
        if (leader) mbar_expect_tx(&full_bar[s], 2 * STAGE_BYTES);
        tma_load_2d_pair(tmW, full0 + s * 8, a, kb * BK, n0);
      }
      tma_load_2d_pair(&tmX, full0 + s * 8, a + A_BYTES, kb * BK, xrow);
    }
  } else if (warp == 1 && lane == 0 && leader) {
    // MMA issuer (the leader only): the descriptors address the same offsets in both CTAs
    for (int kb = 0; kb < num_kb; ++kb) {
      const int s = kb % nst;
      mbar_wait(&full_bar[s], (kb / nst) & 1);
      if (kb == 0) TRACE(4);
      asm volatile("tcgen05.fence::after_thread_sync;");
      const uint8_t* a = smem + s * STAGE_BYTES;
      const uint64_t da = sw128_desc(a), db = sw128_desc(a + A_BYTES);
#pragma unroll
      for (int kk = 0; kk < BK / 16; ++kk) umma_f16_pair(tmem_d, da + 2 * kk, db + 2 * kk, IDESC, (kb | kk) != 0);
      umma_commit_pair(&empty_bar[s]);
    }
    umma_commit_pair(&done_bar);
  }
  __syncwarp();
  if (threadIdx.x == 32) mbar_wait_spin(&done_bar, 0);
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (threadIdx.x == 0) TRACE(5);
  asm volatile("tcgen05.fence::after_thread_sync;");
  store_tile<T, BN, ACT, 0>(smem, tmem_d, sbias, &tmY, n0, m0, ep);
#ifdef DP_GEMM_TRACE
  if (threadIdx.x == 0) {
    TRACE(8);
    unsigned smid;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
    const int b_ = (blockIdx.z * gridDim.y + blockIdx.y) * gridDim.x + blockIdx.x;
    if (b_ < 4096) g_gemm_trace[b_][15] = smid;
  }
#endif
  asm volatile("tcgen05.fence::before_thread_sync;");
  cluster_sync_all();  // both CTAs are done with the pair's TMEM before it is freed
  if (warp == 1) {
    asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem_d), "r"(TMEM_COLS));
  }
}

template <class T, int BN, int ACT, int IOT>
void run(const void* x, int ldx, int ngroups, const void* const* w, const void* const* bias, const long long* ycol,
         const void* res, int ldr, void* y, int ldy, int M, int N, int K, int act, int io, int splits,
         cudaStream_t s) {
  constexpr int KS = ks_for<BN>();
  constexpr int STAGES = stages_for<BN>();
  constexpr size_t STAGE_BYTES = KS * (BM * BK * 2 + BN * BK * 2);
  constexpr size_t smem_max = size_t(STAGES) * STAGE_BYTES + 1024;
  // the output tile (at most fp32) must fit the ring
  constexpr size_t epi_bytes = size_t(BM) * BN * 4;
  static_assert(epi_bytes + 1024 <= smem_max, "epilogue buffers must fit the ring");
  // split-K: unpadded send tile + receive slots, 2 x BM x BN fp32
  const size_t need = splits > 1 ? size_t(2) * BM * BN * 4 : epi_bytes;
  const int min_st = int((need + STAGE_BYTES - 1) / STAGE_BYTES);
  // ring depth: the full ring unless DP_GEMM_STAGES caps it (experiments), and never deeper
  // than the K blocks a CTA streams
  static const int env_st = experiment_env("DP_GEMM_STAGES", 0);
  int nst = env_st > 0 ? std::min(env_st, STAGES) : STAGES;
  nst = std::max(nst, std::max(min_st, 1));
  DP_CHECK(nst <= STAGES, DP_ERR_INVALID, "gemm: epilogue buffers do not fit this tile width");
  const size_t smem = size_t(nst) * STAGE_BYTES + 1024;
  // the single-split and split-K kernels are separate instantiations: each carries only its own
  // epilogue, and a CTA's first pass through its code is instruction-fetch bound (one cold
  // fetch per instruction; a larger split-K epilogue slowed even the kernels that never ran it)
  auto kern = gemm_tc_kernel<T, BN, ACT, false, IOT>;
  if constexpr (BN <= 128) {  // (wider tiles never split: the send + receive buffers would not fit)
    if (splits > 1) kern = gemm_tc_kernel<T, BN, ACT, true, IOT>;
  }
  static std::atomic<unsigned> attr{0}, attr_sp{0};
  if (first_on_device(splits > 1 ? attr_sp : attr))
    DP_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem_max));
  const int dtype = std::is_same<T, __half>::value ? DP_FP16 : DP_BF16;
  GemmGroup g;
  std::memset(&g, 0, sizeof(g));
  for (int i = 0; i < ngroups; ++i) {
    g.w[i] = KS == 1 ? make_kmajor_map(w[i], dtype, N, K, K, BM) : make_kmajor_map3(w[i], dtype, N, K, K, BM, KS);
    g.bias[i] = bias ? bias[i] : nullptr;
    g.ycol[i] = ycol ? ycol[i] : 0;
  }
  CUtensorMap mx = KS == 1 ? make_kmajor_map(x, dtype, M, K, ldx, BN) : make_kmajor_map3(x, dtype, M, K, ldx, BN, KS);
  // the output tile store (single split): Y as [M rows][ldy columns] in the output dtype, box
  // [BN tokens][128 features]
  const bool o32 = (io & IO_OUT_F32) != 0;
  const uint64_t ydims[2] = {(uint64_t)ldy, (uint64_t)M};
  const uint64_t ystr[1] = {(uint64_t)ldy * (o32 ? 4 : 2)};
  const uint32_t ybox[2] = {(uint32_t)BM, (uint32_t)BN};
  CUtensorMap my = make_plain_map(y, o32 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT32
                                         : (dtype == DP_BF16 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16
                                                             : CU_TENSOR_MAP_DATA_TYPE_FLOAT16),
                                  2, ydims, ystr, ybox);
  const int mt = (M + BN - 1) / BN;
  launch_kernel_cluster(kern, dim3(N / BM, mt, ngroups * splits), dim3(NT), smem,
                        dim3(1, 1, splits), s, g, mx, my, res, ldr, y, ldy, M, N, K, act, io, splits, nst);
}

// K2p host side: grid (N / 128, ceil(M / BN), groups), clusters of 2 along x (the pair's two
// 128-row W halves), one wave of BN-token tiles.
template <class T, int BN, int ACT>
void run_pair(const void* x, int ldx, int ngroups, const void* const* w, const void* const* bias,
              const long long* ycol, const void* res, int ldr, void* y, int ldy, int M, int N, int K, int io,
              cudaStream_t s) {
  constexpr int STAGES = stages_for_pair<BN>();
  constexpr size_t STAGE_BYTES = BM * BK * 2 + (BN / 2) * BK * 2;
  constexpr size_t smem_max = size_t(STAGES) * STAGE_BYTES + 1024;
  constexpr size_t epi_bytes = size_t(BM) * BN * 4;
  static_assert(epi_bytes + 1024 <= smem_max, "the output tile must fit the ring");
  static const int env_st = experiment_env("DP_GEMM_STAGES", 0);
  int nst = env_st > 0 ? std::min(env_st, STAGES) : STAGES;
  nst = std::max(nst, int((epi_bytes + STAGE_BYTES - 1) / STAGE_BYTES));
  const size_t smem = size_t(nst) * STAGE_BYTES + 1024;
  static std::atomic<unsigned> attr{0};
  if (first_on_device(attr))
    DP_CUDA(cudaFuncSetAttribute(gemm_tc_pair_kernel<T, BN, ACT>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 (int)smem_max));
  const int dtype = std::is_same<T, __half>::value ? DP_FP16 : DP_BF16;
  GemmGroup g;
  std::memset(&g, 0, sizeof(g));
  for (int i = 0; i < ngroups; ++i) {
    g.w[i] = make_kmajor_map(w[i], dtype, N, K, K, BM);
    g.bias[i] = bias ? bias[i] : nullptr;
    g.ycol[i] = ycol ? ycol[i] : 0;
  }
  CUtensorMap mx = make_kmajor_map(x, dtype, M, K, ldx, BN / 2);
  const bool o32 = (io & IO_OUT_F32) != 0;
  const uint64_t ydims[2] = {(uint64_t)ldy, (uint64_t)M};
  const uint64_t ystr[1] = {(uint64_t)ldy * (o32 ? 4 : 2)};
  const uint32_t ybox[2] = {(uint32_t)BM, (uint32_t)BN};
  CUtensorMap my = make_plain_map(y, o32 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT32
                                         : (dtype == DP_BF16 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16
                                                             : CU_TENSOR_MAP_DATA_TYPE_FLOAT16),
                                  2, ydims, ystr, ybox);
  launch_kernel_cluster(gemm_tc_pair_kernel<T, BN, ACT>, dim3(N / BM, (M + BN - 1) / BN, ngroups), dim3(NT), smem,
                        dim3(2, 1, 1), s, g, mx, my, res, ldr, M, K, io, nst);
}

template <class T>
void dispatch(int bn, bool pair, const void* x, int ldx, int ngroups, const void* const* w, const void* const* bias,
              const long long* ycol, const void* res, int ldr, void* y, int ldy, int M, int N, int K, int act, int io,
              int sp, cudaStream_t s) {
  if (pair) {
#define DP_RUNP(B, A) run_pair<T, B, A>(x, ldx, ngroups, w, bias, ycol, res, ldr, y, ldy, M, N, K, io, s)
#define DP_ACTSP(B)                                            \
  switch (act) {                                               \
    case ACT_NONE: DP_RUNP(B, ACT_NONE); break;                \
    case ACT_GELU_ERF: DP_RUNP(B, ACT_GELU_ERF); break;        \
    case ACT_GELU_TANH: DP_RUNP(B, ACT_GELU_TANH); break;      \
    case ACT_TANH: DP_RUNP(B, ACT_TANH); break;                \
    default: fail(DP_ERR_INVALID, "gemm: unknown activation"); \
  }
    switch (bn) {
      case 64: DP_ACTSP(64); break;
      case 128: DP_ACTSP(128); break;
      case 192: DP_ACTSP(192); break;
      case 256: DP_ACTSP(256); break;
      default: fail(DP_ERR_INVALID, "gemm: CTA-pair BN must be 64/128/192/256");
    }
#undef DP_ACTSP
#undef DP_RUNP
    return;
  }
  // the epilogue I/O variant (EpiIO): the forward pass's two fixed combinations, else generic
  const int iot = (res == nullptr && io == 0) ? 1 : (res != nullptr && io == (IO_RES_F32 | IO_OUT_F32)) ? 2 : 0;
#define DP_RUN(B, A)                                                                                 \
  do {                                                                                               \
    if (iot == 1)                                                                                    \
      run<T, B, A, 1>(x, ldx, ngroups, w, bias, ycol, res, ldr, y, ldy, M, N, K, act, io, sp, s);    \
    else if (iot == 2 && A == ACT_NONE)                                                              \
      run<T, B, A, (A == ACT_NONE ? 2 : 0)>(x, ldx, ngroups, w, bias, ycol, res, ldr, y, ldy, M, N, K, act, io, sp, s); \
    else                                                                                             \
      run<T, B, A, 0>(x, ldx, ngroups, w, bias, ycol, res, ldr, y, ldy, M, N, K, act, io, sp, s);    \
  } while (0)
#define DP_ACTS(B)                                 \
  switch (act) {                                   \
    case ACT_NONE: DP_RUN(B, ACT_NONE); break;           \
    case ACT_GELU_ERF: DP_RUN(B, ACT_GELU_ERF); break;   \
    case ACT_GELU_TANH: DP_RUN(B, ACT_GELU_TANH); break; \
    case ACT_TANH: DP_RUN(B, ACT_TANH); break;           \
    default: fail(DP_ERR_INVALID, "gemm: unknown activation"); \
  }
  switch (bn) {
    case 32: DP_ACTS(32); break;
    case 64: DP_ACTS(64); break;
    case 96: DP_ACTS(96); break;
    case 128: DP_ACTS(128); break;
    case 192: DP_ACTS(192); break;
    case 256: DP_ACTS(256); break;
    default: fail(DP_ERR_INVALID, "gemm: BN must be 32/64/96/128/192/256");
  }
#undef DP_ACTS
#undef DP_RUN
}

}  // namespace

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

// (BN, splits) from a per-CTA ingest model fitted to the B200 sweeps and per-CTA traces
// (profiles/r01_gemm_sweep_v4.txt, r01_gemm_trace.jsonl): a CTA streams its W and X tiles at
// ~100 GB/s (the mainloop time is its bytes / 1e5 B/us), all CTAs together at ~8 TB/s from
// L2/HBM, and the cluster split-K reduction (bulk DSMEM pushes) costs ~1.2 us.  Splits only in
// one wave of <= 148 CTAs, >= 4 k-blocks each, BN <= 128 (the send/receive buffers must fit).
// Picks the best measured configuration at every swept shape.  (Round 2: a refit to the
// back-to-back sweep after the split-K bank-conflict fix -- 0.3 us + pushed bytes at 33 KB/us,
// + 6 ns per token column -- chose other tiles at 3 of 15 shapes, 1% better back to back but
// 2-3% SLOWER in the PDL-chained forwards, profiles/r02_warm_ab_cost_model.jsonl: kept as is.)
struct GemmCfg {
  int bn, sp;
  bool pair;
};
// Hot-path shapes whose tiles were chosen by A/B in the warm forwards themselves (one shape
// forced at a time against the model's choice, instrumented build, DP_GEMM_CFG;
// profiles/r02_warm_ab_gemm_cfg.jsonl) where the model's pick lost: attn-out of BERT-Base
// (0.364 -> 0.347 ms), attn-out and q/k/v of BERT-Large (1.105 -> 1.074), GPT-2 Medium's c_proj
// (1.580 -> 1.516), BERT-Large fc1 on 96-token tiles (1.077 -> 1.065), GPT-2 Medium c_attn on
// 192-token tiles (1.493 -> 1.477).  Every other forward shape kept the model's pick (the
// alternatives tried were slower).  N is the total over the grouped weights (q/k/v: 3 x hidden).
struct MeasuredCfg {
  int M, N, K, bn, sp;
};
constexpr MeasuredCfg kMeasured[] = {
    {128, 768, 768, 32, 4},     // BERT-Base attn-out (S128)
    {384, 1024, 1024, 64, 2},   // BERT-Large / RoBERTa-Large attn-out (S384)
    {384, 3072, 1024, 64, 1},   // BERT-Large / RoBERTa-Large q/k/v (S384)
    {384, 4096, 1024, 96, 1},   // BERT-Large / RoBERTa-Large fc1 (S384): 4 exact 96-token tiles, 128 CTAs
    {1024, 1024, 1024, 64, 1},  // GPT-2 Medium c_proj (S1024)
    {1024, 3072, 1024, 192, 1}, // GPT-2 Medium c_attn (S1024): 144 CTAs in one wave (256-wide: 96)
};

static GemmCfg pick_cfg(int M, int N, int K) {
  for (const auto& c : kMeasured)
    if (c.M == M && c.N == N && c.K == K) return {c.bn, c.sp, false};
  const int ntile = N / BM, kb = K / BK;
  GemmCfg best{pick_bn(M, N), 1, false};
  double best_t = 1e30;
  for (int bn : {32, 64, 128, 256}) {
    if (bn > 32 && M < bn) continue;
    const int tiles = ntile * ((M + bn - 1) / bn);
    for (int sp : {1, 2, 4}) {
      if (sp > 1 && (kb / sp < 4 || tiles * sp > 148 || bn >= 256)) continue;
      const double per = double(kb) / sp * (BM * BK * 2 + bn * BK * 2);
      const int ctas = tiles * sp, waves = (ctas + 147) / 148;
      const double t = std::max(waves * per / 1e5, ctas * per / 8e6) + (sp > 1 ? 1.2 : 0.0);
      if (t < best_t - 1e-9) {
        best_t = t;
        best = {bn, sp, false};
      }
    }
  }
  return best;
}

static void gemm_impl(int dtype, const void* x, int ldx, int ngroups, const void* const* w, const void* const* bias,
                      const long long* ycol, const void* res, int ldr, void* y, int ldy, int M, int N, int K, int act,
                      int io, int bn_hint, int sp_hint, cudaStream_t s) {
  DP_CHECK(gemm_tc_supported(N, K), DP_ERR_UNSUPPORTED, "tcgen05 GEMM needs N % 128 == 0 and K % 64 == 0");
  DP_CHECK(ngroups >= 1 && ngroups <= 3, DP_ERR_INVALID, "gemm: 1..3 weight groups");
  DP_CHECK(ldx % 8 == 0 && ((uintptr_t)x % 16) == 0, DP_ERR_INVALID, "GEMM activations must be 16-byte aligned");
  for (int i = 0; i < ngroups; ++i)
    DP_CHECK(((uintptr_t)w[i] % 16) == 0 && (!ycol || ycol[i] % 8 == 0), DP_ERR_INVALID,
             "GEMM weights / output columns must be 16-byte aligned");
  DP_CHECK(ldy % 8 == 0 && (!res || ldr % 8 == 0), DP_ERR_INVALID, "GEMM output rows must be 16-byte aligned");
  if (M <= 0) return;
  // tuning override for experiments (DP_GEMM_BN), read once
  static const int env_bn = experiment_env("DP_GEMM_BN", 0);
  static const int env_sp = experiment_env("DP_GEMM_SPLIT", 0);
  GemmCfg cfg = pick_cfg(M, N * ngroups, K);
#ifdef DP_INSTRUMENT
  // per-shape override for chain A/B runs (instrumented builds only): DP_GEMM_CFG="M,N,K,bn,sp;..."
  // with N the total across groups (q/k/v: 3 x hidden)
  if (const char* e = std::getenv("DP_GEMM_CFG")) {
    for (const char* p = e; p && *p;) {
      int m, n, k, b, q;
      if (std::sscanf(p, "%d,%d,%d,%d,%d", &m, &n, &k, &b, &q) == 5 && m == M && n == N * ngroups && k == K)
        cfg = {b, q, false};
      p = std::strchr(p, ';');
      if (p) ++p;
    }
  }
#endif
  // bn_hint: 0 = the model's configuration, > 0 = a single-CTA tile of that width, < 0 = a
  // CTA pair (K2p) of width -bn_hint
  const bool hint_pair = bn_hint < 0;
  if (hint_pair) bn_hint = -bn_hint;
  const int bn = bn_hint > 0 ? bn_hint : (env_bn > 0 ? env_bn : cfg.bn);
  int sp = sp_hint > 0 ? sp_hint : env_sp > 0 ? env_sp : (bn_hint > 0 || env_bn > 0 ? 1 : cfg.sp);
  // every split needs >= 1 ring stage of ks_for<bn>() 64-deep K chunks
  const int ks = bn <= 64 ? ks_for<64>() : bn <= 128 ? ks_for<128>() : ks_for<256>();
  sp = std::max(1, std::min(std::min(sp, 8), (K / BK + ks - 1) / ks));
  while (sp & (sp - 1)) --sp;  // a power of two: every rank owns BM / sp rows
  if (bn > 128) sp = 1;        // the send + receive buffers (2 x 128 x BN fp32) must fit the ring
  // CTA pair (K2p): the model's choice unless a tile width is forced; DP_GEMM_PAIR=1 forces it
  // (with DP_GEMM_BN as the pair's tile width) for experiments
  static const int env_pair = experiment_env("DP_GEMM_PAIR", -1);
  bool pair = bn_hint > 0 || env_bn > 0 ? hint_pair : cfg.pair;
  if (env_pair >= 0) pair = env_pair > 0;
  if (pair) {
    DP_CHECK((N / BM) % 2 == 0, DP_ERR_INVALID, "gemm: a CTA pair needs N % 256 == 0");
    sp = 1;
  }
  if (dtype == DP_BF16)
    dispatch<__nv_bfloat16>(bn, pair, x, ldx, ngroups, w, bias, ycol, res, ldr, y, ldy, M, N, K, act, io, sp, s);
  else
    dispatch<__half>(bn, pair, x, ldx, ngroups, w, bias, ycol, res, ldr, y, ldy, M, N, K, act, io, sp, s);
}

void launch_gemm_tc_group(int dtype, const void* x, int ldx, int ngroups, const void* const* w,
                          const void* const* bias, const long long* ycol, const void* res, int ldr, void* y, int ldy,
                          int M, int N, int K, int act, int io, int bn_hint, cudaStream_t s, int sp_hint) {
  if (ablate_mask() & 4) return;
  gemm_impl(dtype, x, ldx, ngroups, w, bias, ycol, res, ldr, y, ldy, M, N, K, act, io, bn_hint, sp_hint, s);
}

void launch_gemm_tc(int dtype, const void* x, int ldx, const void* w, const void* bias, const void* res, int ldr,
                    void* y, int ldy, int M, int N, int K, int act, int io, int bn_hint, cudaStream_t s,
                    int sp_hint) {
  if (ablate_mask() & 4) return;
  launch_gemm_tc_group(dtype, x, ldx, 1, &w, &bias, nullptr, res, ldr, y, ldy, M, N, K, act, io, bn_hint, s,
                       sp_hint);
}

}  // namespace dp

#ifdef DP_GEMM_TRACE
extern "C" __attribute__((visibility("default"))) int dp_debug_gemm_trace(void* host, int nblocks) {
  if (nblocks > 4096) nblocks = 4096;
  return (int)cudaMemcpyFromSymbol(host, dp::g_gemm_trace, size_t(nblocks) * 16 * sizeof(unsigned long long));
}
#endif
