// SM-driven parallel-transmission forwarder (§4.2).
//
// The paper's PT: "each secondary GPU forwards its own partition to the primary GPU
// through NVLink ... we reserve a small amount of memory for storing layers temporarily on
// each GPU".  That is two copies per byte on a secondary: host -> staging ring (its copy
// engine, over its own PCIe link), then staging ring -> primary (a peer copy / NCCL send).
// On B200 one kernel can do both hops: the secondary's SMs read the pinned, mapped arena in
// place (16-byte zero-copy loads that cover whole 128-byte lines -- the DHA access pattern of
// P:99, so the bytes still cross the SECONDARY's PCIe link) and store each vector straight
// into the primary's HBM slot through the NVLink peer mapping.  No staging ring, no second
// copy, no per-piece NCCL call; the NVLink transfer overlaps the PCIe reads vector by vector.
//
// Completion.  In one process the forwarder runs on the secondary's load stream and an event
// after it gates the primary's execution stream (the same event graph as the DMA path).
// Across processes (one process per GPU) there is no shared event, so the ranks exchange
// CUDA IPC handles once (dp_peer_ipc_export / _import) for the model's HBM slots and a small
// mailbox per rank, and synchronise through memory:
//   * go:   the primary releases go = epoch into every secondary's mailbox at the start of a
//           cold start (its execution stream has finished everything before it, so the slots
//           are free to overwrite); a forwarder's CTAs acquire it before their first store;
//   * done: when the last CTA of a piece's forwarder has seen every CTA's system-scope fence,
//           it releases done[slot][piece] = epoch into the PRIMARY's mailbox; the primary's
//           execution stream acquires it (a one-thread wait kernel) right before the first
//           kernel that reads a unit of that piece (P:235's dependency check).
// `epoch` counts cold starts in this mode on every rank, so no flag is ever reset.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <vector>

#include "engine.h"
#include "kernels.h"
#include "peer.h"

namespace dp {

// Mailbox layout (uint32 words).  The primary's done words are written by secondaries; the
// counters are the forwarding rank's own (last-CTA detection per piece).
constexpr int kMbGo = 0;
constexpr int kMbEpoch = 1;  // this rank's current epoch, read by its signal / wait kernels (graph-safe)
constexpr int kMbMaxPieces = 256;
constexpr int kMbDone = 64;                                          // [slot][piece]
constexpr int kMbCount = kMbDone + DP_MAX_DEVICES * kMbMaxPieces;   // [piece]
constexpr int kMbWords = kMbCount + kMbMaxPieces;
constexpr size_t kMbBytes = 16384;
static_assert(kMbWords * 4 <= (int)kMbBytes, "mailbox layout exceeds its allocation");

namespace {

__device__ __forceinline__ uint32_t ld_acquire_sys(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_sys(uint32_t* p, uint32_t v) {
  asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ uint64_t globaltimer() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
// Spin until *flag >= value (wrap-safe).  A peer that never arrives must not hang the GPU:
// after 30 s the kernel traps (the process gets an error instead of a stuck device).
__device__ __forceinline__ void wait_flag(const uint32_t* flag, uint32_t value) {
  const uint64_t t0 = globaltimer();
  while ((int32_t)(ld_acquire_sys(flag) - value) < 0) {
    __nanosleep(128);
    if (globaltimer() - t0 > 30ull * 1000000000ull) __trap();
  }
}

__device__ __forceinline__ uint4 ld_host_v4(const uint4* p) {
  uint4 v;
  asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
               : "l"(p));
  return v;
}

constexpr int kFwdThreads = 256;
constexpr int kFwdUnroll = 4;  // 16-byte loads in flight per thread before the first store

// K7: forward n16 16-byte vectors (+ a byte tail) from host-mapped src to dst (local or peer
// HBM).  Each warp instruction covers 512 contiguous bytes = four whole 128-byte lines; all
// kFwdUnroll loads of a thread are issued before its stores, so a CTA keeps 16 KiB of reads
// in flight over the link.
__global__ void __launch_bounds__(kFwdThreads) pt_forward_kernel(const uint4* __restrict__ src, uint4* dst,
                                                                  long long n16, const uint8_t* src_tail,
                                                                  uint8_t* dst_tail, int tail, const uint32_t* go,
                                                                  uint32_t epoch, uint32_t* counter, uint32_t* done) {
  if (go) {
    if (threadIdx.x == 0) wait_flag(go, epoch);
    __syncthreads();
  }
  const long long step = (long long)gridDim.x * kFwdThreads * kFwdUnroll;
  for (long long base = (long long)blockIdx.x * kFwdThreads * kFwdUnroll + threadIdx.x; base < n16; base += step) {
    uint4 v[kFwdUnroll];
#pragma unroll
    for (int j = 0; j < kFwdUnroll; ++j) {
      const long long i = base + (long long)j * kFwdThreads;
      if (i < n16) v[j] = ld_host_v4(src + i);
    }
#pragma unroll
    for (int j = 0; j < kFwdUnroll; ++j) {
      const long long i = base + (long long)j * kFwdThreads;
      if (i < n16) dst[i] = v[j];
    }
  }
  if (blockIdx.x == 0 && (int)threadIdx.x < tail) dst_tail[threadIdx.x] = src_tail[threadIdx.x];
  if (done) {
    __threadfence_system();  // this thread's stores are visible system-wide before the count
    __syncthreads();
    if (threadIdx.x == 0) {
      const uint32_t prev = atomicAdd(counter, 1u);
      if (prev == gridDim.x - 1) {  // every CTA has fenced: the piece has landed
        atomicExch(counter, 0u);    // reused by the next cold start (stream-ordered)
        __threadfence_system();
        st_release_sys(done, epoch);
      }
    }
  }
}

struct FlagPtrs {
  uint32_t* p[DP_MAX_DEVICES];
};

// value_word != nullptr: the value is read from that device word (the primary's epoch, so a
// captured CUDA graph stays valid across cold starts)
__global__ void pt_signal_kernel(FlagPtrs f, int n, uint32_t value, const uint32_t* value_word) {
  if ((int)threadIdx.x < n) {
    const uint32_t v = value_word ? *value_word : value;
    __threadfence_system();
    st_release_sys(f.p[threadIdx.x], v);
  }
}

__global__ void pt_set_word_kernel(uint32_t* w, uint32_t v) { *w = v; }

__global__ void pt_wait_kernel(const uint32_t* flag, uint32_t value, const uint32_t* value_word) {
  wait_flag(flag, value_word ? *value_word : value);
}

int sm_count(int dev) {
  static int cache[DP_MAX_DEVICES] = {};
  if (dev < 0 || dev >= DP_MAX_DEVICES) return 148;
  if (!cache[dev]) {
    int n = 0;
    if (cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || n <= 0) n = 148;
    cache[dev] = n;
  }
  return cache[dev];
}

}  // namespace

void launch_pt_forward(const void* src, void* dst, int64_t bytes, cudaStream_t s, const uint32_t* go, uint32_t epoch,
                       uint32_t* counter, uint32_t* done) {
  DP_CHECK(bytes >= 0, DP_ERR_INVALID, "negative byte count");
  DP_CHECK(((uintptr_t)src & 15) == 0 && ((uintptr_t)dst & 15) == 0, DP_ERR_INVALID,
           "pt_forward: src/dst must be 16-byte aligned");
  const long long n16 = bytes / 16;
  const int tail = (int)(bytes % 16);
  int dev = 0;
  DP_CUDA(cudaGetDevice(&dev));
  const long long per_cta = (long long)kFwdThreads * kFwdUnroll;
  const long long want = std::max<long long>(1, (n16 + per_cta - 1) / per_cta);
  static const int cta_cap = std::max(0, experiment_env("DP_PT_FWD_CTAS", 0));  // experiments: grid cap
  const int grid = (int)std::min<long long>(want, cta_cap ? cta_cap : 2LL * sm_count(dev));
  pt_forward_kernel<<<grid, kFwdThreads, 0, s>>>(static_cast<const uint4*>(src), static_cast<uint4*>(dst), n16,
                                                static_cast<const uint8_t*>(src) + n16 * 16,
                                                static_cast<uint8_t*>(dst) + n16 * 16, tail, go, epoch, counter,
                                                done);
  DP_CUDA(cudaGetLastError());
}

// ---------------------------------------------------------------------------------------
// Multi-process (CUDA IPC) side of the engine
// ---------------------------------------------------------------------------------------

static uint32_t* done_word(uint32_t* mailbox, int slot, size_t piece) {
  return mailbox + kMbDone + slot * kMbMaxPieces + piece;
}

static void ensure_mailbox(dp_context* ctx) {
  if (ctx->mailbox) return;
  void* p = nullptr;
  if (cudaMalloc(&p, kMbBytes) != cudaSuccess) fail(DP_ERR_OOM, "mailbox cudaMalloc failed");
  DP_CUDA(cudaMemset(p, 0, kMbBytes));
  DP_CUDA(cudaDeviceSynchronize());
  ctx->mailbox = static_cast<uint32_t*>(p);
}

void ipc_set_epoch(dp_context* ctx, uint32_t epoch, cudaStream_t exec) {
  pt_set_word_kernel<<<1, 1, 0, exec>>>(ctx->mailbox + kMbEpoch, epoch);
  DP_CUDA(cudaGetLastError());
}

void ipc_primary_begin(dp_context* ctx, const dp_plan* plan, int prim_rank, cudaStream_t exec) {
  FlagPtrs f{};
  int n = 0;
  for (int s = 1; s < plan->k; ++s) {
    const int r = peer_rank_of_slot(ctx, prim_rank, s);
    DP_CHECK(ctx->peer_mailbox[r], DP_ERR_STATE, "rank " + std::to_string(r) + "'s mailbox is not imported");
    f.p[n++] = ctx->peer_mailbox[r] + kMbGo;
  }
  if (!n) return;
  pt_signal_kernel<<<1, 32, 0, exec>>>(f, n, 0, ctx->mailbox + kMbEpoch);
  DP_CUDA(cudaGetLastError());
}

void launch_pt_wait(const uint32_t* flag, uint32_t value, cudaStream_t s) {
  pt_wait_kernel<<<1, 1, 0, s>>>(flag, value, nullptr);
  DP_CUDA(cudaGetLastError());
}

void ipc_primary_wait(dp_context* ctx, int slot, size_t piece, cudaStream_t exec) {
  DP_CHECK(piece < (size_t)kMbMaxPieces, DP_ERR_UNSUPPORTED, "too many PT pieces for the mailbox");
  pt_wait_kernel<<<1, 1, 0, exec>>>(done_word(ctx->mailbox, slot, piece), 0, ctx->mailbox + kMbEpoch);
  DP_CUDA(cudaGetLastError());
}

__global__ void pt_wait_many_kernel(FlagPtrs f, int n, const uint32_t* value_word) {
  if ((int)threadIdx.x < n) wait_flag(f.p[threadIdx.x], *value_word);
}

void ipc_primary_wait_many(dp_context* ctx, const std::vector<std::pair<int, size_t>>& pieces, cudaStream_t exec) {
  FlagPtrs f{};
  int n = 0;
  for (const auto& sp : pieces) {
    DP_CHECK(sp.second < (size_t)kMbMaxPieces, DP_ERR_UNSUPPORTED, "too many PT pieces for the mailbox");
    DP_CHECK(n < DP_MAX_DEVICES, DP_ERR_INVALID, "internal: more than one wait per link in a batch");
    f.p[n++] = done_word(ctx->mailbox, sp.first, sp.second);
  }
  if (!n) return;
  pt_wait_many_kernel<<<1, 32, 0, exec>>>(f, n, ctx->mailbox + kMbEpoch);
  DP_CUDA(cudaGetLastError());
}

void ipc_check_primary(dp_context* ctx) {
  DP_CHECK(ctx->mailbox, DP_ERR_STATE, "SM transport across processes: call dp_peer_ipc_export/_import first");
}

void ipc_send_rank(dp_context* ctx, dp_model* m, const dp_plan* plan, int primary, dp_run_stats* stats) {
  dp_run_stats st;
  std::memset(&st, 0, sizeof(st));
  if (plan->k <= 1) {  // no PT slots: not a rendezvous, no epoch
    if (stats) *stats = st;
    return;
  }
  const uint32_t epoch = ++ctx->pt_epoch;  // every rank counts the same k > 1 cold starts
  int slot = -1;
  for (int s = 1; s < plan->k; ++s)
    if (peer_rank_of_slot(ctx, primary, s) == ctx->rank) slot = s;
  if (slot < 0) {
    if (stats) *stats = st;
    return;
  }
  DP_CHECK(ctx->mailbox && ctx->peer_mailbox[primary] && m->peer_dbase[primary], DP_ERR_STATE,
           "SM transport across processes: call dp_peer_ipc_export/_import first");
  auto pcs = slot_pieces(m, plan, slot, opt_cap(ctx), opt_tail(ctx));
  DP_CHECK(pcs.size() <= (size_t)kMbMaxPieces, DP_ERR_UNSUPPORTED, "too many PT pieces for the mailbox");
  if (!ctx->comm_stream) DP_CUDA(cudaStreamCreateWithFlags(&ctx->comm_stream, cudaStreamNonBlocking));
  uint8_t* dst = static_cast<uint8_t*>(m->peer_dbase[primary]);
  const bool ce = ctx->opts.pt_transport == DP_PT_CE;
  if (ce && !pcs.empty()) {  // the copy engine cannot poll: a one-thread kernel acquires `go`
    pt_wait_kernel<<<1, 1, 0, ctx->comm_stream>>>(ctx->mailbox + kMbGo, epoch, nullptr);
    DP_CUDA(cudaGetLastError());
  }
  for (size_t r = 0; r < pcs.size(); ++r) {
    const Piece& pc = pcs[r];
    if (ctx->opts.debug_delay_us > 0) launch_spin((long long)ctx->opts.debug_delay_us * 2000, ctx->comm_stream);
    if (ce) {  // one DMA host -> the primary's slot through the IPC mapping, then release done
      DP_CUDA(cudaMemcpyAsync(dst + pc.off, static_cast<const uint8_t*>(m->arena) + pc.off, pc.bytes,
                              cudaMemcpyDefault, ctx->comm_stream));
      FlagPtrs f{};
      f.p[0] = done_word(ctx->peer_mailbox[primary], slot, r);
      pt_signal_kernel<<<1, 32, 0, ctx->comm_stream>>>(f, 1, epoch, nullptr);
      DP_CUDA(cudaGetLastError());
      st.h2d_bytes[slot] += pc.bytes;
      st.nvlink_bytes[slot] += pc.bytes;
      ++st.n_copies;
      continue;
    }
    launch_pt_forward(static_cast<const uint8_t*>(m->arena) + pc.off, dst + pc.off, pc.bytes, ctx->comm_stream,
                      r == 0 ? ctx->mailbox + kMbGo : nullptr, epoch, ctx->mailbox + kMbCount + r,
                      done_word(ctx->peer_mailbox[primary], slot, r));
    st.h2d_bytes[slot] += pc.bytes;
    st.nvlink_bytes[slot] += pc.bytes;
  }
  if (stats) *stats = st;
}

void ipc_close(dp_context* ctx) {
  for (int r = 0; r < DP_MAX_DEVICES; ++r)
    if (ctx->peer_mailbox[r]) {
      cudaIpcCloseMemHandle(ctx->peer_mailbox[r]);
      ctx->peer_mailbox[r] = nullptr;
    }
  if (ctx->mailbox) cudaFree(ctx->mailbox);
  ctx->mailbox = nullptr;
}

void ipc_close_model(dp_model* m) {
  for (int r = 0; r < DP_MAX_DEVICES; ++r)
    if (m->peer_dbase[r]) {
      cudaIpcCloseMemHandle(m->peer_dbase[r]);
      m->peer_dbase[r] = nullptr;
    }
}

}  // namespace dp

using namespace dp;

extern "C" dp_status dp_pt_forward(const void* src, void* dst, int64_t bytes, void* stream) {
  return guard([&] {
    DP_CHECK(src && dst, DP_ERR_INVALID, "NULL argument");
    launch_pt_forward(src, dst, bytes, (cudaStream_t)stream, nullptr, 0, nullptr, nullptr);
  });
}

extern "C" dp_status dp_peer_init_ipc(dp_context* ctx, int32_t rank, int32_t nranks) {
  return guard([&] {
    DP_CHECK(ctx, DP_ERR_INVALID, "NULL argument");
    DP_CHECK(nranks >= 1 && nranks <= DP_MAX_DEVICES && rank >= 0 && rank < nranks, DP_ERR_INVALID,
             "bad rank/nranks");
    DP_CHECK(ctx->devs.size() == 1, DP_ERR_INVALID, "multi-process PT needs a one-device context per process");
    DP_CHECK(!ctx->multiproc(), DP_ERR_STATE, "peer transport already initialised");
    ctx->rank = rank;
    ctx->nranks = nranks;
  });
}

extern "C" dp_status dp_peer_ipc_export(dp_context* ctx, dp_model* m, void* out) {
  return guard([&] {
    DP_CHECK(ctx && m && out, DP_ERR_INVALID, "NULL argument");
    DP_CHECK(ctx->multiproc(), DP_ERR_STATE, "call dp_peer_init or dp_peer_init_ipc first");
    static_assert(2 * sizeof(cudaIpcMemHandle_t) <= DP_IPC_HANDLE_BYTES, "IPC block too small");
    const int dev = ctx->devs[0];
    ctx->on(dev);
    int prev = 0;
    DP_CUDA(cudaGetDevice(&prev));
    DP_CUDA(cudaSetDevice(dev));
    try {
      pin_full_slots(m, dev);
      ensure_mailbox(ctx);
      cudaIpcMemHandle_t h[2];
      DP_CUDA(cudaIpcGetMemHandle(&h[0], m->dev[dev].dbase));
      DP_CUDA(cudaIpcGetMemHandle(&h[1], ctx->mailbox));
      std::memset(out, 0, DP_IPC_HANDLE_BYTES);
      std::memcpy(out, h, sizeof(h));
    } catch (...) {
      cudaSetDevice(prev);
      throw;
    }
    cudaSetDevice(prev);
  });
}

extern "C" dp_status dp_peer_ipc_import(dp_context* ctx, dp_model* m, const void* all) {
  return guard([&] {
    DP_CHECK(ctx && m && all, DP_ERR_INVALID, "NULL argument");
    DP_CHECK(ctx->multiproc(), DP_ERR_STATE, "call dp_peer_init or dp_peer_init_ipc first");
    DP_CHECK(ctx->mailbox, DP_ERR_STATE, "call dp_peer_ipc_export first");
    int prev = 0;
    DP_CUDA(cudaGetDevice(&prev));
    DP_CUDA(cudaSetDevice(ctx->devs[0]));
    try {
      for (int r = 0; r < ctx->nranks; ++r) {
        if (r == ctx->rank) continue;
        cudaIpcMemHandle_t h[2];
        std::memcpy(h, static_cast<const uint8_t*>(all) + (size_t)r * DP_IPC_HANDLE_BYTES, sizeof(h));
        if (!m->peer_dbase[r]) {
          void* p = nullptr;
          DP_CUDA(cudaIpcOpenMemHandle(&p, h[0], cudaIpcMemLazyEnablePeerAccess));
          m->peer_dbase[r] = p;
        }
        if (!ctx->peer_mailbox[r]) {
          void* p = nullptr;
          DP_CUDA(cudaIpcOpenMemHandle(&p, h[1], cudaIpcMemLazyEnablePeerAccess));
          ctx->peer_mailbox[r] = static_cast<uint32_t*>(p);
        }
      }
    } catch (...) {
      cudaSetDevice(prev);
      throw;
    }
    cudaSetDevice(prev);
  });
}
