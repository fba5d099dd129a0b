// Parallel transmission across processes (one process per GPU): the reduce phase of
// PAPER.md §4.2 -- "each secondary GPU forwards its own partition to the primary
// GPU through NVLink ... we can overlap the reduce phase with the transmission for the
// first partition" -- implemented with NCCL point-to-point send/recv only (no collective).
//
// Secondary rank r serving slot s: for each piece (whole units, forward order) it DMAs the
// piece from the pinned arena over ITS OWN PCIe link into a staging ring ("we reserve
// a small amount of memory for storing layers temporarily on each GPU"), then ncclSend()s
// it to the primary as soon as it lands (parallel-pipeline).  The primary posts one
// NCCL group per round (piece r of every secondary) straight into the model's HBM slots and
// records one event per round; the execution stream waits on it before the first kernel of
// those units.  NCCL is loaded at run time (the copy torch already loaded).
#include <dlfcn.h>

#include <algorithm>
#include <cstring>

#include <nccl.h>

#include "peer.h"

namespace dp {

namespace {

struct Nccl {
  void* h = nullptr;
  decltype(&ncclGetUniqueId) getUniqueId = nullptr;
  decltype(&ncclCommInitRank) commInitRank = nullptr;
  decltype(&ncclCommDestroy) commDestroy = nullptr;
  decltype(&ncclSend) send = nullptr;
  decltype(&ncclRecv) recv = nullptr;
  decltype(&ncclGroupStart) groupStart = nullptr;
  decltype(&ncclGroupEnd) groupEnd = nullptr;
  decltype(&ncclGetErrorString) errStr = nullptr;
};

Nccl& nccl() {
  static Nccl n;
  if (n.h) return n;
  n.h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
  DP_CHECK(n.h != nullptr, DP_ERR_NCCL, std::string("cannot load libnccl.so.2: ") + dlerror());
  auto sym = [&](const char* name) {
    void* p = dlsym(n.h, name);
    DP_CHECK(p != nullptr, DP_ERR_NCCL, std::string("NCCL symbol missing: ") + name);
    return p;
  };
  n.getUniqueId = (decltype(n.getUniqueId))sym("ncclGetUniqueId");
  n.commInitRank = (decltype(n.commInitRank))sym("ncclCommInitRank");
  n.commDestroy = (decltype(n.commDestroy))sym("ncclCommDestroy");
  n.send = (decltype(n.send))sym("ncclSend");
  n.recv = (decltype(n.recv))sym("ncclRecv");
  n.groupStart = (decltype(n.groupStart))sym("ncclGroupStart");
  n.groupEnd = (decltype(n.groupEnd))sym("ncclGroupEnd");
  n.errStr = (decltype(n.errStr))sym("ncclGetErrorString");
  return n;
}

#define DP_NCCL(x)                                                                                          \
  do {                                                                                                      \
    ncclResult_t r__ = (x);                                                                                 \
    if (r__ != ncclSuccess) ::dp::fail(DP_ERR_NCCL, std::string(#x) + " failed: " + nccl().errStr(r__)); \
  } while (0)

struct PeerState {
  cudaStream_t h2d = nullptr;  // secondary: load stream into the ring
  void* ring = nullptr;
  int64_t ring_bytes = 0;
  std::vector<cudaEvent_t> ev;  // recycled
  size_t used = 0;
  cudaEvent_t last = nullptr;   // primary: last recv round
  // secondary: the previous cold start's last send (its ring slots are free only after it);
  // the next call's first H2D into the ring waits on it (ncclSend blocks until the
  // primary posts its recv, so the previous call's sends may still be reading the ring)
  cudaEvent_t sends_done = nullptr;
  bool sends_pending = false;
  cudaEvent_t get() {
    if (used == ev.size()) {
      cudaEvent_t e;
      DP_CUDA(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
      ev.push_back(e);
    }
    return ev[used++];
  }
};

PeerState& ps(dp_context* ctx) {
  static PeerState* s = nullptr;  // one per process (one comm per process)
  if (!s) s = new PeerState();
  return *s;
}

constexpr int kRing = 3;

}  // namespace

int peer_rank_of_slot(const dp_context* ctx, int primary, int slot) {
  // a map set by dp_peer_set_slot_ranks (e.g. from dp_select_secondaries on the measured link
  // matrix) for this primary, else the fixed rotation
  if (slot > 0 && ctx->slot_map_primary == primary && slot < DP_MAX_DEVICES && ctx->slot_rank[slot] >= 0)
    return ctx->slot_rank[slot];
  return (primary + slot) % ctx->nranks;
}

void peer_recv_all(dp_context* ctx, dp_model* m, const dp_plan* plan, int primary, int dev, cudaEvent_t fork,
                   std::vector<cudaEvent_t>& unit_ev, dp_run_stats& st) {
  PeerState& p = ps(ctx);
  p.used = 0;
  DP_CHECK(plan->k <= ctx->nranks, DP_ERR_INVALID, "plan.k exceeds the number of ranks");
  const int64_t cap = std::max<int64_t>(ctx->opts.chunk_bytes, 4096);
  std::vector<std::vector<Piece>> pcs(plan->k);
  size_t rounds = 0;
  for (int s = 1; s < plan->k; ++s) {
    pcs[s] = slot_pieces(m, plan, s, cap, opt_tail(ctx));
    rounds = std::max(rounds, pcs[s].size());
  }
  DP_CUDA(cudaStreamWaitEvent(ctx->comm_stream, fork, 0));
  auto* comm = static_cast<ncclComm_t>(ctx->comm);
  for (size_t r = 0; r < rounds; ++r) {
    DP_NCCL(nccl().groupStart());
    for (int s = 1; s < plan->k; ++s) {
      if (r >= pcs[s].size()) continue;
      const Piece& pc = pcs[s][r];
      DP_NCCL(nccl().recv(m->device(dev, pc.first_unit), pc.bytes, ncclUint8, peer_rank_of_slot(ctx, primary, s), comm,
                          ctx->comm_stream));
      st.nvlink_bytes[s] += pc.bytes;
    }
    DP_NCCL(nccl().groupEnd());
    cudaEvent_t e = p.get();
    DP_CUDA(cudaEventRecord(e, ctx->comm_stream));
    ++st.n_events;
    for (int s = 1; s < plan->k; ++s)
      if (r < pcs[s].size()) bind_units(unit_ev, pcs[s][r], e);
    p.last = e;
  }
}

void peer_join(dp_context* ctx, cudaStream_t exec) {
  PeerState& p = ps(ctx);
  if (p.last) DP_CUDA(cudaStreamWaitEvent(exec, p.last, 0));
  p.last = nullptr;
}

void peer_send_rank(dp_context* ctx, dp_model* m, const dp_plan* plan, int primary, dp_run_stats* stats) {
  PeerState& p = ps(ctx);
  p.used = 0;
  int slot = -1;
  for (int s = 1; s < plan->k; ++s)
    if (peer_rank_of_slot(ctx, primary, s) == ctx->rank) slot = s;
  dp_run_stats st;
  std::memset(&st, 0, sizeof(st));
  if (slot < 0) {  // this rank carries no partition of the plan
    if (stats) *stats = st;
    return;
  }
  const int64_t cap = std::max<int64_t>(ctx->opts.chunk_bytes, 4096);
  auto pcs = slot_pieces(m, plan, slot, cap, opt_tail(ctx));
  int64_t big = 0;
  for (auto& pc : pcs) big = std::max(big, pc.bytes);
  if (!p.h2d) DP_CUDA(cudaStreamCreateWithFlags(&p.h2d, cudaStreamNonBlocking));
  if (!p.sends_done) DP_CUDA(cudaEventCreateWithFlags(&p.sends_done, cudaEventDisableTiming));
  if (p.sends_pending) DP_CUDA(cudaStreamWaitEvent(p.h2d, p.sends_done, 0));
  if (p.ring_bytes < kRing * big) {
    if (p.ring) {
      DP_CUDA(cudaStreamSynchronize(ctx->comm_stream));  // earlier sends still read the old ring
      DP_CUDA(cudaFree(p.ring));
    }
    p.ring = nullptr;
    if (cudaMalloc(&p.ring, kRing * big) != cudaSuccess) fail(DP_ERR_OOM, "staging ring cudaMalloc failed");
    p.ring_bytes = kRing * big;
  }
  auto* comm = static_cast<ncclComm_t>(ctx->comm);
  std::vector<cudaEvent_t> sent(pcs.size(), nullptr);
  for (size_t r = 0; r < pcs.size(); ++r) {
    const Piece& pc = pcs[r];
    uint8_t* stage = static_cast<uint8_t*>(p.ring) + (r % kRing) * big;
    if (r >= (size_t)kRing) DP_CUDA(cudaStreamWaitEvent(p.h2d, sent[r - kRing], 0));
    DP_CUDA(cudaMemcpyAsync(stage, static_cast<const uint8_t*>(m->arena) + pc.off, pc.bytes, cudaMemcpyHostToDevice,
                            p.h2d));
    st.h2d_bytes[slot] += pc.bytes;
    ++st.n_copies;
    cudaEvent_t landed = p.get();
    DP_CUDA(cudaEventRecord(landed, p.h2d));
    DP_CUDA(cudaStreamWaitEvent(ctx->comm_stream, landed, 0));
    DP_NCCL(nccl().send(stage, pc.bytes, ncclUint8, primary, comm, ctx->comm_stream));
    st.nvlink_bytes[slot] += pc.bytes;
    cudaEvent_t done = p.get();
    DP_CUDA(cudaEventRecord(done, ctx->comm_stream));
    sent[r] = done;
    st.n_events += 2;
  }
  DP_CUDA(cudaEventRecord(p.sends_done, ctx->comm_stream));
  p.sends_pending = true;
  if (stats) *stats = st;
}

void peer_destroy(dp_context* ctx) {
  if (!ctx->comm) return;
  nccl().commDestroy(static_cast<ncclComm_t>(ctx->comm));
  ctx->comm = nullptr;
  if (ctx->comm_stream) cudaStreamDestroy(ctx->comm_stream);
  ctx->comm_stream = nullptr;
}

}  // namespace dp

using namespace dp;

extern "C" dp_status dp_peer_unique_id(void* out128) {
  return guard([&] {
    DP_CHECK(out128, DP_ERR_INVALID, "NULL argument");
    static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId is 128 bytes");
    ncclUniqueId id;
    DP_NCCL(nccl().getUniqueId(&id));
    std::memcpy(out128, &id, sizeof(id));
  });
}

extern "C" dp_status dp_peer_set_slot_ranks(dp_context* ctx, int32_t primary, const int32_t* rank_of_slot,
                                            int32_t k) {
  return guard([&] {
    DP_CHECK(ctx && ctx->multiproc(), DP_ERR_STATE, "call dp_peer_init or dp_peer_init_ipc first");
    DP_CHECK(primary >= 0 && primary < ctx->nranks && k >= 1 && k <= ctx->nranks && (k == 1 || rank_of_slot),
             DP_ERR_INVALID, "bad primary / k");
    std::vector<char> seen(ctx->nranks, 0);
    seen[primary] = 1;
    for (int s = 1; s < k; ++s) {
      const int r = rank_of_slot[s - 1];
      DP_CHECK(r >= 0 && r < ctx->nranks && !seen[r], DP_ERR_INVALID, "slot ranks must be distinct non-primary ranks");
      seen[r] = 1;
    }
    ctx->slot_map_primary = primary;
    for (int s = 0; s < DP_MAX_DEVICES; ++s) ctx->slot_rank[s] = (s >= 1 && s < k) ? rank_of_slot[s - 1] : -1;
  });
}

extern "C" dp_status dp_peer_init(dp_context* ctx, const void* uid128, int32_t rank, int32_t nranks) {
  return guard([&] {
    DP_CHECK(ctx && uid128, DP_ERR_INVALID, "NULL argument");
    DP_CHECK(nranks >= 1 && rank >= 0 && rank < nranks, DP_ERR_INVALID, "bad rank/nranks");
    DP_CHECK(ctx->devs.size() == 1, DP_ERR_INVALID, "multi-process PT needs a one-device context per process");
    DP_CHECK(!ctx->comm, DP_ERR_STATE, "peer transport already initialised");
    DP_CUDA(cudaSetDevice(ctx->devs[0]));
    ncclUniqueId id;
    std::memcpy(&id, uid128, sizeof(id));
    ncclComm_t comm;
    DP_NCCL(nccl().commInitRank(&comm, nranks, id, rank));
    ctx->comm = comm;
    ctx->rank = rank;
    ctx->nranks = nranks;
    DP_CUDA(cudaStreamCreateWithFlags(&ctx->comm_stream, cudaStreamNonBlocking));
  });
}
