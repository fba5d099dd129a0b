// Context, cold-start / warm inference, eviction and the per-layer profiler.
//
// Cold start = §4.3.4 + Fig.9:
//   * slot-0 LOAD units: H2D over the primary's own PCIe link on the load stream(s), one
//     completion event per coalesced chunk;
//   * slot-s LOAD units (PT): H2D over the link of the slot's GPU into a staging
//     ring, then forwarded into the primary's HBM slot by that GPU's migration stream
//     (cudaMemcpyPeerAsync over NVLink; a D2D copy in loopback; NCCL send/recv across
//     processes -- peer.cpp), one event per forwarded piece; or, with opts.pt_transport =
//     DP_PT_SM / DP_PT_CE (pt_forward.cu), in ONE hop by a forwarder kernel or a
//     DMA on the secondary straight into the primary's slot (across processes over CUDA IPC,
//     with release/acquire mailbox words instead of events);
//   * DHA units: no transfer; their kernels read the arena in place ("we can skip
//     the dependency check");
//   * the execution stream (the caller's) waits on a unit's piece right before the first
//     kernel that reads it, batched per round of links (the pieces of the next units on the
//     other links that land no later are waited for in the same batch).
#include <algorithm>
#include <chrono>
#include <cstdlib>
#include <cstring>
#include <numeric>
#include <vector>

#include <cuda.h>

#include "engine.h"
#include "kernels.h"
#include "launch.cuh"
#include "peer.h"

namespace dp {

static thread_local std::string g_last_error;
void set_last_error(const std::string& msg) { g_last_error = msg; }

struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int d) {
    cudaGetDevice(&prev);
    DP_CUDA(cudaSetDevice(d));
  }
  ~DeviceGuard() {
    if (prev >= 0) cudaSetDevice(prev);
  }
};

}  // namespace dp

using namespace dp;

dp::DevCtx& dp_context::on(int dev) {
  DP_CHECK(dev >= 0 && dev < DP_MAX_DEVICES, DP_ERR_INVALID, "device ordinal out of range");
  DevCtx& d = dc[dev];
  DP_CHECK(d.ready, DP_ERR_INVALID, "device " + std::to_string(dev) + " is not part of this context");
  return d;
}

static void init_device(dp_context* ctx, int dev) {
  DevCtx& d = ctx->dc[dev];
  if (d.ready) return;
  DeviceGuard g(dev);
  d.ord = dev;
  d.events.dev = dev;
  d.ready = true;
}

static void ensure_h2d_streams(dp_context* ctx, int dev) {
  DevCtx& d = ctx->on(dev);
  const int want = std::max(1, ctx->opts.n_h2d_streams);
  if ((int)d.h2d.size() >= want) return;
  DeviceGuard g(dev);
  while ((int)d.h2d.size() < want) {
    cudaStream_t s;
    DP_CUDA(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
    d.h2d.push_back(s);
  }
}

constexpr int64_t kRingSlots = 3;  // staging ring depth of a two-hop PT slot

static SlotRes& slot_res(dp_context* ctx, int slot, int dev, int64_t ring_bytes) {
  auto& r = ctx->slots[{slot, dev}];
  DeviceGuard g(dev);
  if (!r.h2d) {
    r.dev = dev;
    DP_CUDA(cudaStreamCreateWithFlags(&r.h2d, cudaStreamNonBlocking));
    DP_CUDA(cudaStreamCreateWithFlags(&r.mig, cudaStreamNonBlocking));
  }
  if (r.ring_bytes < ring_bytes) {
    // a captured graph may reference the old ring: synchronise before freeing it, and make
    // every graph key that named it unreachable (stale-pointer replay)
    ++ctx->ring_gen;
    if (r.ring) {
      DP_CUDA(cudaDeviceSynchronize());
      DP_CUDA(cudaFree(r.ring));
    }
    r.ring = nullptr;
    if (cudaMalloc(&r.ring, ring_bytes) != cudaSuccess) fail(DP_ERR_OOM, "staging ring cudaMalloc failed");
    r.ring_bytes = ring_bytes;
  }
  return r;
}

// ---------------------------------------------------------------------------------------
// HBM slots: a per-device pool of blocks; a model holds one block while resident, laid out
// like the arena minus the DHA units' ranges (DHA layers occupy no GPU memory).
// ---------------------------------------------------------------------------------------

namespace dp {

constexpr int64_t kPoolGrain = 2 << 20;  // block sizes are rounded to 2 MiB (easier reuse)

// Free every unused block of the pool (back to the driver); returns the bytes released.
static int64_t pool_trim(HbmPool& p, int dev) {
  DeviceGuard g(dev);
  int64_t freed = 0;
  for (auto& kv : p.free_) {
    DP_CUDA(cudaFree(kv.second));
    p.size_.erase(kv.second);
    freed += kv.first;
  }
  p.free_.clear();
  p.reserved -= freed;
  return freed;
}

// A block of >= bytes: the first of `prefer` that is free and fits (a model re-acquiring a block
// it has captured graphs on keeps them valid: no re-capture), else the best fit among the free
// blocks not more than 2x too large, else a new cudaMalloc (trimming the free blocks and retrying
// once if HBM is exhausted).
static void* pool_alloc(HbmPool& p, int dev, int64_t bytes, const std::vector<void*>& prefer) {
  bytes = (bytes + kPoolGrain - 1) / kPoolGrain * kPoolGrain;
  auto take = [&](std::multimap<int64_t, void*>::iterator it) {
    void* b = it->second;
    p.in_use += it->first;
    p.free_.erase(it);
    return b;
  };
  for (void* want : prefer) {
    if (!want) continue;
    for (auto it = p.free_.begin(); it != p.free_.end(); ++it)
      if (it->second == want && it->first >= bytes && it->first <= 2 * bytes) return take(it);
  }
  auto it = p.free_.lower_bound(bytes);
  if (it != p.free_.end() && it->first <= 2 * bytes) return take(it);
  DeviceGuard g(dev);
  void* b = nullptr;
  if (cudaMalloc(&b, bytes) != cudaSuccess) {
    cudaGetLastError();
    pool_trim(p, dev);
    if (cudaMalloc(&b, bytes) != cudaSuccess) {
      cudaGetLastError();
      fail(DP_ERR_OOM, "HBM slot allocation for the model failed");
    }
  }
  p.size_[b] = bytes;
  p.reserved += bytes;
  p.in_use += bytes;
  return b;
}

static void pool_free(HbmPool& p, void* b) {
  auto it = p.size_.find(b);
  DP_CHECK(it != p.size_.end(), DP_ERR_STATE, "internal: block not owned by this pool");
  p.in_use -= it->second;
  p.free_.emplace(it->second, b);
}

// Compact layout: loaded units keep the arena's relative offsets; each DHA unit's arena span
// (its bytes plus alignment padding up to the next unit) is left out.  Units between which no DHA
// unit lies stay contiguous, so every DMA piece (consecutive loaded units) is one contiguous
// destination range.
static int64_t compact_layout(const dp_model* m, const int8_t* method, std::vector<int64_t>& doff) {
  const int n = (int)m->units.size();
  doff.assign(n, -1);
  int64_t removed = 0;
  for (int u = 0; u < n; ++u) {
    const int64_t end = u + 1 < n ? m->units[u + 1].off : m->arena_bytes;
    if (method && method[u] == DP_DHA) {
      removed += end - m->units[u].off;
      continue;
    }
    doff[u] = m->units[u].off - removed;
  }
  return m->arena_bytes - removed;
}

// HBM bytes a cold start under `method` holds while resident (the compact layout's size).
int64_t plan_resident_bytes(const dp_model* m, const int8_t* method) {
  std::vector<int64_t> doff;
  return compact_layout(m, method, doff);
}

void acquire_slots(dp_context* ctx, dp_model* m, int dev, const int8_t* method) {
  DevState& ds = m->dev[dev];
  if (ds.pinned_full) {  // IPC-exported: the peers write into the full arena layout
    compact_layout(m, nullptr, ds.doff);
    return;
  }
  DP_CHECK(!ds.dbase, DP_ERR_STATE, "internal: HBM slots already held");
  std::vector<int64_t> doff;
  const int64_t bytes = std::max<int64_t>(compact_layout(m, method, doff), 256);
  std::vector<void*> prefer{ds.last_block};
  prefer.insert(prefer.end(), ds.graph_blocks.begin(), ds.graph_blocks.end());
  ds.dbase = pool_alloc(ctx->on(dev).pool, dev, bytes, prefer);
  ds.dbytes = bytes;
  ds.doff.swap(doff);
}

void release_slots(dp_context* ctx, dp_model* m, int dev) {
  DevState& ds = m->dev[dev];
  if (ds.pinned_full || !ds.dbase) return;
  pool_free(ctx->on(dev).pool, ds.dbase);
  ds.last_block = ds.dbase;
  ds.dbase = nullptr;
  ds.dbytes = 0;
}

void pin_full_slots(dp_model* m, int dev) {
  DevState& ds = m->dev[dev];
  if (ds.pinned_full) return;
  DP_CHECK(!ds.resident && !ds.dbase, DP_ERR_STATE, "export the model's slots before its first cold start");
  DeviceGuard g(dev);
  if (cudaMalloc(&ds.dbase, m->arena_bytes) != cudaSuccess) {
    ds.dbase = nullptr;
    fail(DP_ERR_OOM, "HBM slot allocation for the model failed");
  }
  ds.dbytes = m->arena_bytes;
  ds.pinned_full = true;
  compact_layout(m, nullptr, ds.doff);
}

}  // namespace dp

// Single-process SM forwarding to another GPU stores through the peer mapping.
static void ensure_peer_access(int from, int to) {
  static bool done[DP_MAX_DEVICES][DP_MAX_DEVICES] = {};
  if (from == to || done[from][to]) return;
  int ok = 0;
  DP_CUDA(cudaDeviceCanAccessPeer(&ok, from, to));
  DP_CHECK(ok, DP_ERR_UNSUPPORTED, "SM PT forwarder: device " + std::to_string(from) + " cannot access device " +
                                       std::to_string(to) + "'s memory");
  DeviceGuard g(from);
  cudaError_t e = cudaDeviceEnablePeerAccess(to, 0);
  if (e == cudaErrorPeerAccessAlreadyEnabled) {
    cudaGetLastError();
  } else {
    DP_CUDA(e);
  }
  done[from][to] = true;
}

extern "C" const char* dp_last_error(void) { return g_last_error.c_str(); }
extern "C" int32_t dp_abi_version(void) { return 2; }  // 2: round-2 structs (serve result, opts)

extern "C" dp_status dp_context_create(const int32_t* devs, int32_t ndev, dp_context** out) {
  dp_context* ctx = nullptr;
  dp_status st = guard([&] {
    DP_CHECK(out && devs && ndev >= 1 && ndev <= DP_MAX_DEVICES, DP_ERR_INVALID, "bad device list");
    int count = 0;
    DP_CUDA(cudaGetDeviceCount(&count));
    ctx = new dp_context();
    ctx->opts.chunk_bytes = 4 << 20;
    ctx->opts.n_h2d_streams = 1;
    ctx->opts.use_graph = 0;
    ctx->opts.gemm_bn = 0;
    ctx->opts.use_pdl = 1;
    ctx->opts.tail_bytes = 2 << 20;
    ctx->opts.chunk_bytes = 32 << 20;
    ctx->opts.profile_chain = 1;
    for (int i = 0; i < ndev; ++i) {
      DP_CHECK(devs[i] >= 0 && devs[i] < count && devs[i] < DP_MAX_DEVICES, DP_ERR_INVALID,
               "device " + std::to_string(devs[i]) + " does not exist");
      ctx->devs.push_back(devs[i]);
      init_device(ctx, devs[i]);
    }
    *out = ctx;
  });
  if (st != DP_OK) delete ctx;
  return st;
}

extern "C" dp_status dp_context_destroy(dp_context* ctx) {
  return guard([&] {
    if (!ctx) return;
    for (int d : ctx->devs) {
      DeviceGuard g(d);
      cudaDeviceSynchronize();
      DevCtx& dc = ctx->dc[d];
      for (auto& kv : dc.pool.size_) cudaFree(kv.first);  // models must be destroyed first
      dc.pool = HbmPool();
      for (auto s : dc.h2d) cudaStreamDestroy(s);
      dc.events.destroy();
      if (dc.flush) cudaFree(dc.flush);
    }
    for (auto& kv : ctx->slots) {
      DeviceGuard g(kv.second.dev);
      if (kv.second.h2d) cudaStreamDestroy(kv.second.h2d);
      if (kv.second.mig) cudaStreamDestroy(kv.second.mig);
      if (kv.second.ring) cudaFree(kv.second.ring);
      if (kv.second.tail) cudaEventDestroy(kv.second.tail);
    }
    if (!ctx->devs.empty()) {
      DeviceGuard g(ctx->devs[0]);
      ipc_close(ctx);
    }
    peer_destroy(ctx);
    delete ctx;
  });
}

extern "C" dp_status dp_context_set_opts(dp_context* ctx, const dp_engine_opts* o) {
  return guard([&] {
    DP_CHECK(ctx && o, DP_ERR_INVALID, "NULL argument");
    DP_CHECK(o->chunk_bytes >= 4096, DP_ERR_INVALID, "chunk_bytes must be >= 4096");
    DP_CHECK(o->n_h2d_streams >= 1 && o->n_h2d_streams <= 8, DP_ERR_INVALID, "n_h2d_streams must be 1..8");
    DP_CHECK(o->gemm_bn == 0 || o->gemm_bn == 32 || o->gemm_bn == 64 || o->gemm_bn == 96 || o->gemm_bn == 128 ||
                 o->gemm_bn == 256 || o->gemm_bn == -64 || o->gemm_bn == -128 || o->gemm_bn == -192 ||
                 o->gemm_bn == -256,
             DP_ERR_INVALID, "gemm_bn must be 0/32/64/96/128/256 (one CTA) or -64/-128/-192/-256 (a CTA pair)");
    DP_CHECK(o->pt_transport == DP_PT_DMA || o->pt_transport == DP_PT_SM || o->pt_transport == DP_PT_CE,
             DP_ERR_INVALID, "pt_transport must be DP_PT_DMA, DP_PT_SM or DP_PT_CE");
    // measured slower and moved out of the library (tools/experiments)
    DP_CHECK(o->attention_tc >= 0 && o->attention_tc <= 2, DP_ERR_INVALID, "attention_tc must be 0, 1 or 2");
    DP_CHECK(!o->fuse_ln && !o->persistent, DP_ERR_UNSUPPORTED,
             "fuse_ln / persistent: experiments kept in tools/experiments, not built into the library");
    ctx->opts = *o;
  });
}

extern "C" dp_status dp_context_get_opts(dp_context* ctx, dp_engine_opts* out) {
  return guard([&] {
    DP_CHECK(ctx && out, DP_ERR_INVALID, "NULL argument");
    *out = ctx->opts;
  });
}

// ---------------------------------------------------------------------------------------
// Cold start
// ---------------------------------------------------------------------------------------

namespace dp {

// Coalesce runs of units (forward order) selected by `pick` that are contiguous in the
// arena into pieces of at most `cap` bytes.  A unit is never split: one bigger than cap
// is a piece of its own (one DMA per unit is cheapest; its event covers the whole unit).
template <class Pick>
std::vector<Piece> make_pieces(const dp_model* m, Pick pick, int64_t cap) {
  std::vector<Piece> out;
  const int n = (int)m->units.size();
  Piece cur;
  auto flush = [&] {
    if (cur.bytes > 0) out.push_back(cur);
    cur = Piece();
  };
  for (int u = 0; u < n; ++u) {
    if (!pick(u)) {
      flush();
      continue;
    }
    const auto& un = m->units[u];
    if (un.bytes == 0) continue;
    if (cur.bytes > 0 && (cur.off + cur.bytes != un.off || cur.bytes + un.bytes > cap)) flush();
    if (cur.bytes == 0) {
      cur.off = un.off;
      cur.first_unit = u;
    }
    cur.bytes += un.bytes;
    cur.last_unit = u;
  }
  flush();
  return out;
}

std::vector<Piece> slot_pieces(const dp_model* m, const dp_plan* plan, int slot, int64_t cap, int64_t tail) {
  auto p = make_pieces(m, [&](int u) { return plan->method[u] == DP_LOAD && plan->slot[u] == slot; }, cap);
  // Cold-start latency = (last byte lands) + (compute of what it carried): the link never
  // waits for compute, so only the LAST piece's size matters for the pipeline tail.  Peel
  // trailing units off the last piece until it holds <= `tail` bytes (or one unit).
  if (tail > 0 && !p.empty() && p.back().bytes > tail) {
    Piece& b = p.back();
    int64_t acc = 0;
    int first = b.last_unit + 1;
    for (int u = b.last_unit; u > b.first_unit; --u) {  // longest suffix <= tail, b keeps >= 1 unit
      if (acc + m->units[u].bytes > tail) break;
      acc += m->units[u].bytes;
      first = u;
    }
    if (first <= b.last_unit) {
      Piece q;
      q.first_unit = first;
      q.last_unit = b.last_unit;
      q.off = m->units[first].off;
      q.bytes = b.off + b.bytes - q.off;
      b.bytes = q.off - b.off;
      b.last_unit = first - 1;
      p.push_back(q);
    }
  }
  return p;
}

}  // namespace dp

extern "C" dp_status dp_transfer_schedule(const dp_model_config* cfg, const dp_plan* plan, int32_t slot,
                                          int64_t chunk_bytes, int64_t tail_bytes, int64_t* piece_off,
                                          int64_t* piece_bytes,
                                          int32_t* first_unit, int32_t* last_unit, int32_t cap, int32_t* count) {
  return dp::guard([&] {
    DP_CHECK(cfg && plan && count, DP_ERR_INVALID, "NULL argument");
    dp_model tmp;
    tmp.cfg = *cfg;
    tmp.params = dp::config_params(*cfg);
    dp::build_units(&tmp);
    DP_CHECK(plan->n == (int)tmp.units.size() && plan->method && plan->slot, DP_ERR_INVALID, "plan/model mismatch");
    DP_CHECK(slot >= 0 && slot < plan->k, DP_ERR_INVALID, "slot out of range");
    auto pcs = dp::slot_pieces(&tmp, plan, slot, std::max<int64_t>(chunk_bytes, 4096), tail_bytes);
    *count = (int32_t)pcs.size();
    for (int i = 0; i < (int)pcs.size() && i < cap; ++i) {
      if (piece_off) piece_off[i] = pcs[i].off;
      if (piece_bytes) piece_bytes[i] = pcs[i].bytes;
      if (first_unit) first_unit[i] = pcs[i].first_unit;
      if (last_unit) last_unit[i] = pcs[i].last_unit;
    }
  });
}

namespace dp {

void bind_units(std::vector<cudaEvent_t>& unit_ev, const Piece& p, cudaEvent_t e) {
  for (int u = p.first_unit; u <= p.last_unit; ++u) unit_ev[u] = e;
}

static void validate_plan(const dp_model* m, const dp_plan* p) {
  DP_CHECK(p && p->method && p->slot, DP_ERR_INVALID, "plan is NULL");
  DP_CHECK(p->n == (int)m->units.size(), DP_ERR_INVALID, "plan.n does not match the model's unit count");
  DP_CHECK(p->k >= 1 && p->k <= DP_MAX_DEVICES, DP_ERR_INVALID, "plan.k out of range");
  for (int i = 0; i < p->n; ++i) {
    DP_CHECK(p->method[i] == DP_LOAD || p->method[i] == DP_DHA, DP_ERR_INVALID, "bad method value");
    DP_CHECK(p->slot[i] >= 0 && p->slot[i] < p->k, DP_ERR_INVALID, "slot out of range");
    DP_CHECK(!(p->slot[i] > 0 && p->method[i] == DP_DHA), DP_ERR_INVALID, "a PT unit (slot > 0) must be LOAD");
  }
}

// Host-link bytes a unit's DHA kernels must read (algorithmic; Table 1's closed forms).
static int64_t unit_dha_bytes(const dp_model* m, int u, int T, int seq) {
  const int64_t row = int64_t(m->cfg.hidden) * dtype_bytes(m->cfg.dtype);
  switch (m->units[u].role) {
    case R_WORD: case R_WTE: return int64_t(T) * row;  // one row per token
    case R_POS: case R_WPE: return int64_t(std::min<int64_t>(seq, m->cfg.max_pos)) * row;
    case R_TYPE: return row;
    default: return m->units[u].bytes;  // LN gamma/beta, linear weights: every byte once
  }
}

static int64_t dha_bytes(const dp_model* m, const int8_t* method, int T, int seq) {
  int64_t s = 0;
  for (size_t u = 0; u < m->units.size(); ++u)
    if (method[u] == DP_DHA) s += unit_dha_bytes(m, (int)u, T, seq);
  return s;
}

// `primary` is the serving device ordinal; `prim_rank` its rank when the PT gather runs over
// NCCL between processes (then secondaries are ranks, see peer.cpp).
static dp_run_stats enqueue_cold(dp_context* ctx, dp_model* m, const dp_plan* plan, int primary, int prim_rank,
                                 const int32_t* secondaries, const int32_t* ids, int batch, int seq, void* out,
                                 void* pooled, cudaStream_t stream);

// Key of a captured cold-start / warm graph: everything the enqueued work depends on.
static std::string graph_key(const dp_context* ctx, const DevState& ds, const dp_plan* plan,
                             const int32_t* secondaries, const void* ids, int batch, int seq, const void* out,
                             const void* pooled) {
  // every device buffer the captured work touches: the HBM slots, the workspace, the staging
  // rings (by generation) -- a graph is never replayed on memory that was reallocated
  std::string k = std::to_string((uintptr_t)ds.dbase) + "/" + std::to_string((uintptr_t)ds.ws.base) + "/" +
                  std::to_string(ds.ws.tokens) + "/" + std::to_string(ctx->ring_gen) + "|";
  if (plan) {
    k.append(reinterpret_cast<const char*>(plan->method), plan->n);
    k.append(reinterpret_cast<const char*>(plan->slot), plan->n);
    k += "|" + std::to_string(plan->k);
    for (int s = 1; s < plan->k; ++s) k += "," + (secondaries ? std::to_string(secondaries[s - 1]) : "r");
  }
  k += "|" + std::to_string((uintptr_t)ids) + "|" + std::to_string((uintptr_t)out) + "|" +
       std::to_string((uintptr_t)pooled) + "|" + std::to_string(batch) + "x" + std::to_string(seq) + "|" +
       std::to_string(ctx->opts.chunk_bytes) + "," + std::to_string(ctx->opts.n_h2d_streams) + "," +
       std::to_string(ctx->opts.gemm_bn) + "," + std::to_string(ctx->opts.debug_delay_us) + "," +
       std::to_string(ctx->opts.use_pdl) + "," + std::to_string(ctx->opts.attention_tc) + "," +
       std::to_string(ctx->opts.pt_transport);
  return k;
}

// Capture `body` (which enqueues on `stream` and joins every side stream back into it) into
// a CUDA graph once per key; afterwards replay it.  Replay removes the host enqueue cost and
// turns the per-piece events into graph edges.
// Capture happens on a private stream (the caller's may be the legacy stream, which cannot
// be captured); the executable graph is then launched on the caller's stream.
// A key seen for the first time runs eagerly; the graph is captured on its second use.  A
// capture + instantiate costs a few ms, so keys that never repeat (a serving instance on a pool
// block it never gets again) must not pay it; keys that repeat (a bench loop, a resident
// instance's warm runs) are replayed from the second time on.
template <class Body>
static dp_run_stats run_graph(DevState& ds, const std::string& key, cudaStream_t stream, Body body) {
  auto it = ds.graphs.find(key);
  if (it == ds.graphs.end() && ds.graph_seen[key]++ == 0) return body(stream);
  if (it == ds.graphs.end()) {
    if (!ds.capture) DP_CUDA(cudaStreamCreateWithFlags(&ds.capture, cudaStreamNonBlocking));
    cudaStream_t cs = ds.capture;
    cudaGraph_t gph = nullptr;
    DP_CUDA(cudaStreamBeginCapture(cs, cudaStreamCaptureModeRelaxed));
    dp_run_stats st;
    try {
      st = body(cs);
    } catch (...) {
      cudaStreamEndCapture(cs, &gph);
      if (gph) cudaGraphDestroy(gph);
      throw;
    }
    DP_CUDA(cudaStreamEndCapture(cs, &gph));
    cudaGraphExec_t ex = nullptr;
    cudaError_t e = cudaGraphInstantiate(&ex, gph, 0);
    cudaGraphDestroy(gph);
    DP_CUDA(e);
    it = ds.graphs.emplace(key, GraphEntry{ex, st}).first;
    if (ds.dbase && std::find(ds.graph_blocks.begin(), ds.graph_blocks.end(), ds.dbase) == ds.graph_blocks.end())
      ds.graph_blocks.push_back(ds.dbase);
  }
  DP_CUDA(cudaGraphLaunch(it->second.exec, stream));
  return it->second.stats;
}

void infer_cold(dp_context* ctx, dp_model* m, const dp_plan* plan, int primary, int prim_rank,
                const int32_t* secondaries, int nsec, const int32_t* ids, int batch, int seq, void* out, void* pooled,
                cudaStream_t stream, dp_run_stats* stats) {
  NvtxRange nv("dp_infer_cold");
  auto t0 = std::chrono::steady_clock::now();
  validate_plan(m, plan);
  ctx->on(primary);
  DevState& ds = m->dev[primary];
  DP_CHECK(!ds.resident, DP_ERR_STATE, "model already resident on the primary; evict it first");
  DP_CHECK(ctx->multiproc() || nsec >= plan->k - 1, DP_ERR_INVALID, "need k-1 secondaries for the plan");
  DP_CHECK(batch > 0 && seq > 0 && ids && out, DP_ERR_INVALID, "bad inference arguments");
  DP_CHECK(seq + (m->cfg.family == DP_FAMILY_ROBERTA ? m->cfg.pad_idx + 1 : 0) <= m->cfg.max_pos, DP_ERR_INVALID,
           "sequence longer than the position table");
  DeviceGuard g(primary);
  acquire_slots(ctx, m, primary, plan->method);
  // a failure before the model became resident hands the block back (the model stays usable)
  struct ReleaseOnError {
    dp_context* c;
    dp_model* mm;
    int d;
    bool armed = true;
    ~ReleaseOnError() {
      if (!armed) return;
      try {
        cudaDeviceSynchronize();  // transfers already enqueued into the block must finish first
        release_slots(c, mm, d);
      } catch (...) {
      }
    }
  } release_on_error{ctx, m, primary};
  ensure_h2d_streams(ctx, primary);
  ensure_workspace(m, primary, int64_t(batch) * seq);
  // across processes: the IPC transports capture (the epoch lives in a device word); the NCCL
  // gather does not
  const bool ipc_pt = ctx->multiproc() && ctx->opts.pt_transport != DP_PT_DMA && plan->k > 1;
  bool graph = ctx->opts.use_graph != 0 && !ctx->opts.trace_units && (!ctx->multiproc() || ipc_pt || plan->k == 1);
  for (int s = 1; s < plan->k && graph && !ctx->multiproc(); ++s)
    graph = secondaries[s - 1] == primary;  // single-device graphs only
  // staging rings of the two-hop PT slots are sized before any capture (their pointers are
  // part of the graph key)
  if (!ctx->multiproc() && ctx->opts.pt_transport == DP_PT_DMA) {
    const int64_t cap = std::max<int64_t>(ctx->opts.chunk_bytes, 4096);
    for (int s = 1; s < plan->k; ++s) {
      auto pcs = slot_pieces(m, plan, s, cap, opt_tail(ctx));
      int64_t slot_bytes = 0;
      for (const auto& p : pcs) slot_bytes = std::max(slot_bytes, p.bytes);
      const int sdev = secondaries[s - 1];
      DP_CHECK(sdev >= 0 && sdev < DP_MAX_DEVICES && ctx->dc[sdev].ready, DP_ERR_INVALID,
               "secondary device not in the context");
      if (slot_bytes > 0) slot_res(ctx, s, sdev, kRingSlots * slot_bytes);
    }
  }
  if (ipc_pt) {
    ipc_check_primary(ctx);
    ipc_set_epoch(ctx, ++ctx->pt_epoch, stream);  // every rank counts the same k > 1 cold starts
  }
  dp_run_stats st;
  if (graph) {
    st = run_graph(ds, graph_key(ctx, ds, plan, secondaries, ids, batch, seq, out, pooled), stream, [&](cudaStream_t cs) {
      return enqueue_cold(ctx, m, plan, primary, prim_rank, secondaries, ids, batch, seq, out, pooled, cs);
    });
  } else {
    st = enqueue_cold(ctx, m, plan, primary, prim_rank, secondaries, ids, batch, seq, out, pooled, stream);
  }
  ds.resident = true;
  release_on_error.armed = false;
  ds.method.assign(plan->method, plan->method + plan->n);
  st.wall_enqueue_us =
      std::chrono::duration<float, std::micro>(std::chrono::steady_clock::now() - t0).count();
  if (stats) *stats = st;
}

static dp_run_stats enqueue_cold(dp_context* ctx, dp_model* m, const dp_plan* plan, int primary, int prim_rank,
                                 const int32_t* secondaries, const int32_t* ids, int batch, int seq, void* out,
                                 void* pooled, cudaStream_t stream) {
  DevCtx& pd = ctx->on(primary);
  DevState& ds = m->dev[primary];
  pd.events.reset();
  const int n = (int)m->units.size();
  const int8_t* method = plan->method;
  dp_run_stats st;
  std::memset(&st, 0, sizeof(st));
  st.n_units = n;
  std::vector<cudaEvent_t> unit_ev(n, nullptr);
  // Wait points, per link (slot): every piece in the order its link delivers it, with the bytes
  // its link has carried through its end (the landing-time proxy) and its completion (an event,
  // or across processes a done word).  Pieces of one link complete in order, so waiting on
  // piece r covers every earlier piece of that link.
  struct WaitPt {
    int64_t proxy = 0;
    cudaEvent_t ev = nullptr;
  };
  std::vector<std::vector<WaitPt>> wp(std::max(1, plan->k));
  std::vector<std::pair<int, int>> unit_wp(n, {-1, -1});  // (slot, piece) of a loaded unit
  bool fifo0 = true;                                       // slot 0 on one load stream
  auto add_wp = [&](int slot, const Piece& p, cudaEvent_t e) {
    const int64_t prev = wp[slot].empty() ? 0 : wp[slot].back().proxy;
    wp[slot].push_back({prev + p.bytes, e});
    for (int u = p.first_unit; u <= p.last_unit; ++u) unit_wp[u] = {slot, (int)wp[slot].size() - 1};
  };

  // fork: side streams start when the execution stream reaches this call
  cudaEvent_t fork = pd.events.get();
  DP_CUDA(cudaEventRecord(fork, stream));
  ++st.n_events;
  // opts.trace_units: timing events for dp_run_timeline (eager only: graphs are off)
  const bool trace = ctx->opts.trace_units != 0;
  UnitTrace& tr = ds.trace;
  auto stamp = [&](cudaStream_t on) {  // a globaltimer slot written when `on` reaches this point
    DP_CHECK(tr.used < tr.cap, DP_ERR_STATE, "internal: trace buffer full");
    launch_timestamp(tr.dbuf + tr.used, on);
    return tr.used++;
  };
  if (trace) {
    const int cap = 3 * n + 2 * 1024 + 8;
    if (tr.cap < cap) {
      if (tr.dbuf) DP_CUDA(cudaFree(tr.dbuf));
      tr.dbuf = nullptr;
      DP_CUDA(cudaMalloc(&tr.dbuf, sizeof(uint64_t) * cap));
      tr.cap = cap;
    }
    DP_CUDA(cudaMemsetAsync(tr.dbuf, 0, sizeof(uint64_t) * tr.cap, stream));
    tr.valid = false;
    tr.used = 0;
    tr.ready.assign(n, -1);
    tr.pre.assign(n, -1);
    tr.start.assign(n, -1);
    tr.t0 = stamp(stream);
    tr.last_stream = stream;
  }
  auto trace_piece = [&](const Piece& p, cudaStream_t on) {  // the piece's bytes have landed
    if (!trace) return;
    const int sl = stamp(on);
    for (int u = p.first_unit; u <= p.last_unit; ++u) tr.ready[u] = sl;
  };

  // (1) slot-0 loads on the primary's link
  NvtxRange nv_load("enqueue slot-0 loads");
  const int64_t cap = std::max<int64_t>(ctx->opts.chunk_bytes, 4096);
  auto pieces0 = slot_pieces(m, plan, 0, cap, opt_tail(ctx));
  const int nh = std::min((int)pd.h2d.size(), std::max(1, ctx->opts.n_h2d_streams));
  fifo0 = nh == 1;
  for (int i = 0; i < nh; ++i) DP_CUDA(cudaStreamWaitEvent(pd.h2d[i], fork, 0));
  for (size_t c = 0; c < pieces0.size(); ++c) {
    const Piece& p = pieces0[c];
    cudaStream_t hs = pd.h2d[c % nh];
    if (ctx->opts.debug_delay_us > 0) launch_spin((long long)ctx->opts.debug_delay_us * 2000, hs);
    DP_CUDA(cudaMemcpyAsync(m->device(primary, p.first_unit), static_cast<const uint8_t*>(m->arena) + p.off, p.bytes,
                            cudaMemcpyHostToDevice, hs));
    ++st.n_copies;
    st.h2d_bytes[0] += p.bytes;
    cudaEvent_t e = pd.events.get();
    DP_CUDA(cudaEventRecord(e, hs));
    ++st.n_events;
    bind_units(unit_ev, p, e);  // every unit inside this piece completes with it
    add_wp(0, p, e);
    trace_piece(p, hs);
  }

  // (2) PT slots
  const bool one_hop = ctx->opts.pt_transport != DP_PT_DMA;  // single hop: SM forwarder or direct DMA
  const bool ce_fwd = ctx->opts.pt_transport == DP_PT_CE;
  // across processes with the SM forwarder: (slot, piece) a loaded unit arrives in
  std::vector<size_t> slot_npieces(plan->k, 0);
  if (!ctx->multiproc())
    for (int s = 1; s < plan->k; ++s) {
      const int sdev = secondaries[s - 1];
      DP_CHECK(sdev >= 0 && sdev < DP_MAX_DEVICES && ctx->dc[sdev].ready, DP_ERR_INVALID,
               "secondary device not in the context");
      if (sdev != primary) ctx->dc[sdev].events.reset();
    }
  if (ctx->multiproc() && plan->k > 1 && !one_hop) {
    DP_CHECK(ctx->comm, DP_ERR_STATE, "DMA transport across processes needs dp_peer_init (NCCL)");
    peer_recv_all(ctx, m, plan, prim_rank, primary, fork, unit_ev, st);
  }
  if (ctx->multiproc() && one_hop && plan->k > 1) {
    // go to every secondary; their forwarders store into our slots and release done words
    ipc_check_primary(ctx);  // the epoch word was set by infer_cold
    ipc_primary_begin(ctx, plan, prim_rank, stream);
    for (int s = 1; s < plan->k; ++s) {
      auto pcs = slot_pieces(m, plan, s, cap, opt_tail(ctx));
      slot_npieces[s] = pcs.size();
      for (size_t r = 0; r < pcs.size(); ++r) {
        add_wp(s, pcs[r], nullptr);
        st.nvlink_bytes[s] += pcs[r].bytes;
      }
    }
  }
  for (int s = 1; s < plan->k && !ctx->multiproc(); ++s) {
    auto pcs = slot_pieces(m, plan, s, cap, opt_tail(ctx));
    if (pcs.empty()) continue;
    const int sdev = secondaries[s - 1];
    const int64_t ring_slots = kRingSlots;
    int64_t slot_bytes = 0;
    for (const auto& p : pcs) slot_bytes = std::max(slot_bytes, p.bytes);
    SlotRes& r = slot_res(ctx, s, sdev, one_hop ? 0 : ring_slots * slot_bytes);
    DevCtx& sd = ctx->dc[sdev];
    {
      DeviceGuard gs(sdev);
      DP_CUDA(cudaStreamWaitEvent(r.h2d, fork, 0));
    }
    if (one_hop) {  // one hop per piece on the secondary, host -> primary HBM
      if (!ce_fwd) ensure_peer_access(sdev, primary);
      DeviceGuard gs(sdev);
      for (const Piece& p : pcs) {
        if (ctx->opts.debug_delay_us > 0) launch_spin((long long)ctx->opts.debug_delay_us * 2000, r.h2d);
        if (ce_fwd) {
          DP_CUDA(cudaMemcpyAsync(m->device(primary, p.first_unit), static_cast<const uint8_t*>(m->arena) + p.off,
                                  p.bytes, cudaMemcpyDefault, r.h2d));
          ++st.n_copies;
        } else {
          launch_pt_forward(static_cast<const uint8_t*>(m->arena) + p.off, m->device(primary, p.first_unit), p.bytes,
                            r.h2d, nullptr, 0, nullptr, nullptr);
        }
        st.h2d_bytes[s] += p.bytes;
        st.nvlink_bytes[s] += p.bytes;
        cudaEvent_t done = sd.events.get();
        DP_CUDA(cudaEventRecord(done, r.h2d));
        ++st.n_events;
        bind_units(unit_ev, p, done);
        add_wp(s, p, done);
        if (sdev == primary) trace_piece(p, r.h2d);  // timing events only within one device
      }
      // the end-of-cold-start join waits on the migration stream: chain it behind the loads
      cudaEvent_t last = sd.events.get();
      DP_CUDA(cudaEventRecord(last, r.h2d));
      DP_CUDA(cudaStreamWaitEvent(r.mig, last, 0));
      continue;
    }
    std::vector<cudaEvent_t> fwd_done(pcs.size(), nullptr);
    // eager enqueue only: a captured graph's branches are ordered by the graph launches on the
    // caller's stream, and a capture may not wait on work recorded outside it
    cudaStreamCaptureStatus cap = cudaStreamCaptureStatusNone;
    DP_CUDA(cudaStreamIsCapturing(stream, &cap));
    const bool eager = cap == cudaStreamCaptureStatusNone;
    if (eager) {
      DeviceGuard gs(sdev);
      if (!r.tail) DP_CUDA(cudaEventCreateWithFlags(&r.tail, cudaEventDisableTiming));
      if (r.tail_set) DP_CUDA(cudaStreamWaitEvent(r.h2d, r.tail, 0));
    }
    for (size_t c = 0; c < pcs.size(); ++c) {
      const Piece& p = pcs[c];
      uint8_t* stage = static_cast<uint8_t*>(r.ring) + (c % ring_slots) * slot_bytes;
      DeviceGuard gs(sdev);
      if (c >= (size_t)ring_slots) DP_CUDA(cudaStreamWaitEvent(r.h2d, fwd_done[c - ring_slots], 0));
      if (ctx->opts.debug_delay_us > 0) launch_spin((long long)ctx->opts.debug_delay_us * 2000, r.h2d);
      DP_CUDA(cudaMemcpyAsync(stage, static_cast<const uint8_t*>(m->arena) + p.off, p.bytes, cudaMemcpyHostToDevice,
                              r.h2d));
      ++st.n_copies;
      st.h2d_bytes[s] += p.bytes;
      cudaEvent_t landed = sd.events.get();
      DP_CUDA(cudaEventRecord(landed, r.h2d));
      DP_CUDA(cudaStreamWaitEvent(r.mig, landed, 0));
      if (ctx->opts.debug_delay_us > 0) launch_spin((long long)ctx->opts.debug_delay_us * 2000, r.mig);
      uint8_t* dst = m->device(primary, p.first_unit);
      if (sdev == primary)
        DP_CUDA(cudaMemcpyAsync(dst, stage, p.bytes, cudaMemcpyDeviceToDevice, r.mig));
      else
        DP_CUDA(cudaMemcpyPeerAsync(dst, primary, stage, sdev, p.bytes, r.mig));
      st.nvlink_bytes[s] += p.bytes;
      cudaEvent_t done = sd.events.get();
      DP_CUDA(cudaEventRecord(done, r.mig));
      st.n_events += 2;
      fwd_done[c] = done;
      bind_units(unit_ev, p, done);
      add_wp(s, p, done);
      if (sdev == primary) trace_piece(p, r.mig);
    }
    if (eager) {
      DeviceGuard gs(sdev);
      DP_CUDA(cudaEventRecord(r.tail, r.mig));
      r.tail_set = true;
    }
  }

  // (3) execution stream: wait per unit, then its kernels
  NvtxRange nv_fwd("enqueue forward (event-gated)");
  std::vector<char> waited_ev;
  cudaEvent_t last_waited = nullptr;
  ForwardArgs a;
  a.m = m;
  a.dev = primary;
  a.method = method;
  a.ids = ids;
  a.batch = batch;
  a.seq = seq;
  a.out = out;
  a.pooled = pooled;
  a.stream = stream;
  a.bn_hint = ctx->opts.gemm_bn;
  // Before a loaded unit's first kernel, wait for its piece -- and, in the same batch,
  // for every OTHER link's pieces that land no later than it plus kWaitSlack bytes of link
  // time: with PT the next units come from the other links at about the same time, so one
  // batch covers a round of them and the execution stream pays one dependency point (and
  // loses one PDL overlap) per round instead of per unit (a wait costs ~0.6 us in a graph,
  // ~3.6 us as a kernel outside one: tools/wait_cost.py).  On the unit's own link nothing
  // later than its piece is waited for, so one link (k = 1) waits exactly as before.
  static const bool coalesce = experiment_env("DP_NO_WAIT_COALESCE", 0) == 0;  // A/B experiments
  constexpr int64_t kWaitSlack = 2 << 20;
  std::vector<int> waited(std::max(1, plan->k), -1);
  std::vector<char> done0(wp[0].size(), 0);
  a.before_unit = [&](int u) {
    if (method[u] == DP_DHA) return;  // DHA layers skip the dependency check
    const int s0 = unit_wp[u].first, r0 = unit_wp[u].second;
    if (s0 < 0) {  // NCCL rounds (peer.cpp): one event per round, bound per unit
      cudaEvent_t e = unit_ev[u];
      DP_CHECK(e != nullptr, DP_ERR_STATE, "internal: loaded unit has no completion event");
      if (e == last_waited) return;
      DP_CUDA(cudaStreamWaitEvent(stream, e, 0));
      pdl_state().block_next = true;
      last_waited = e;
      return;
    }
    if (s0 == 0 && !fifo0) {  // several load streams: pieces of link 0 may complete out of order
      if (done0[r0]) return;
      done0[r0] = 1;
    } else if (r0 <= waited[s0]) {
      return;  // covered by an earlier wait on this link
    }
    // candidates: the pieces of the next 2k units (forward order) on the other links, if they
    // land no later than this one plus the slack -- pieces needed soon, never a later
    // partition's (with contiguous partitions the next units share this link: no batching)
    const int64_t horizon = wp[s0][r0].proxy + kWaitSlack;
    std::vector<int> want(wp.size(), -1);
    want[s0] = r0;
    for (int v = u + 1; coalesce && v < n && v <= u + 2 * (int)wp.size(); ++v) {
      const int s = unit_wp[v].first, r = unit_wp[v].second;
      if (s < 0 || s == s0 || (s == 0 && !fifo0) || r <= waited[s]) continue;
      if (wp[s][r].proxy <= horizon) want[s] = std::max(want[s], r);
    }
    std::vector<std::pair<int, int>> batch{{s0, r0}};
    for (int s = 0; s < (int)wp.size(); ++s)
      if (s != s0 && want[s] > waited[s]) batch.push_back({s, want[s]});
    std::vector<std::pair<int, size_t>> flags;  // across processes: done words, one wait kernel
    for (auto& b : batch) {
      cudaEvent_t e = wp[b.first][b.second].ev;
      if (e != nullptr)
        DP_CUDA(cudaStreamWaitEvent(stream, e, 0));
      else
        flags.push_back({b.first, (size_t)b.second});
    }
    if (!flags.empty()) ipc_primary_wait_many(ctx, flags, stream);
    for (auto& b : batch) waited[b.first] = std::max(waited[b.first], b.second);
    pdl_state().block_next = true;  // the next kernel must see the landed weights: no PDL overlap
  };
  a.pdl = ctx->opts.use_pdl != 0;
  a.attention_tc = ctx->opts.attention_tc;
  if (trace) {  // an event on each side of the unit's dependency wait
    auto gate = a.before_unit;
    a.before_unit = [&, gate](int u) {
      tr.pre[u] = stamp(stream);
      gate(u);
      tr.start[u] = stamp(stream);
    };
  }
  run_forward(a);
  if (trace) {
    tr.fin = stamp(stream);
    tr.valid = true;
  }
  // join every side stream (units never read, e.g. an unused pooler, still finish loading)
  for (int i = 0; i < nh; ++i) {
    cudaEvent_t e = pd.events.get();
    DP_CUDA(cudaEventRecord(e, pd.h2d[i]));
    DP_CUDA(cudaStreamWaitEvent(stream, e, 0));
    ++st.n_events;
  }
  for (int s = 1; s < plan->k && ctx->multiproc() && one_hop; ++s)  // every piece landed
    if (slot_npieces[s] > 0) ipc_primary_wait(ctx, s, slot_npieces[s] - 1, stream);
  for (int s = 1; s < plan->k && !ctx->multiproc(); ++s) {
    auto it = ctx->slots.find({s, secondaries[s - 1]});
    if (it == ctx->slots.end()) continue;
    DeviceGuard gs(it->second.dev);
    cudaEvent_t e = ctx->dc[it->second.dev].events.get();
    DP_CUDA(cudaEventRecord(e, it->second.mig));
    DeviceGuard gp(primary);
    DP_CUDA(cudaStreamWaitEvent(stream, e, 0));
  }
  if (ctx->comm && !one_hop) peer_join(ctx, stream);
  st.n_kernels = a.kernels;
  st.dha_weight_bytes = dha_bytes(m, method, batch * seq, seq);
  return st;
}

}  // namespace dp

extern "C" dp_status dp_infer_cold(dp_context* ctx, dp_model* m, const dp_plan* plan, int32_t primary,
                                   const int32_t* secondaries, int32_t nsec, const int32_t* d_ids, int32_t batch,
                                   int32_t seq, void* d_out, void* d_pooled, void* stream, dp_run_stats* stats) {
  return guard([&] {
    DP_CHECK(ctx && m, DP_ERR_INVALID, "NULL context/model");
    if (ctx->multiproc()) {  // multi-process PT: `primary` is a rank, each process has one device
      validate_plan(m, plan);
      DP_CHECK(primary >= 0 && primary < ctx->nranks, DP_ERR_INVALID, "primary rank out of range");
      if (ctx->rank != primary) {  // secondary rank: only its transfers
        DeviceGuard g(ctx->devs[0]);
        if (ctx->opts.pt_transport != DP_PT_DMA) {
          ipc_send_rank(ctx, m, plan, primary, stats);
        } else {
          DP_CHECK(ctx->comm, DP_ERR_STATE, "DMA transport across processes needs dp_peer_init (NCCL)");
          peer_send_rank(ctx, m, plan, primary, stats);
        }
        return;
      }
      infer_cold(ctx, m, plan, ctx->devs[0], primary, nullptr, 0, d_ids, batch, seq, d_out, d_pooled,
                 (cudaStream_t)stream, stats);
      return;
    }
    infer_cold(ctx, m, plan, primary, -1, secondaries, nsec, d_ids, batch, seq, d_out, d_pooled, (cudaStream_t)stream,
               stats);
  });
}

extern "C" dp_status dp_run_timeline(dp_context* ctx, dp_model* m, int32_t dev, int32_t n, int64_t* ready_ns,
                                     int64_t* start_ns, int64_t* end_ns, int64_t* stall_ns) {
  return guard([&] {
    DP_CHECK(ctx && m, DP_ERR_INVALID, "NULL context/model");
    ctx->on(dev);
    UnitTrace& tr = m->dev[dev].trace;
    DP_CHECK(tr.valid, DP_ERR_STATE, "no traced cold start (set opts.trace_units) of this model on this device");
    DP_CHECK(n == (int)m->units.size() && (int)tr.pre.size() == n, DP_ERR_INVALID, "n must be the unit count");
    DeviceGuard g(dev);
    DP_CUDA(cudaDeviceSynchronize());  // pieces on side streams may land after the forward's end
    std::vector<uint64_t> h(tr.used);
    DP_CUDA(cudaMemcpy(h.data(), tr.dbuf, sizeof(uint64_t) * tr.used, cudaMemcpyDeviceToHost));
    auto ns = [&](int slot) -> int64_t {
      if (slot < 0 || h[slot] == 0) return -1;
      return (int64_t)h[slot] - (int64_t)h[tr.t0];
    };    const int8_t* method = m->dev[dev].method.data();
    for (int u = 0; u < n; ++u) {
      const int64_t pre = ns(tr.pre[u]), start = ns(tr.start[u]);
      int64_t end = -1;
      if (start >= 0) {
        int v = u + 1;
        while (v < n && tr.pre[v] < 0) ++v;
        end = v < n ? ns(tr.pre[v]) : ns(tr.fin);
      }
      if (ready_ns) ready_ns[u] = method[u] == DP_DHA ? 0 : ns(tr.ready[u]);
      if (start_ns) start_ns[u] = start;
      if (end_ns) end_ns[u] = end;
      if (stall_ns) stall_ns[u] = (start >= 0 && pre >= 0) ? std::max<int64_t>(0, start - pre) : -1;
    }
  });
}

extern "C" dp_status dp_infer_warm(dp_context* ctx, dp_model* m, int32_t dev, const int32_t* d_ids, int32_t batch,
                                   int32_t seq, void* d_out, void* d_pooled, void* stream, dp_run_stats* stats) {
  return guard([&] {
    DP_CHECK(ctx && m, DP_ERR_INVALID, "NULL context/model");
    ctx->on(dev);
    DevState& ds = m->dev[dev];
    DP_CHECK(ds.resident, DP_ERR_STATE, "model is not resident on this device");
    DP_CHECK(batch > 0 && seq > 0 && d_ids && d_out, DP_ERR_INVALID, "bad inference arguments");
    NvtxRange nv("dp_infer_warm");
    DeviceGuard g(dev);
    auto t0 = std::chrono::steady_clock::now();
    ForwardArgs a;
    a.m = m;
    a.dev = dev;
    a.method = ds.method.data();
    a.ids = d_ids;
    a.batch = batch;
    a.seq = seq;
    a.out = d_out;
    a.pooled = d_pooled;
    a.stream = (cudaStream_t)stream;
    a.bn_hint = ctx->opts.gemm_bn;
    a.pdl = ctx->opts.use_pdl != 0;
  a.attention_tc = ctx->opts.attention_tc;
    // Experiment (tools/wait_cost.py): the cost of a dependency wait before every unit on the
    // execution stream, all already satisfied -- 1: event wait, 2: one-thread acquire-spin
    // kernel on a device word, 3: cuStreamWaitValue32 (stream memory op)
    static const int dbg_waits = experiment_env("DP_DEBUG_WARM_WAITS", 0);
    static uint32_t* dbg_word = nullptr;
    static cudaStream_t dbg_side = nullptr;
    static cudaEvent_t dbg_fork = nullptr, dbg_ev = nullptr;
    using WaitValueFn = CUresult (*)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);
    static WaitValueFn wait_value = nullptr;
    if (dbg_waits) {
      if (!dbg_word) {
        DP_CUDA(cudaMalloc(&dbg_word, 64));
        DP_CUDA(cudaMemset(dbg_word, 1, 64));
        DP_CUDA(cudaStreamCreateWithFlags(&dbg_side, cudaStreamNonBlocking));
        DP_CUDA(cudaEventCreateWithFlags(&dbg_fork, cudaEventDisableTiming));
        DP_CUDA(cudaEventCreateWithFlags(&dbg_ev, cudaEventDisableTiming));
        cudaDriverEntryPointQueryResult q;
        DP_CUDA(cudaGetDriverEntryPoint("cuStreamWaitValue32", reinterpret_cast<void**>(&wait_value),
                                        cudaEnableDefault, &q));
      }
      a.before_unit = [&](int u) {
        if (ds.method[u] == DP_DHA) return;
        if (dbg_waits == 1) {
          DP_CUDA(cudaStreamWaitEvent(a.stream, dbg_ev, 0));
        } else if (dbg_waits == 2) {
          launch_pt_wait(dbg_word, 1, a.stream);
        } else {
          DP_CHECK(wait_value(a.stream, (CUdeviceptr)dbg_word, 1, CU_STREAM_WAIT_VALUE_GEQ) == CUDA_SUCCESS,
                   DP_ERR_CUDA, "cuStreamWaitValue32 failed");
        }
        pdl_state().block_next = true;
      };
    }
    auto dbg_fork_side = [&](cudaStream_t st) {
      if (dbg_waits != 1) return;
      DP_CUDA(cudaEventRecord(dbg_fork, st));
      DP_CUDA(cudaStreamWaitEvent(dbg_side, dbg_fork, 0));
      DP_CUDA(cudaEventRecord(dbg_ev, dbg_side));
    };
    if (ctx->opts.use_graph) {
      std::string key = "warm|" + std::string(reinterpret_cast<const char*>(ds.method.data()), ds.method.size()) +
                        graph_key(ctx, ds, nullptr, nullptr, d_ids, batch, seq, d_out, d_pooled);
      if (dbg_waits) key += "|dbgwait" + std::to_string(dbg_waits);
      dp_run_stats gs = run_graph(ds, key, (cudaStream_t)stream, [&](cudaStream_t cs) {
        a.stream = cs;
        dbg_fork_side(cs);
        run_forward(a);
        dp_run_stats s{};
        s.n_kernels = a.kernels;
        return s;
      });
      a.kernels = gs.n_kernels;
    } else {
      dbg_fork_side(a.stream);
      run_forward(a);
    }
    if (stats) {
      std::memset(stats, 0, sizeof(*stats));
      stats->n_kernels = a.kernels;
      stats->n_units = (int)m->units.size();
      stats->dha_weight_bytes = dha_bytes(m, ds.method.data(), batch * seq, seq);
      stats->wall_enqueue_us =
          std::chrono::duration<float, std::micro>(std::chrono::steady_clock::now() - t0).count();
    }
  });
}

extern "C" dp_status dp_lm_head(dp_context* ctx, dp_model* m, int32_t dev, const void* d_hidden, int32_t ld_hidden,
                                int32_t rows, float* d_logits, void* stream) {
  return guard([&] {
    DP_CHECK(ctx && m && d_hidden && d_logits, DP_ERR_INVALID, "NULL argument");
    DP_CHECK(m->cfg.family == DP_FAMILY_GPT2, DP_ERR_UNSUPPORTED, "tied LM head: GPT-2 models only");
    DP_CHECK(rows >= 0 && ld_hidden >= m->cfg.hidden && ld_hidden % 8 == 0, DP_ERR_INVALID, "bad rows / ld_hidden");
    ctx->on(dev);
    DeviceGuard g(dev);
    const DevState& ds = m->dev[dev];
    // unit 0 = wte; its weight is the first parameter of the unit
    const bool in_hbm = ds.resident && !ds.method.empty() && ds.method[0] == DP_LOAD;
    const void* wte = in_hbm ? static_cast<const void*>(m->device(dev, 0)) : static_cast<const void*>(m->host(0));
    launch_skinny_linear(m->cfg.dtype, d_hidden, ld_hidden, wte, nullptr, nullptr, 0, d_logits, m->cfg.vocab, rows,
                         m->cfg.vocab, m->cfg.hidden, ACT_NONE, IO_OUT_F32, (cudaStream_t)stream);
  });
}

extern "C" dp_status dp_model_evict(dp_context* ctx, dp_model* m, int32_t dev) {
  return guard([&] {
    DP_CHECK(ctx && m, DP_ERR_INVALID, "NULL context/model");
    ctx->on(dev);
    DeviceGuard g(dev);
    DP_CUDA(cudaDeviceSynchronize());
    if (ctx->opts.debug_poison && m->dev[dev].dbase) {
      DP_CUDA(cudaMemset(m->dev[dev].dbase, 0xFF, m->dev[dev].dbytes));
      DP_CUDA(cudaDeviceSynchronize());
    }
    m->dev[dev].resident = false;
    release_slots(ctx, m, dev);  // the block returns to the device's pool
  });
}

extern "C" int64_t dp_model_resident_bytes(const dp_model* m, int32_t dev) {
  if (!m || dev < 0 || dev >= DP_MAX_DEVICES || !m->dev[dev].resident) return 0;
  return m->dev[dev].dbytes;
}

extern "C" int64_t dp_plan_resident_bytes(const dp_model* m, const dp_plan* plan) {
  if (!m || !plan || !plan->method || plan->n != (int)m->units.size()) return -1;
  return plan_resident_bytes(m, plan->method);
}

extern "C" dp_status dp_pool_stats(dp_context* ctx, int32_t dev, int64_t* reserved, int64_t* in_use) {
  return guard([&] {
    DP_CHECK(ctx && reserved && in_use, DP_ERR_INVALID, "NULL argument");
    const HbmPool& p = ctx->on(dev).pool;
    *reserved = p.reserved;
    *in_use = p.in_use;
  });
}

extern "C" dp_status dp_pool_trim(dp_context* ctx, int32_t dev, int64_t* freed) {
  return guard([&] {
    DP_CHECK(ctx, DP_ERR_INVALID, "NULL context");
    const int64_t f = pool_trim(ctx->on(dev).pool, dev);
    if (freed) *freed = f;
  });
}

extern "C" int32_t dp_model_is_resident(const dp_model* m, int32_t dev) {
  if (!m || dev < 0 || dev >= DP_MAX_DEVICES) return 0;
  return m->dev[dev].resident ? 1 : 0;
}

extern "C" dp_status dp_model_destroy(dp_context* ctx, dp_model* m) {
  return guard([&] {
    if (!m) return;
    for (int d = 0; d < DP_MAX_DEVICES; ++d) {
      DevState& ds = m->dev[d];
      if (ds.dbase || ds.ws.base) {
        DeviceGuard g(d);
        cudaDeviceSynchronize();
        for (auto& kv : ds.graphs) cudaGraphExecDestroy(kv.second.exec);
        ds.graphs.clear();
        if (ds.trace.dbuf) cudaFree(ds.trace.dbuf);
        if (ds.capture) cudaStreamDestroy(ds.capture);
        if (ds.pinned_full) {
          cudaFree(ds.dbase);
        } else if (ds.dbase && ctx) {
          release_slots(ctx, m, d);
        }
        if (ds.ws.base) cudaFree(ds.ws.base);
      }
    }
    ipc_close_model(m);
    delete m;  // the last instance sharing the arena frees it
  });
}

// ---------------------------------------------------------------------------------------
// Profiler (§4.3.1; 10 iterations per Table 5)
// ---------------------------------------------------------------------------------------

namespace dp {

static int64_t median_ns(std::vector<float>& ms) {
  std::sort(ms.begin(), ms.end());
  const size_t k = ms.size();
  const double med = k % 2 ? ms[k / 2] : 0.5 * (ms[k / 2 - 1] + ms[k / 2]);
  return (int64_t)llround(med * 1e6);
}

struct CostOut {  // the caller-owned output arrays of a dp_cost_table
  int64_t *bytes, *load_ns, *fwd_ns, *exe_mem_ns, *exe_dha_ns;
};

void profile(dp_context* ctx, dp_model* m, int dev, int batch, int seq, int iters, dp_cost_table* table) {
  NvtxRange nv("dp_profile");
  DP_CHECK(table && table->n == (int)m->units.size(), DP_ERR_INVALID, "cost table size mismatch");
  DP_CHECK(table->bytes && table->load_ns && table->fwd_ns && table->exe_mem_ns && table->exe_dha_ns, DP_ERR_INVALID,
           "cost table arrays are NULL");
  CostOut o{const_cast<int64_t*>(table->bytes), const_cast<int64_t*>(table->load_ns),
            const_cast<int64_t*>(table->fwd_ns), const_cast<int64_t*>(table->exe_mem_ns),
            const_cast<int64_t*>(table->exe_dha_ns)};
  CostOut* out = &o;
  DP_CHECK(iters >= 1 && batch > 0 && seq > 0, DP_ERR_INVALID, "bad profiling arguments");
  DevCtx& d = ctx->on(dev);
  DevState& ds = m->dev[dev];
  DP_CHECK(!ds.resident, DP_ERR_STATE, "evict the model before profiling");
  DeviceGuard g(dev);
  acquire_slots(ctx, m, dev, nullptr);  // every unit resident for the in-memory runs (full layout)
  struct Release {
    dp_context* c;
    dp_model* mm;
    int d;
    ~Release() {
      try {
        cudaDeviceSynchronize();
        release_slots(c, mm, d);
      } catch (...) {
      }
    }
  } release_at_exit{ctx, m, dev};
  const int T = batch * seq;
  ensure_workspace(m, dev, T);
  if (!d.flush) {
    d.flush_bytes = 256ll << 20;  // > 126 MB L2
    DP_CUDA(cudaMalloc(&d.flush, d.flush_bytes));
  }
  cudaStream_t s;
  DP_CUDA(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  int32_t* ids = nullptr;
  DP_CUDA(cudaMalloc(&ids, sizeof(int32_t) * T));
  {
    std::vector<int32_t> h(T);
    const int lo = m->cfg.family == DP_FAMILY_ROBERTA ? 3 : 0;
    for (int t = 0; t < T; ++t) h[t] = lo + int((uint64_t(t) * 2654435761ull) % uint64_t(m->cfg.vocab - lo));
    DP_CUDA(cudaMemcpy(ids, h.data(), sizeof(int32_t) * T, cudaMemcpyHostToDevice));
  }
  DP_CUDA(cudaMemset(m->dev[dev].ws.base, 0, 1));
  // all weights resident for the in-memory runs
  DP_CUDA(cudaMemcpy(ds.dbase, m->arena, m->arena_bytes, cudaMemcpyHostToDevice));  // full layout
  cudaEvent_t e0, e1;
  DP_CUDA(cudaEventCreate(&e0));
  DP_CUDA(cudaEventCreate(&e1));
  const int warm = 3;
  const int n = (int)m->units.size();
  auto timed = [&](auto&& body, bool flush, long long spin = 60000) {
    std::vector<float> v;
    for (int it = 0; it < warm + iters; ++it) {
      if (flush) launch_l2_flush(d.flush, d.flush_bytes, s);
      // keep the stream busy while the host enqueues the measured work, so the interval
      // e0..e1 holds device time only (not the host's launch latency)
      launch_spin(spin, s);
      DP_CUDA(cudaEventRecord(e0, s));
      body();
      DP_CUDA(cudaEventRecord(e1, s));
      DP_CUDA(cudaEventSynchronize(e1));
      float ms = 0;
      DP_CUDA(cudaEventElapsedTime(&ms, e0, e1));
      if (it >= warm) v.push_back(ms);
    }
    return median_ns(v);
  };
  // embedding units share one fused kernel: attribute T(all HBM) evenly, and each unit's
  // DHA cost as the marginal time of reading that table from host (DESIGN.md §3 R8)
  std::vector<int> emb;
  for (int u = 0; u < n; ++u)
    if (m->units[u].role == R_WORD || m->units[u].role == R_POS || m->units[u].role == R_TYPE ||
        m->units[u].role == R_EMB_LN || m->units[u].role == R_WTE || m->units[u].role == R_WPE)
      emb.push_back(u);
  int64_t emb_all_mem = 0;
  if (!emb.empty())
    emb_all_mem = timed([&] { run_unit(m, dev, emb[0], false, ids, batch, seq, s, ctx->opts.gemm_bn); }, true);
  for (int u = 0; u < n; ++u) {
    const auto& un = m->units[u];
    out->bytes[u] = un.bytes;
    uint8_t* dst = m->device(dev, u);
    const uint8_t* src = static_cast<const uint8_t*>(m->arena) + un.off;
    out->load_ns[u] = timed([&] { DP_CUDA(cudaMemcpyAsync(dst, src, un.bytes, cudaMemcpyHostToDevice, s)); }, false);
    uint8_t* scratch = static_cast<uint8_t*>(d.flush);
    const int64_t fb = std::min<int64_t>(un.bytes, d.flush_bytes / 2);
    out->fwd_ns[u] = timed([&] { DP_CUDA(cudaMemcpyAsync(scratch, dst, fb, cudaMemcpyDeviceToDevice, s)); }, false);
    const bool is_emb = std::find(emb.begin(), emb.end(), u) != emb.end();
    if (is_emb) {
      const int64_t share = emb_all_mem / (int64_t)emb.size();
      const int64_t with_host = timed([&] { run_unit(m, dev, u, true, ids, batch, seq, s, ctx->opts.gemm_bn); }, true);
      out->exe_mem_ns[u] = share;
      out->exe_dha_ns[u] = share + std::max<int64_t>(0, with_host - emb_all_mem);
    } else {
      out->exe_mem_ns[u] = timed([&] { run_unit(m, dev, u, false, ids, batch, seq, s, ctx->opts.gemm_bn); }, true);
      out->exe_dha_ns[u] = timed([&] { run_unit(m, dev, u, true, ids, batch, seq, s, ctx->opts.gemm_bn); }, true);
    }
  }
  // R23: the chained warm forward (every unit resident, PDL chain as the engine runs it, L2
  // flushed before it) against the sum of the isolated unit times; Exe(InMem) is rescaled to
  // it, Exe(DHA) keeps its absolute extra (the host reads) over Exe(InMem)
  if (ctx->opts.profile_chain) {
    std::vector<int8_t> all_load(n, DP_LOAD);
    ForwardArgs fa;
    fa.m = m;
    fa.dev = dev;
    fa.method = all_load.data();
    fa.ids = ids;
    fa.batch = batch;
    fa.seq = seq;
    void* chain_out = nullptr;
    DP_CUDA(cudaMalloc(&chain_out, size_t(T) * m->cfg.hidden * 4));
    fa.out = chain_out;
    fa.pooled = nullptr;
    fa.stream = s;
    fa.bn_hint = ctx->opts.gemm_bn;
    fa.pdl = ctx->opts.use_pdl != 0;
    fa.attention_tc = ctx->opts.attention_tc;
    // the host enqueues ~100 launches behind a ~1.5 ms spin, so e0..e1 is device time only
    const int64_t chain = timed([&] { run_forward(fa); }, true, 3000000);
    DP_CUDA(cudaStreamSynchronize(s));
    cudaFree(chain_out);
    int64_t sum = 0;
    for (int u = 0; u < n; ++u) sum += out->exe_mem_ns[u];
    // loads: the engine coalesces adjacent loaded units into large DMAs (R18), so a unit's
    // marginal link time is its share of one copy of the whole arena, not an isolated copy
    // (which carries ~4 us of per-copy cost: 98 BERT-Base units would add ~0.4 ms)
    const int64_t all_ns = timed([&] {
      DP_CUDA(cudaMemcpyAsync(ds.dbase, m->arena, m->arena_bytes, cudaMemcpyHostToDevice, s));
    }, false);
    for (int u = 0; u < n; ++u)
      out->load_ns[u] = (int64_t)llround(double(all_ns) * double(out->bytes[u]) / double(m->arena_bytes));
    if (chain > 0 && sum > chain) {
      const double f = double(chain) / double(sum);
      for (int u = 0; u < n; ++u) {
        const int64_t mem = (int64_t)llround(double(out->exe_mem_ns[u]) * f);
        if (out->exe_dha_ns[u] < DP_INF_NS) out->exe_dha_ns[u] = std::max<int64_t>(0, mem + out->exe_dha_ns[u] - out->exe_mem_ns[u]);
        out->exe_mem_ns[u] = mem;
      }
    }
  }
  // link time of each unit's DHA reads (link-aware modes): the unit's own measured load time
  // scaled by the fraction of its bytes a DHA execution touches -- a linear or LayerNorm reads
  // every byte (no link time freed), an embedding only the used rows (R19)
  if (table->dha_link_ns) {
    int64_t* dl = const_cast<int64_t*>(table->dha_link_ns);
    for (int u = 0; u < n; ++u) {
      const int64_t touched = std::min(unit_dha_bytes(m, u, T, seq), out->bytes[u]);
      dl[u] = out->bytes[u] > 0 ? (int64_t)llround(double(out->load_ns[u]) * double(touched) / double(out->bytes[u]))
                                : 0;
    }
  }
  DP_CUDA(cudaStreamSynchronize(s));
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  cudaFree(ids);
  cudaStreamDestroy(s);
}

}  // namespace dp

extern "C" dp_status dp_measure_h2d(int32_t dev, int64_t bytes, int32_t reps, double* gbs) {
  void* h = nullptr;
  void* d = nullptr;
  cudaStream_t s = nullptr;
  cudaEvent_t e0 = nullptr, e1 = nullptr;
  dp_status st = guard([&] {
    DP_CHECK(gbs && bytes > 0 && reps >= 1, DP_ERR_INVALID, "bad arguments");
    DeviceGuard g(dev);
    if (cudaHostAlloc(&h, bytes, cudaHostAllocPortable | cudaHostAllocMapped) != cudaSuccess) {
      h = nullptr;
      fail(DP_ERR_OOM, "cudaHostAlloc failed");
    }
    std::memset(h, 1, bytes);
    if (cudaMalloc(&d, bytes) != cudaSuccess) {
      d = nullptr;
      fail(DP_ERR_OOM, "cudaMalloc failed");
    }
    DP_CUDA(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
    DP_CUDA(cudaEventCreate(&e0));
    DP_CUDA(cudaEventCreate(&e1));
    float best = 1e30f;
    for (int r = 0; r <= reps; ++r) {  // first copy is a warm-up
      DP_CUDA(cudaEventRecord(e0, s));
      DP_CUDA(cudaMemcpyAsync(d, h, bytes, cudaMemcpyHostToDevice, s));
      DP_CUDA(cudaEventRecord(e1, s));
      DP_CUDA(cudaEventSynchronize(e1));
      float ms = 0;
      DP_CUDA(cudaEventElapsedTime(&ms, e0, e1));
      if (r > 0) best = std::min(best, ms);
    }
    *gbs = double(bytes) / (double(best) * 1e-3) / 1e9;
  });
  if (e0) cudaEventDestroy(e0);
  if (e1) cudaEventDestroy(e1);
  if (s) cudaStreamDestroy(s);
  if (d) cudaFree(d);
  if (h) cudaFreeHost(h);
  return st;
}

extern "C" dp_status dp_profile(dp_context* ctx, dp_model* m, int32_t dev, int32_t batch, int32_t seq, int32_t iters,
                                dp_cost_table* out) {
  return guard([&] {
    DP_CHECK(ctx && m, DP_ERR_INVALID, "NULL context/model");
    profile(ctx, m, dev, batch, seq, iters, out);
  });
}
