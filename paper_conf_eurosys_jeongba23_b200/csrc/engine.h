// Execution engine internals: context, per-device resources, forward program.
#pragma once
#include <cuda_runtime.h>

#include <functional>
#include <map>
#include <vector>

#include "model.h"

namespace dp {

struct EventPool {
  int dev = -1;
  std::vector<cudaEvent_t> ev;
  size_t used = 0;
  cudaEvent_t get();
  void reset() { used = 0; }
  void destroy();
};

// Resources of one PT slot served by device `dev`: its load stream, its migration stream
// ("an additional migration stream on each secondary GPU") and the staging ring
// ("we reserve a small amount of memory for storing layers temporarily").
struct SlotRes {
  int dev = -1;
  cudaStream_t h2d = nullptr, mig = nullptr;
  void* ring = nullptr;
  int64_t ring_bytes = 0;
  // the last cold start's final forward out of the ring: the next cold start using this slot
  // resource (e.g. a concurrent one on another primary, in serving) waits for it before its first
  // H2D into the ring
  cudaEvent_t tail = nullptr;
  bool tail_set = false;
};

// A contiguous byte range of the arena moved by one DMA (and one forward for PT): the
// whole units first_unit..last_unit (all selected by the plan for the same link).
struct Piece {
  int64_t off = 0, bytes = 0;
  int first_unit = -1, last_unit = -1;
};

// Device-memory pool of one device (infer.cu): the HBM slot blocks of the models.  Evicting a
// model returns its block here (not to the driver), so the next cold start of any model reuses
// it; dp_pool_trim releases the free blocks to the driver.
struct HbmPool {
  std::multimap<int64_t, void*> free_;  // free blocks by size
  std::map<void*, int64_t> size_;       // every block the pool owns -> its size
  int64_t reserved = 0, in_use = 0;
};

struct DevCtx {
  int ord = -1;
  HbmPool pool;
  bool ready = false;
  std::vector<cudaStream_t> h2d;  // load streams ("load stream")
  EventPool events;
  void* flush = nullptr;  // L2 flush buffer (profiling)
  int64_t flush_bytes = 0;
};

struct ForwardArgs {
  dp_model* m = nullptr;
  int dev = 0;
  const int8_t* method = nullptr;  // per unit DP_LOAD / DP_DHA (where the weights are read from)
  const int32_t* ids = nullptr;
  int batch = 0, seq = 0;
  void* out = nullptr;
  void* pooled = nullptr;
  cudaStream_t stream = nullptr;
  std::function<void(int)> before_unit;  // called before the first kernel using a unit
  int kernels = 0;
  int bn_hint = 0;
  bool pdl = false;  // chain kernels with programmatic dependent launch (opts.use_pdl)
  int attention_tc = 0;  // attention core choice (opts.attention_tc: 0 by length, 1 K5t, 2 K5 / K5b)
};

void ensure_workspace(dp_model* m, int dev, int64_t tokens);
// HBM slots of the units `method` loads (compact layout, from the pool; infer.cu), their release,
// and the full-arena slots of an IPC-exported model.
void acquire_slots(dp_context* ctx, dp_model* m, int dev, const int8_t* method);
void release_slots(dp_context* ctx, dp_model* m, int dev);
void pin_full_slots(dp_model* m, int dev);
// Destroy every captured graph / K6 program of a device state (their buffers are going away).
void drop_graphs(DevState& ds);
void run_forward(ForwardArgs& a);

// Execute one unit's ops in isolation (profiling): inputs are the workspace buffers.
void run_unit(dp_model* m, int dev, int unit, bool dha, const int32_t* ids, int batch, int seq, cudaStream_t s,
              int bn_hint);

}  // namespace dp

struct dp_context {
  std::vector<int> devs;
  dp::DevCtx dc[DP_MAX_DEVICES];
  dp_engine_opts opts{};
  std::map<std::pair<int, int>, dp::SlotRes> slots;  // (slot, device) -> resources
  // multi-process PT: NCCL (dp_peer_init) or CUDA IPC + SM forwarder (dp_peer_init_ipc)
  void* comm = nullptr;
  int rank = -1, nranks = 0;  // nranks > 0: multi-process (`primary` is a rank)
  cudaStream_t comm_stream = nullptr;
  uint32_t* mailbox = nullptr;                    // this rank's (pt_forward.cu layout)
  uint32_t* peer_mailbox[DP_MAX_DEVICES] = {};     // other ranks' (IPC-mapped), by rank
  uint32_t pt_epoch = 0;                          // cold starts run in SM/IPC mode so far
  uint64_t ring_gen = 0;  // bumped whenever a staging ring is reallocated (part of graph keys)
  int slot_map_primary = -1;              // dp_peer_set_slot_ranks: the primary the map is for
  int slot_rank[DP_MAX_DEVICES] = {-1, -1, -1, -1, -1, -1, -1, -1};  // slot s -> rank
  bool multiproc() const { return nranks > 0; }
  dp::DevCtx& on(int dev);
};
