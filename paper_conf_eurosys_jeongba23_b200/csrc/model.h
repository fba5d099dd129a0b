// Model registration: parameter list, planning units, pinned host arena, per-device state.
#pragma once
#include <cuda_runtime.h>

#include <map>
#include <memory>
#include <string>
#include <vector>

#include "common.h"

namespace dp {

enum Role {
  R_WORD, R_POS, R_TYPE, R_EMB_LN,                                 // BERT/RoBERTa embeddings
  R_Q, R_K, R_V, R_ATTN_OUT, R_LN1, R_FC1, R_FC2, R_LN2, R_POOLER,  // BERT/RoBERTa layer + pooler
  R_WTE, R_WPE,                                                    // GPT-2 embeddings
  R_LN_1, R_C_ATTN, R_C_PROJ, R_LN_2, R_C_FC, R_MLP_PROJ, R_LN_F   // GPT-2 block + final LN
};

struct ParamDesc {
  std::string hf;
  int ndim = 1;
  int64_t shape[2] = {0, 0};
  int unit = -1;
  int64_t bytes = 0;
  bool transpose = false;  // GPT-2 Conv1D [in,out] -> stored [out,in]
  int64_t off = 0;         // arena offset
};

struct UnitDesc {
  std::string name;
  int kind = DP_UNIT_LINEAR;
  int role = 0;
  int layer = -1;
  int first_param = 0, nparams = 0;
  int64_t off = 0, bytes = 0;
  int64_t N = 0, K = 0;  // linear: W [N, K] at off, bias [N] at off + N*K*(element bytes)
};

// Activation workspace on one device for T tokens.
struct Workspace {
  int64_t tokens = 0;
  void* x = nullptr;    // [T, H]
  void* qkv = nullptr;  // [T, 3H]
  void* ctx = nullptr;  // [T, H]
  void* tmp = nullptr;  // [T, H] fp32 (pre-LayerNorm sums)
  void* x1 = nullptr;   // [T, H]
  void* h = nullptr;    // [T, F]
  void* xr = nullptr;   // [T, H] fp32: BERT/RoBERTa residual stream (copy of x)
  void* x1r = nullptr;  // [T, H] fp32: copy of x1
  void* base = nullptr;
};


struct GraphEntry {
  cudaGraphExec_t exec = nullptr;
  dp_run_stats stats{};
};

// Per-unit timestamps of a traced cold start (opts.trace_units; dp_run_timeline): one-thread
// kernels write %globaltimer into slots of a device buffer (timing events were measured to lag by
// up to ~25 us on the execution stream while a DMA is in flight, which swamps per-unit stalls).
struct UnitTrace {
  bool valid = false;
  uint64_t* dbuf = nullptr;  // device slots
  int cap = 0, used = 0;
  int t0 = -1, fin = -1;
  std::vector<int> ready, pre, start;  // per unit: slot index (-1: not observed)
  cudaStream_t last_stream = nullptr;
};

struct DevState {
  // HBM slots of the loaded units: one block from the context's pool (infer.cu), laid out like
  // the arena with the DHA units' ranges left out (they stay in host memory: DeepPlan
  // "serves more instances" because DHA layers take no GPU memory)
  void* dbase = nullptr;
  int64_t dbytes = 0;          // bytes of the block
  std::vector<int64_t> doff;   // per unit: offset in the block, -1 for a DHA unit (read in place)
  bool pinned_full = false;    // IPC-exported slots: full arena layout, outside the pool, kept
  void* last_block = nullptr;  // the block released by the last eviction (reacquired if free)
  std::vector<void*> graph_blocks;  // blocks this model has captured graphs on (preferred next)
  bool resident = false;
  std::vector<int8_t> method;  // per unit, fixed when the model became resident
  Workspace ws;
  std::map<std::string, GraphEntry> graphs;  // captured cold / warm runs (opts.use_graph)
  std::map<std::string, int> graph_seen;     // keys run so far (captured on the second use)
  UnitTrace trace;                           // last traced cold start
  cudaStream_t capture = nullptr;            // private stream the graphs are captured on
};

std::vector<ParamDesc> config_params(const dp_model_config& c);
// topo.cpp
int device_numa_node(int dev);
void* host_alloc_on_node(int64_t bytes, int node);
void validate_config(const dp_model_config& c);

}  // namespace dp

struct dp_model;
namespace dp {
// Units + arena layout for m->cfg / m->params (host-only; no allocation).
void build_units(dp_model* m);
}  // namespace dp

struct dp_model {
  dp_model_config cfg{};
  std::vector<dp::ParamDesc> params;
  std::vector<dp::UnitDesc> units;
  void* arena = nullptr;  // cudaHostAlloc(Portable | Mapped), on NUMA node arena_node
  int arena_node = -1;
  std::shared_ptr<void> arena_owner;  // shared by dp_model_clone instances
  int64_t arena_bytes = 0;
  dp::DevState dev[DP_MAX_DEVICES];
  void* peer_dbase[DP_MAX_DEVICES] = {};  // other ranks' HBM slots, IPC-mapped (by rank)

  const uint8_t* host(int u) const { return static_cast<const uint8_t*>(arena) + units[u].off; }
  uint8_t* device(int d, int u) const { return static_cast<uint8_t*>(dev[d].dbase) + dev[d].doff[u]; }
};
