// Multi-instance serving harness (§5.3).
//
// "As Clockwork [13], our execution engine is designed for each GPU to run one
// inference request at a time."  P:338: "To evict an instance due to the lack of GPU
// memory, we select the least recently used instance."  P:328: Poisson arrivals spread
// uniformly over the instances.  The dispatch policy (DESIGN.md §3 R11) is decided per
// request at its arrival, in arrival order:
//   * instance resident on GPU g        -> warm on g (queue behind g's earlier requests);
//   * otherwise                         -> cold start on the GPU that frees up first (ties:
//     lowest index), evicting LRU instances there until its resident bytes fit the budget;
//   * start = max(arrival, GPU free time); finish = start + latency; the GPU's LRU list is
//     touched.  PT borrows other GPUs' PCIe links, not their compute (Table 4).
// dry_run = 1 replays with a latency table; the live mode (serve_live.cu) is an online
// dispatcher on the GPUs' observed state with real cold / warm inferences and evictions.
#include <algorithm>
#include <list>
#include <vector>

#include "common.h"
#include "serve.h"

namespace dp {

void serve_decide(const dp_serve_opts& o, const dp_trace_event* trace, int nreq, dp_serve_result* out,
                  std::vector<int64_t>* order_lat) {
  DP_CHECK(o.ngpu >= 1 && o.ngpu <= 64, DP_ERR_INVALID, "ngpu out of range");
  DP_CHECK(o.nmodels >= 1 && o.cold_ns && o.warm_ns && o.resident_bytes, DP_ERR_INVALID, "latency table missing");
  DP_CHECK(o.ninstances >= 1 && o.model_of_instance, DP_ERR_INVALID, "instance table missing");
  const int G = o.ngpu;
  std::vector<int64_t> busy(G, 0), used(G, 0);
  std::vector<std::list<int>> lru(G);     // front = least recently used
  std::vector<int> where(o.ninstances, -1);
  int64_t prev_arrival = INT64_MIN;
  for (int r = 0; r < nreq; ++r) {
    const int inst = trace[r].instance;
    DP_CHECK(inst >= 0 && inst < o.ninstances, DP_ERR_INVALID, "trace instance out of range");
    DP_CHECK(trace[r].arrival_ns >= prev_arrival, DP_ERR_INVALID, "trace must be sorted by arrival");
    prev_arrival = trace[r].arrival_ns;
    const int model = o.model_of_instance[inst];
    DP_CHECK(model >= 0 && model < o.nmodels, DP_ERR_INVALID, "model index out of range");
    dp_serve_result& res = out[r];
    res = dp_serve_result{};
    int g = where[inst];
    if (g >= 0) {
      res.cold = 0;
      lru[g].remove(inst);
    } else {
      g = 0;
      for (int j = 1; j < G; ++j)
        if (busy[j] < busy[g]) g = j;
      const int64_t need = o.resident_bytes[model];
      DP_CHECK(need <= o.per_gpu_budget_bytes, DP_ERR_INVALID, "an instance does not fit the per-GPU budget");
      while (used[g] + need > o.per_gpu_budget_bytes) {
        const int victim = lru[g].front();
        lru[g].pop_front();
        used[g] -= o.resident_bytes[o.model_of_instance[victim]];
        where[victim] = -1;
        ++res.nevicted;
      }
      used[g] += need;
      where[inst] = g;
      res.cold = 1;
    }
    lru[g].push_back(inst);
    res.gpu = g;
    res.start_ns = std::max(trace[r].arrival_ns, busy[g]);
    res.finish_ns = res.start_ns + (res.cold ? o.cold_ns[model] : o.warm_ns[model]);
    res.decide_ns = trace[r].arrival_ns;
    busy[g] = res.finish_ns;
  }
  (void)order_lat;
}

}  // namespace dp

using namespace dp;

extern "C" dp_status dp_serve_run(dp_context* ctx, dp_model* const* models, int32_t nmodels, const dp_trace_event* trace,
                                  int32_t nreq, const dp_serve_opts* opts, dp_serve_result* out) {
  return guard([&] {
    DP_CHECK(opts && (nreq == 0 || (trace && out)), DP_ERR_INVALID, "NULL argument");
    DP_CHECK(nreq >= 0, DP_ERR_INVALID, "nreq < 0");
    if (opts->dry_run) {
      serve_decide(*opts, trace, nreq, out, nullptr);
      return;
    }
    serve_live(ctx, models, nmodels, trace, nreq, *opts, out);
  });
}
