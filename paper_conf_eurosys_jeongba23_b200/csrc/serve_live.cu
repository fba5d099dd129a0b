// Live multi-instance serving (§5.3): an ONLINE dispatcher on the GPUs' live state.
//
// One host thread owns the context (no lock: every enqueue is its own) and runs an event loop
// over three kinds of events, in this order per iteration:
//   1. completions: a GPU's running request finished (its completion event fired) -- stamped
//      with the time the loop observed it;
//   2. arrivals whose wall-clock time has come (P:328 trace), decided at once on the current
//      state (R11-live):
//        * the instance is (or is becoming) resident on GPU g -> warm, queued on g;
//        * otherwise cold, on the GPU with the fewest outstanding requests (running + queued;
//          ties: lowest index);
//        * then, while that GPU's resident bytes exceed the per-GPU budget, the least recently
//          used instance other than this one with no outstanding request is evicted.
//          Resident bytes are the instance's LOADED units only (its plan's compact slot layout):
//          DHA units stay in host memory, which is how DeepPlan "serves more instances";
//   3. starts: every idle GPU with a queued request runs the next one (one request per GPU
//      at a time): the evictions decided for it (dp_model_evict -- the HBM block returns to the
//      pool), then dp_infer_cold / dp_infer_warm on the GPU's stream and a completion event.
//      A cold start with a PT plan (k > 1) borrows k-1 other GPUs' PCIe links and copy engines
//      (not their compute, P:322 / Table 4): idle GPUs first (no running or queued request),
//      then the ones with the fewest outstanding requests.
// Every decision depends only on what the loop had observed when it made it, so the oracle
// (oracle/serving.py replay_online) re-derives it from the recorded decide / finish times.
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <deque>
#include <list>
#include <thread>
#include <vector>

#include "engine.h"
#include "serve.h"

namespace dp {
void infer_cold(dp_context* ctx, dp_model* m, const dp_plan* plan, int primary, int prim_rank,
                const int32_t* secondaries, int nsec, const int32_t* ids, int batch, int seq, void* out, void* pooled,
                cudaStream_t stream, dp_run_stats* stats);
int64_t plan_resident_bytes(const dp_model* m, const int8_t* method);
}  // namespace dp

extern "C" dp_status dp_infer_warm(dp_context* ctx, dp_model* m, int32_t dev, const int32_t* d_ids, int32_t batch,
                                   int32_t seq, void* d_out, void* d_pooled, void* stream, dp_run_stats* stats);
extern "C" dp_status dp_model_evict(dp_context* ctx, dp_model* m, int32_t dev);

namespace dp {

namespace {

struct Job {
  int req = -1;
  std::vector<int> victims;
};

struct Gpu {
  int dev = -1;
  cudaStream_t s = nullptr;
  cudaEvent_t done = nullptr;
  int32_t* ids = nullptr;
  void* y = nullptr;
  void* pooled = nullptr;
  int running = -1;        // request index
  bool running_cold = false;
  std::deque<Job> queue;   // decided, not started
  int64_t used = 0;        // resident bytes (logical, at decision time)
  std::list<int> lru;      // resident instances, front = least recently used
};

}  // namespace

void serve_live(dp_context* ctx, dp_model* const* models, int nmodels, const dp_trace_event* trace, int nreq,
                const dp_serve_opts& o, dp_serve_result* out) {
  DP_CHECK(ctx && models, DP_ERR_INVALID, "live serving needs a context and models");
  DP_CHECK(nmodels == o.ninstances, DP_ERR_INVALID, "live serving: one dp_model per instance");
  DP_CHECK(o.plans != nullptr, DP_ERR_INVALID, "live serving: plans missing");
  DP_CHECK(o.ngpu >= 1 && o.ngpu <= (int)ctx->devs.size(), DP_ERR_INVALID, "ngpu: 1 .. the context's devices");
  DP_CHECK(o.batch > 0 && o.seq > 0, DP_ERR_INVALID, "batch/seq");
  const int G = o.ngpu;
  for (int g = 0; g < G; ++g)
    for (int h = 0; h < g; ++h)
      DP_CHECK(ctx->devs[g] != ctx->devs[h], DP_ERR_INVALID, "live serving: the context's devices must be distinct");
  for (int i = 0; i < nmodels; ++i) {
    DP_CHECK(models[i] && o.plans[i], DP_ERR_INVALID, "NULL model / plan");
    DP_CHECK(o.plans[i]->k <= G, DP_ERR_INVALID, "a plan needs more GPUs than are served");
  }
  auto seq_of = [&](int inst) { return o.seq_of_model ? o.seq_of_model[o.model_of_instance[inst]] : o.seq; };
  int maxH = 0, max_seq = o.seq;
  for (int i = 0; i < nmodels; ++i) {
    maxH = std::max(maxH, models[i]->cfg.hidden);
    max_seq = std::max(max_seq, seq_of(i));
  }
  const int T = o.batch * max_seq;
  std::vector<int64_t> rbytes(nmodels);
  for (int i = 0; i < nmodels; ++i) {
    rbytes[i] = plan_resident_bytes(models[i], o.plans[i]->method);
    DP_CHECK(rbytes[i] <= o.per_gpu_budget_bytes, DP_ERR_INVALID, "an instance does not fit the per-GPU budget");
  }
  // per-GPU resources; token ids 3 + (t * 7919) % 997 (reproducible by the caller)
  std::vector<Gpu> gpu(G);
  auto cleanup = [&] {
    for (auto& q : gpu) {
      if (q.dev < 0) continue;
      cudaSetDevice(q.dev);
      if (q.s) cudaStreamSynchronize(q.s);
      if (q.ids) cudaFree(q.ids);
      if (q.y) cudaFree(q.y);
      if (q.pooled) cudaFree(q.pooled);
      if (q.done) cudaEventDestroy(q.done);
      if (q.s) cudaStreamDestroy(q.s);
    }
  };
  try {
    for (int g = 0; g < G; ++g) {
      Gpu& q = gpu[g];
      q.dev = ctx->devs[g];
      DP_CUDA(cudaSetDevice(q.dev));
      DP_CUDA(cudaStreamCreateWithFlags(&q.s, cudaStreamNonBlocking));
      DP_CUDA(cudaEventCreateWithFlags(&q.done, cudaEventDisableTiming));
      DP_CUDA(cudaMalloc(&q.ids, sizeof(int32_t) * T));
      DP_CUDA(cudaMalloc(&q.y, size_t(T) * maxH * 4));  // room for any storage dtype
      DP_CUDA(cudaMalloc(&q.pooled, size_t(o.batch) * maxH * 4));
      std::vector<int32_t> h(T);
      for (int t = 0; t < T; ++t) h[t] = 3 + (t * 7919) % 997;
      DP_CUDA(cudaMemcpy(q.ids, h.data(), sizeof(int32_t) * T, cudaMemcpyHostToDevice));
    }
    auto pick_secondaries = [&](int g, int k, int32_t* mask) {
      std::vector<int> cand;
      for (int j = 0; j < G; ++j)
        if (j != g) cand.push_back(j);
      auto load = [&](int j) { return (gpu[j].running >= 0 ? 1 : 0) + (int)gpu[j].queue.size(); };
      std::stable_sort(cand.begin(), cand.end(), [&](int a, int b) { return load(a) < load(b); });
      std::vector<int32_t> sec;
      for (int i = 0; i < k - 1; ++i) {
        sec.push_back(gpu[cand[i]].dev);
        *mask |= 1 << cand[i];
      }
      return sec;
    };
    auto start_job = [&](int g, const Job& j) {
      NvtxRange nv("serve start (evict + enqueue)");
      Gpu& q = gpu[g];
      const int r = j.req, inst = trace[r].instance;
      dp_model* m = models[inst];
      for (int v : j.victims) {
        if (models[v]->dev[q.dev].resident) {
          const dp_status st = dp_model_evict(ctx, models[v], q.dev);  // HBM back to the pool
          DP_CHECK(st == DP_OK, st, "eviction failed");
        }
      }
      DP_CUDA(cudaSetDevice(q.dev));
      void* pool = m->cfg.family == DP_FAMILY_GPT2 ? nullptr : q.pooled;
      if (out[r].cold) {
        const dp_plan* plan = o.plans[inst];
        int32_t mask = 0;
        auto sec = pick_secondaries(g, plan->k, &mask);
        out[r].sec_mask = mask;
        infer_cold(ctx, m, plan, q.dev, -1, sec.data(), (int)sec.size(), q.ids, o.batch, seq_of(inst), q.y, pool, q.s,
                   nullptr);
      } else {
        const dp_status st = dp_infer_warm(ctx, m, q.dev, q.ids, o.batch, seq_of(inst), q.y, pool, q.s, nullptr);
        DP_CHECK(st == DP_OK, st, "warm inference failed");
      }
      DP_CUDA(cudaEventRecord(q.done, q.s));
      q.running = r;
      q.running_cold = out[r].cold != 0;
    };
    // live serving starts from every instance non-resident on the served GPUs
    for (int g = 0; g < G; ++g)
      for (int i = 0; i < nmodels; ++i)
        if (models[i]->dev[gpu[g].dev].resident)
          DP_CHECK(dp_model_evict(ctx, models[i], gpu[g].dev) == DP_OK, DP_ERR_CUDA, "eviction failed");
    // pre-warm: every instance once on every GPU (workspace, first-use host costs), then evicted
    // -- the trace measures serving, not first-touch allocation (graphs are captured on a key's
    // second use, so instances that keep a pool block capture during the trace)
    if (!o.no_prewarm) {
      for (int g = 0; g < G; ++g) {
        for (int i = 0; i < nmodels; ++i) {
          dp_model* m = models[i];
          const dp_plan* plan = o.plans[i];
          DP_CUDA(cudaSetDevice(gpu[g].dev));
          std::vector<int32_t> sec;
          for (int k = 1; k < plan->k; ++k) sec.push_back(gpu[(g + k) % G].dev);
          void* pool = m->cfg.family == DP_FAMILY_GPT2 ? nullptr : gpu[g].pooled;
          infer_cold(ctx, m, plan, gpu[g].dev, -1, sec.data(), (int)sec.size(), gpu[g].ids, o.batch, seq_of(i),
                     gpu[g].y, pool, gpu[g].s, nullptr);
          const dp_status st = dp_infer_warm(ctx, m, gpu[g].dev, gpu[g].ids, o.batch, seq_of(i), gpu[g].y, pool,
                                             gpu[g].s, nullptr);
          DP_CHECK(st == DP_OK, st, "warm inference failed");
          DP_CHECK(dp_model_evict(ctx, m, gpu[g].dev) == DP_OK, DP_ERR_CUDA, "eviction failed");
        }
      }
    }
    for (int g = 0; g < G; ++g) {
      DP_CUDA(cudaSetDevice(gpu[g].dev));
      DP_CUDA(cudaDeviceSynchronize());
    }
    std::vector<int> where(nmodels, -1);  // GPU the instance is (becoming) resident on
    std::vector<int> pending(nmodels, 0); // decided, not yet observed complete
    using clk = std::chrono::steady_clock;
    const clk::time_point t0 = clk::now() + std::chrono::milliseconds(5);
    auto since = [&](clk::time_point t) { return (int64_t)std::chrono::duration_cast<std::chrono::nanoseconds>(t - t0).count(); };
    int next = 0, done = 0;
    while (done < nreq) {
      const int64_t now = since(clk::now());
      // (1) completions observed now
      for (int g = 0; g < G; ++g) {
        Gpu& q = gpu[g];
        if (q.running < 0) continue;
        DP_CUDA(cudaSetDevice(q.dev));
        const cudaError_t e = cudaEventQuery(q.done);
        if (e == cudaErrorNotReady) continue;
        DP_CUDA(e);
        out[q.running].finish_ns = now;
        --pending[trace[q.running].instance];
        q.running = -1;
        ++done;
      }
      // (2) arrivals up to now, decided on the observed state
      while (next < nreq && trace[next].arrival_ns <= now) {
        const int r = next++;
        NvtxRange nv("serve decide");
        const int inst = trace[r].instance;
        DP_CHECK(inst >= 0 && inst < nmodels, DP_ERR_INVALID, "trace instance out of range");
        DP_CHECK(r == 0 || trace[r].arrival_ns >= trace[r - 1].arrival_ns, DP_ERR_INVALID,
                 "trace must be sorted by arrival");
        dp_serve_result& res = out[r];
        res = dp_serve_result{};
        res.decide_ns = now;
        Job j;
        j.req = r;
        int g = where[inst];
        if (g >= 0) {
          res.cold = 0;
          gpu[g].lru.remove(inst);
        } else {
          g = 0;
          auto outstanding = [&](int x) { return (gpu[x].running >= 0 ? 1 : 0) + (int)gpu[x].queue.size(); };
          for (int x = 1; x < G; ++x)
            if (outstanding(x) < outstanding(g)) g = x;
          gpu[g].used += rbytes[inst];
          where[inst] = g;
          res.cold = 1;
        }
        // while the GPU is over its budget: evict the least recently used resident instance other
        // than this one with no outstanding request; if none can go, it stays over budget
        // until a later decision on this GPU can evict
        {
          Gpu& q = gpu[g];
          for (auto it = q.lru.begin(); it != q.lru.end() && q.used > o.per_gpu_budget_bytes;) {
            const int v = *it;
            if (v == inst || pending[v] > 0) {
              ++it;
              continue;
            }
            it = q.lru.erase(it);
            q.used -= rbytes[v];
            where[v] = -1;
            j.victims.push_back(v);
          }
          res.nevicted = (int32_t)j.victims.size();
        }
        gpu[g].lru.push_back(inst);
        res.gpu = g;
        ++pending[inst];
        gpu[g].queue.push_back(std::move(j));
      }
      // (3) idle GPUs start their next request
      for (int g = 0; g < G; ++g) {
        Gpu& q = gpu[g];
        if (q.running >= 0 || q.queue.empty()) continue;
        Job j = std::move(q.queue.front());
        q.queue.pop_front();
        out[j.req].start_ns = since(clk::now());
        start_job(g, j);
      }
      if (done < nreq) {
        // OS sleeps wake ~50-60 us late (timer slack): sleep only while nothing can happen for
        // longer than that, otherwise spin (the dispatcher owns one host core)
        bool busy = false;
        for (auto& q : gpu) busy |= q.running >= 0;
        if (!busy && next < nreq) {
          const auto wake = t0 + std::chrono::nanoseconds(trace[next].arrival_ns) - std::chrono::microseconds(200);
          if (wake > clk::now()) std::this_thread::sleep_until(wake);
        }
      }
    }
  } catch (...) {
    cleanup();
    throw;
  }
  cleanup();
}

}  // namespace dp
