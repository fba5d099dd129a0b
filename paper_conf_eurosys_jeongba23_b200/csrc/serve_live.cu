// Live execution of the serving decisions (serve.cpp) on real GPUs: one worker thread per
// GPU runs its requests in dispatch order, each no earlier than its wall-clock arrival,
// with real cold starts (dp_infer_cold under the instance's plan) and warm inferences.
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <atomic>
#include <mutex>
#include <thread>
#include <vector>

#include "engine.h"
#include "serve.h"

namespace dp {
void infer_cold(dp_context* ctx, dp_model* m, const dp_plan* plan, int primary, int prim_rank,
                const int32_t* secondaries, int nsec, const int32_t* ids, int batch, int seq, void* out, void* pooled,
                cudaStream_t stream, dp_run_stats* stats);
}

extern "C" dp_status dp_infer_warm(dp_context* ctx, dp_model* m, int32_t dev, const int32_t* d_ids, int32_t batch,
                                   int32_t seq, void* d_out, void* d_pooled, void* stream, dp_run_stats* stats);

namespace dp {

void serve_live(dp_context* ctx, dp_model* const* models, int nmodels, const dp_trace_event* trace, int nreq,
                const dp_serve_opts& o, dp_serve_result* out) {
  DP_CHECK(ctx && models, DP_ERR_INVALID, "live serving needs a context and models");
  DP_CHECK(nmodels == o.ninstances, DP_ERR_INVALID, "live serving: one dp_model per instance");
  DP_CHECK(o.plans != nullptr, DP_ERR_INVALID, "live serving: plans missing");
  DP_CHECK(o.ngpu <= (int)ctx->devs.size(), DP_ERR_INVALID, "more GPUs than the context has");
  DP_CHECK(o.batch > 0 && o.seq > 0, DP_ERR_INVALID, "batch/seq");
  const int G = o.ngpu;
  // victims per request: replay the LRU bookkeeping to learn WHICH instances to evict
  std::vector<std::vector<int>> victims(nreq);
  {
    std::vector<int64_t> used(G, 0);
    std::vector<std::vector<int>> lru(G);
    std::vector<int> where(o.ninstances, -1);
    for (int r = 0; r < nreq; ++r) {
      const int inst = trace[r].instance, g = out[r].gpu;
      if (out[r].cold) {
        for (int k = 0; k < out[r].nevicted; ++k) {
          const int v = lru[g].front();
          lru[g].erase(lru[g].begin());
          used[g] -= o.resident_bytes[o.model_of_instance[v]];
          where[v] = -1;
          victims[r].push_back(v);
        }
        where[inst] = g;
      } else {
        lru[g].erase(std::find(lru[g].begin(), lru[g].end(), inst));
      }
      lru[g].push_back(inst);
    }
  }
  int maxH = 0;
  for (int i = 0; i < nmodels; ++i) maxH = std::max(maxH, models[i]->cfg.hidden);
  auto seq_of = [&](int inst) { return o.seq_of_model ? o.seq_of_model[o.model_of_instance[inst]] : o.seq; };
  int max_seq = o.seq;
  for (int i = 0; i < o.ninstances; ++i) max_seq = std::max(max_seq, seq_of(i));
  const int T = o.batch * max_seq;
  std::vector<std::vector<int>> queue(G);
  for (int r = 0; r < nreq; ++r) queue[out[r].gpu].push_back(r);
  // Workers first pre-warm every instance they will serve (HBM slots, workspace, captured
  // graphs: one cold + one warm run, then evict), so the timed trace measures serving, not
  // first-touch allocation.  The trace clock t0 starts when every worker is ready.
  std::atomic<int> ready{0};
  std::atomic<bool> go{false};
  std::chrono::steady_clock::time_point t0;
  std::vector<std::string> errors(G);
  std::mutex enqueue_mu;  // the context's stream/event/slot bookkeeping is not thread-safe
  std::vector<std::thread> workers;
  for (int g = 0; g < G; ++g) {
    workers.emplace_back([&, g] {
      try {
        const int dev = ctx->devs[g];
        DP_CUDA(cudaSetDevice(dev));
        cudaStream_t s;
        DP_CUDA(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
        int32_t* ids;
        void *y, *pooled;
        DP_CUDA(cudaMalloc(&ids, sizeof(int32_t) * T));
        DP_CUDA(cudaMalloc(&y, size_t(T) * maxH * 4));  // room for any storage dtype
        DP_CUDA(cudaMalloc(&pooled, size_t(o.batch) * maxH * 4));
        std::vector<int32_t> h(T);
        for (int t = 0; t < T; ++t) h[t] = 3 + (t * 7919) % 997;
        DP_CUDA(cudaMemcpy(ids, h.data(), sizeof(int32_t) * T, cudaMemcpyHostToDevice));
        {
          std::vector<char> seen(nmodels, 0);
          for (int r : queue[g]) {
            const int inst = trace[r].instance;
            if (seen[inst]) continue;
            seen[inst] = 1;
            dp_model* m = models[inst];
            void* pool = m->cfg.family == DP_FAMILY_GPT2 ? nullptr : pooled;
            const dp_plan* plan = o.plans[inst];
            std::vector<int32_t> sec;
            for (int k = 1; k < plan->k; ++k) sec.push_back(ctx->devs[(g + k) % G]);
            std::lock_guard<std::mutex> lk(enqueue_mu);
            m->dev[dev].resident = false;
            infer_cold(ctx, m, plan, dev, -1, sec.data(), (int)sec.size(), ids, o.batch, seq_of(inst), y, pool, s, nullptr);
            dp_status st = dp_infer_warm(ctx, m, dev, ids, o.batch, seq_of(inst), y, pool, s, nullptr);
            DP_CHECK(st == DP_OK, st, "warm inference failed");
            DP_CUDA(cudaStreamSynchronize(s));
            m->dev[dev].resident = false;
          }
        }
        ready.fetch_add(1);
        while (!go.load()) std::this_thread::yield();
        for (int r : queue[g]) {
          const int inst = trace[r].instance;
          dp_model* m = models[inst];
          std::this_thread::sleep_until(t0 + std::chrono::nanoseconds(trace[r].arrival_ns));
          const auto start = std::chrono::steady_clock::now();
          for (int v : victims[r]) {
            if (models[v]->dev[dev].resident) {
              DP_CUDA(cudaStreamSynchronize(s));
              models[v]->dev[dev].resident = false;
            }
          }
          void* pool = m->cfg.family == DP_FAMILY_GPT2 ? nullptr : pooled;
          if (out[r].cold) {
            const dp_plan* plan = o.plans[inst];
            std::vector<int32_t> sec;
            for (int k = 1; k < plan->k; ++k) sec.push_back(ctx->devs[(g + k) % G]);
            if (m->dev[dev].resident) m->dev[dev].resident = false;  // defensive: decisions say cold
            std::lock_guard<std::mutex> lk(enqueue_mu);
            infer_cold(ctx, m, plan, dev, -1, sec.data(), (int)sec.size(), ids, o.batch, seq_of(inst), y, pool, s, nullptr);
          } else {
            std::lock_guard<std::mutex> lk(enqueue_mu);
            dp_status st = dp_infer_warm(ctx, m, dev, ids, o.batch, seq_of(inst), y, pool, s, nullptr);
            DP_CHECK(st == DP_OK, st, "warm inference failed");
          }
          DP_CUDA(cudaStreamSynchronize(s));
          const auto fin = std::chrono::steady_clock::now();
          out[r].start_ns = std::chrono::duration_cast<std::chrono::nanoseconds>(start - t0).count();
          out[r].finish_ns = std::chrono::duration_cast<std::chrono::nanoseconds>(fin - t0).count();
        }
        cudaFree(ids);
        cudaFree(y);
        cudaFree(pooled);
        cudaStreamDestroy(s);
      } catch (const std::exception& e) {
        errors[g] = e.what();
      }
    });
  }
  while (ready.load() < G) {
    bool failed = false;
    for (int g = 0; g < G; ++g) failed |= !errors[g].empty();
    if (failed) break;
    std::this_thread::sleep_for(std::chrono::milliseconds(1));
  }
  t0 = std::chrono::steady_clock::now() + std::chrono::milliseconds(20);
  go.store(true);
  for (auto& w : workers) w.join();
  for (int g = 0; g < G; ++g) DP_CHECK(errors[g].empty(), DP_ERR_CUDA, "serving worker " + std::to_string(g) + ": " + errors[g]);
}

}  // namespace dp
