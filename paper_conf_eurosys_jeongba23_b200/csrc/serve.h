#pragma once
#include <vector>

#include "common.h"

namespace dp {
// Dispatch decisions (gpu, cold, evictions) and replayed start/finish times.
void serve_decide(const dp_serve_opts& o, const dp_trace_event* trace, int nreq, dp_serve_result* out,
                  std::vector<int64_t>* unused);
// Execute decided requests on the GPUs at their wall-clock arrival times; overwrites
// start_ns / finish_ns with measured times.
void serve_live(dp_context* ctx, dp_model* const* models, int nmodels, const dp_trace_event* trace, int nreq,
                const dp_serve_opts& o, dp_serve_result* out);
}  // namespace dp
