#pragma once
#include <vector>

#include "common.h"

namespace dp {
// Dispatch decisions (gpu, cold, evictions) and replayed start/finish times.
void serve_decide(const dp_serve_opts& o, const dp_trace_event* trace, int nreq, dp_serve_result* out,
                  std::vector<int64_t>* unused);
// Online serving on the GPUs: requests decided at their wall-clock arrival on the observed
// state, executed one per GPU at a time, real evictions (serve_live.cu).
void serve_live(dp_context* ctx, dp_model* const* models, int nmodels, const dp_trace_event* trace, int nreq,
                const dp_serve_opts& o, dp_serve_result* out);
}  // namespace dp
