// Kernel launch with optional programmatic dependent launch (PDL).
//
// Inside a forward pass consecutive kernels on the execution stream are chained with PDL:
// a kernel starts its prologue (barrier init, TMEM alloc, and -- for weights, which never
// depend on the previous kernel -- its first weight tiles) while its predecessor drains,
// then `griddepcontrol.wait`s before touching activations.  Right after an event wait
// (a layer that just landed) the next launch is a plain stream-ordered one.
#pragma once
#include <cuda_runtime.h>

#include <atomic>
#include <cstdlib>

#include "common.h"

namespace dp {

// Engine-controlled state (thread-local: one host thread drives a context at a time).
struct PdlState {
  bool enabled = false;     // inside run_forward with PDL allowed
  bool block_next = true;   // the next launch must not overlap its predecessor
};
PdlState& pdl_state();

inline bool take_pdl() {
  PdlState& s = pdl_state();
  const bool r = s.enabled && !s.block_next;
  s.block_next = false;
  return r;
}

template <class... KArgs, class... Args>
inline void launch_kernel(void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t s,
                          Args&&... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  if (take_pdl()) {
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
  }
  DP_CUDA(cudaLaunchKernelEx(&cfg, kern, static_cast<KArgs>(args)...));
}

// The same with thread-block clusters of shape `cluster` (1 x 1 x 1: none).
template <class... KArgs, class... Args>
inline void launch_kernel_cluster(void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem, dim3 cluster,
                                  cudaStream_t s, Args&&... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute at[2];
  int n = 0;
  if (take_pdl()) {
    at[n].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[n++].val.programmaticStreamSerializationAllowed = 1;
  }
  if (cluster.x * cluster.y * cluster.z > 1) {
    at[n].id = cudaLaunchAttributeClusterDimension;
    at[n].val.clusterDim.x = cluster.x;
    at[n].val.clusterDim.y = cluster.y;
    at[n++].val.clusterDim.z = cluster.z;
  }
  cfg.attrs = n ? at : nullptr;
  cfg.numAttrs = n;
  DP_CUDA(cudaLaunchKernelEx(&cfg, kern, static_cast<KArgs>(args)...));
}

// Function attributes (dynamic shared memory size, non-portable clusters) are per device: a
// call site sets them the first time it runs on each device.  `seen` is the call site's
// static bit mask of devices (atomic: the serving harness drives devices from several threads).
inline bool first_on_device(std::atomic<unsigned>& seen) {
  int d = 0;
  DP_CUDA(cudaGetDevice(&d));
  const unsigned bit = 1u << d;
  return (seen.fetch_or(bit) & bit) == 0;
}

// Timing ablation (tools/ablate.py only, instrumented builds: DP_NVCC_EXTRA=-DDP_INSTRUMENT):
// DP_ABLATE is a bit mask of kernel families whose launches are skipped -- 1 attention,
// 2 LayerNorm, 4 resident GEMM (query, key and value grouped or not), 8 skinny linear / GEMV.
// Outputs are garbage; the warm forward's time without a family is what its share of the
// chain is.  The release library compiles it to 0 (no environment variable can drop kernels).
inline int ablate_mask() {
#ifdef DP_INSTRUMENT
  static const int m = [] {
    const char* e = std::getenv("DP_ABLATE");
    return e ? std::atoi(e) : 0;
  }();
  return m;
#else
  return 0;
#endif
}

// Device side: no-ops when the grid was not launched with PDL.
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }

}  // namespace dp
