// Internal helpers shared by the library's translation units (not part of the ABI).
#pragma once
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <stdexcept>
#include <string>

#include <nvtx3/nvToolsExt.h>

#include "deepplan.h"

namespace dp {

// An error that carries its dp_status across internal layers; converted at the ABI edge.
struct Error : std::runtime_error {
  dp_status code;
  Error(dp_status c, const std::string& m) : std::runtime_error(m), code(c) {}
};

void set_last_error(const std::string& msg);

[[noreturn]] inline void fail(dp_status code, const std::string& msg) { throw Error(code, msg); }

#define DP_CUDA(x)                                                                              \
  do {                                                                                          \
    cudaError_t e__ = (x);                                                                      \
    if (e__ != cudaSuccess)                                                                     \
      ::dp::fail(DP_ERR_CUDA, std::string(#x) + " failed: " + cudaGetErrorString(e__) + " at " + \
                                  __FILE__ + ":" + std::to_string(__LINE__));                   \
  } while (0)

#define DP_CHECK(cond, code, msg)                            \
  do {                                                       \
    if (!(cond)) ::dp::fail((code), std::string(msg));       \
  } while (0)

// NVTX range for the host-side phases (visible in nsys / ncu timelines): cold / warm inference,
// the enqueue of each link's transfers, the forward's kernels, profiling, serving decisions.
struct NvtxRange {
  explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
  ~NvtxRange() { nvtxRangePop(); }
  NvtxRange(const NvtxRange&) = delete;
  NvtxRange& operator=(const NvtxRange&) = delete;
};

// Run body, translating exceptions into a dp_status + last error.
template <class F>
dp_status guard(F&& body) {
  try {
    body();
    return DP_OK;
  } catch (const Error& e) {
    set_last_error(e.what());
    return e.code;
  } catch (const std::bad_alloc&) {
    set_last_error("host allocation failed");
    return DP_ERR_OOM;
  } catch (const std::exception& e) {
    set_last_error(e.what());
    return DP_ERR_INVALID;
  }
}

// Experiment knobs (tools/ sweeps and A/B runs) read from the environment ONLY in instrumented
// builds (DP_NVCC_EXTRA=-DDP_INSTRUMENT); the release library always uses `dflt`, so no
// environment variable can change what it computes or launches.
inline int experiment_env(const char* name, int dflt) {
#ifdef DP_INSTRUMENT
  const char* e = std::getenv(name);
  return e ? std::atoi(e) : dflt;
#else
  (void)name;
  return dflt;
#endif
}

inline int dtype_bytes(int dtype) { return dtype == DP_FP32 ? 4 : 2; }  // storage element bytes

}  // namespace dp
