// K6: persistent layer-program kernel (persist.cu) -- host interface.
#pragma once
#include <cuda_runtime.h>

#include <memory>

#include "model.h"

namespace dp {

struct PersistProgram;

// True when every layer unit of the plan is resident (method DP_LOAD) and the shapes fit K6
// (hidden <= 1024 and a multiple of 128, ffn a multiple of 128, head dim 64, > 16 tokens).
bool persist_supported(const dp_model* m, const int8_t* method, int tokens);
// The op list, tensor maps and partial-sum workspace for (model, device, batch, seq); the maps
// capture the HBM slots and the device workspace (ensure_workspace first).
std::shared_ptr<PersistProgram> build_persist_program(dp_model* m, int dev, int batch, int seq);
// One cooperative launch (grid = #SMs) running every layer; the last op writes final_out.
void launch_persist(const PersistProgram& p, void* final_out, cudaStream_t s);
int persist_num_ops(const PersistProgram& p);

}  // namespace dp
