// Internal kernel launchers (host side).  All take a cudaStream_t and return after enqueue.
#pragma once
#include <cuda_runtime.h>
#include <cstdint>

namespace dp {

// Epilogue activations (dp_linear's `act`).
enum Act { ACT_NONE = 0, ACT_GELU_ERF = 1, ACT_GELU_TANH = 2, ACT_TANH = 3 };
// Linear epilogue I/O precision (the pre-LN GPT-2 residual stream is kept in fp32).
enum Io { IO_RES_F32 = 1, IO_OUT_F32 = 2 };

// K1: fused embedding gather (+ LayerNorm) -- SURVEY §8(a) a10.  Table pointers may be
// host-mapped (direct-host-access).  ln_g == nullptr -> no LN (GPT-2).
void launch_embed(int dtype, const int32_t* ids, int ntok, int seq, int pos_off, const void* word, const void* pos,
                  const void* type, const void* ln_g, const void* ln_b, int H, float eps, void* out, bool out_f32,
                  cudaStream_t s, void* out32 = nullptr,  // out32: optional fp32 copy of the LN output
                  int vocab = 0,                          // > 0: ids are clamped to [0, vocab) (engine path)
                  bool shared_host = false);  // type / gamma / beta host-mapped: read once per cluster

// K4: y = LN(x (+ r)) * g + b; g/b may be host-mapped.
void launch_layernorm(int dtype, const void* x, const void* r, const void* g, const void* b, void* y, int rows,
                      int n, float eps, bool in_f32, cudaStream_t s, void* y32 = nullptr,  // y32: optional fp32 copy
                      bool gb_host = false);  // gamma/beta host-mapped (DHA): read once per launch (cluster)

// K3: skinny linear reading W exactly once (W may be host-mapped) -- a11.
void launch_skinny_linear(int dtype, const void* x, int ldx, const void* w, const void* bias, const void* res,
                          int ldr, void* y, int ldy, int M, int N, int K, int act, int io, cudaStream_t s);

// K5: attention core (mma.sync flash attention, d = 64).
void launch_attention(int dtype, const void* qkv, int ldqkv, void* ctx, int batch, int seq, int H, int heads,
                      bool causal, cudaStream_t s, int tc_mode = 0);  // tc_mode: opts.attention_tc

// K5t: attention on tcgen05 (attn_tc.cu): S and O in TMEM, the softmax row per thread.
bool attention_tc_supported(int ldqkv, int H, int heads, const void* qkv);
void launch_attention_tc(int dtype, const void* qkv, int ldqkv, void* ctx, int batch, int seq, int H, int heads,
                         bool causal, cudaStream_t s);

// K2: resident tcgen05/TMA GEMM -- a12.  W must be device memory.
struct GemmPlan;  // cached tensor map for a weight
bool gemm_tc_supported(int N, int K);
void launch_gemm_tc(int dtype, const void* x, int ldx, const void* w, const void* bias, const void* res, int ldr,
                    void* y, int ldy, int M, int N, int K, int act, int io, int bn_hint, cudaStream_t s,
                    int sp_hint = 0);
// bn_hint: 0 = the cost model's tile, > 0 one CTA per 128 x bn_hint tile, < 0 a CTA pair per
// 256 x -bn_hint tile; sp_hint > 0 forces that many K splits (single-CTA tiles only).
// ngroups (1..3) weights sharing X; group i writes y at column offset ycol[i].
void launch_gemm_tc_group(int dtype, const void* x, int ldx, int ngroups, const void* const* w,
                          const void* const* bias, const long long* ycol, const void* res, int ldr, void* y, int ldy,
                          int M, int N, int K, int act, int io, int bn_hint, cudaStream_t s, int sp_hint = 0);

// fp32 storage (DP_FP32, kernels_f32.cu): CUDA-core kernels with the same contracts; the
// launchers above dispatch to them when dtype == DP_FP32 (all activations are then fp32).
void launch_embed_f32(const int32_t* ids, int ntok, int seq, int pos_off, const void* word, const void* pos,
                      const void* type, const void* g, const void* b, int H, float eps, void* out, void* out32,
                      int vocab, cudaStream_t s);
void launch_layernorm_f32(const void* x, const void* r, const void* g, const void* b, void* y, int rows, int n,
                          float eps, cudaStream_t s, void* y32);
void launch_linear_f32(const void* x, int ldx, const void* w, const void* bias, const void* res, int ldr, void* y,
                       int ldy, int M, int N, int K, int act, cudaStream_t s);
void launch_attention_f32(const void* qkv, int ldqkv, void* ctx, int batch, int seq, int H, int heads, bool causal,
                          cudaStream_t s);

// Scratch kernels
void launch_l2_flush(void* buf, size_t bytes, cudaStream_t s);
void launch_spin(long long cycles, cudaStream_t s);
// Trace: one thread writes %globaltimer (ns) to *slot when the stream reaches it.
void launch_timestamp(uint64_t* slot, cudaStream_t s);

}  // namespace dp
