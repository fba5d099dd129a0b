// C-ABI kernel entry points (parity-test hooks) and pinned host allocation.
// They launch exactly the kernels the executor launches.
#include <cuda_runtime.h>

#include "common.h"
#include "kernels.h"

using namespace dp;

extern "C" dp_status dp_host_alloc(int64_t bytes, void** out) {
  return guard([&] {
    DP_CHECK(out && bytes > 0, DP_ERR_INVALID, "bad arguments");
    cudaError_t e = cudaHostAlloc(out, bytes, cudaHostAllocPortable | cudaHostAllocMapped);
    if (e != cudaSuccess) fail(DP_ERR_OOM, std::string("cudaHostAlloc failed: ") + cudaGetErrorString(e));
  });
}

extern "C" dp_status dp_host_free(void* p) {
  return guard([&] {
    if (p) DP_CUDA(cudaFreeHost(p));
  });
}

static bool is_host_ptr(const void* p) {
  if (!p) return false;
  cudaPointerAttributes at;
  if (cudaPointerGetAttributes(&at, p) != cudaSuccess) {
    cudaGetLastError();
    return true;  // unregistered host memory
  }
  return at.type == cudaMemoryTypeHost || at.type == cudaMemoryTypeUnregistered;
}

static void check_dtype(int32_t dtype) {
  DP_CHECK(dtype == DP_FP16 || dtype == DP_BF16 || dtype == DP_FP32, DP_ERR_UNSUPPORTED,
           "dtype must be DP_FP16, DP_BF16 or DP_FP32");
}

extern "C" dp_status dp_embed(const int32_t* d_ids, int32_t ntok, int32_t seq, int32_t pos_offset, const void* word,
                              const void* pos, const void* type, const void* ln_g, const void* ln_b, int32_t hidden,
                              double eps, int32_t dtype, int32_t out_f32, void* d_out, void* stream) {
  return guard([&] {
    check_dtype(dtype);
    DP_CHECK(d_ids && word && pos && d_out, DP_ERR_INVALID, "NULL pointer");
    DP_CHECK((ln_g == nullptr) == (ln_b == nullptr), DP_ERR_INVALID, "ln_g and ln_b must both be set or NULL");
    launch_embed(dtype, d_ids, ntok, seq, pos_offset, word, pos, type, ln_g, ln_b, hidden, (float)eps, d_out,
                 out_f32 != 0, (cudaStream_t)stream, nullptr, 0, is_host_ptr(type) || is_host_ptr(ln_g));
  });
}

extern "C" dp_status dp_linear(const void* x, int32_t ldx, const void* w, const void* b, const void* residual,
                               int32_t ldr, void* y, int32_t ldy, int32_t M, int32_t N, int32_t K, int32_t act,
                               int32_t path, int32_t dtype, int32_t io, void* stream) {
  return guard([&] {
    check_dtype(dtype);
    DP_CHECK(x && w && y, DP_ERR_INVALID, "NULL pointer");
    DP_CHECK(M >= 0 && N > 0 && K > 0 && ldx >= K && ldy >= N && (!residual || ldr >= N), DP_ERR_INVALID,
             "bad shapes / strides");
    DP_CHECK(act >= 0 && act <= 3, DP_ERR_INVALID, "act must be 0..3");
    if (path == 0) {
      DP_CHECK(dtype != DP_FP32, DP_ERR_UNSUPPORTED, "the tcgen05 path has no fp32 kind: use path 1 for fp32");
      cudaPointerAttributes at;
      DP_CUDA(cudaPointerGetAttributes(&at, w));
      DP_CHECK(at.type == cudaMemoryTypeDevice, DP_ERR_INVALID, "the tcgen05 path needs W in device memory");
      launch_gemm_tc(dtype, x, ldx, w, b, residual, ldr, y, ldy, M, N, K, act, io, 0, (cudaStream_t)stream);
    } else if (path == 1) {
      launch_skinny_linear(dtype, x, ldx, w, b, residual, ldr, y, ldy, M, N, K, act, io, (cudaStream_t)stream);
    } else {
      fail(DP_ERR_INVALID, "path must be 0 (tcgen05) or 1 (skinny/DHA)");
    }
  });
}

extern "C" dp_status dp_gemm_tc(const void* x, int32_t ldx, const void* w, const void* b, const void* residual,
                                int32_t ldr, void* y, int32_t ldy, int32_t M, int32_t N, int32_t K, int32_t act,
                                int32_t dtype, int32_t io, int32_t bn, int32_t split, void* stream) {
  return guard([&] {
    check_dtype(dtype);
    DP_CHECK(dtype != DP_FP32, DP_ERR_UNSUPPORTED, "the tcgen05 path has no fp32 kind");
    DP_CHECK(x && w && y, DP_ERR_INVALID, "NULL pointer");
    DP_CHECK(M >= 0 && N > 0 && K > 0 && ldx >= K && ldy >= N && (!residual || ldr >= N), DP_ERR_INVALID,
             "bad shapes / strides");
    DP_CHECK(act >= 0 && act <= 3, DP_ERR_INVALID, "act must be 0..3");
    DP_CHECK(bn == 0 || bn == 32 || bn == 64 || bn == 96 || bn == 128 || bn == 192 || bn == 256 || bn == -64 ||
                 bn == -128 || bn == -192 || bn == -256,
             DP_ERR_INVALID, "bn must be 0, 32/64/96/128/192/256 or -64/-128/-192/-256");
    DP_CHECK(bn >= 0 || N % 256 == 0, DP_ERR_INVALID, "a CTA pair needs N % 256 == 0");
    DP_CHECK(split == 0 || split == 1 ||
                 ((split & (split - 1)) == 0 && split <= 8 && bn > 0 && bn <= 128 && split <= K / 64),
             DP_ERR_INVALID, "split must be 0, 1, or 2/4/8 <= K/64 with a single-CTA bn <= 128");
    cudaPointerAttributes at;
    DP_CUDA(cudaPointerGetAttributes(&at, w));
    DP_CHECK(at.type == cudaMemoryTypeDevice, DP_ERR_INVALID, "the tcgen05 path needs W in device memory");
    launch_gemm_tc(dtype, x, ldx, w, b, residual, ldr, y, ldy, M, N, K, act, io, bn, (cudaStream_t)stream, split);
  });
}

extern "C" dp_status dp_layernorm(const void* x, const void* r, const void* g, const void* b, void* y, int32_t rows,
                                  int32_t n, double eps, int32_t dtype, int32_t x_f32, void* stream) {
  return guard([&] {
    check_dtype(dtype);
    DP_CHECK(x && g && b && y && rows >= 0, DP_ERR_INVALID, "bad arguments");
    launch_layernorm(dtype, x, r, g, b, y, rows, n, (float)eps, x_f32 != 0, (cudaStream_t)stream, nullptr,
                     is_host_ptr(g));
  });
}

extern "C" dp_status dp_attention_tc(const void* qkv, int32_t ldqkv, void* ctx_out, int32_t batch, int32_t seq,
                                     int32_t hidden, int32_t heads, int32_t causal, int32_t dtype, void* stream) {
  return guard([&] {
    DP_CHECK(dtype == DP_FP16 || dtype == DP_BF16, DP_ERR_UNSUPPORTED, "tcgen05 attention: fp16 / bf16");
    DP_CHECK(qkv && ctx_out && ldqkv >= 3 * hidden && attention_tc_supported(ldqkv, hidden, heads, qkv), DP_ERR_INVALID,
             "bad arguments (head dim 64, 16-byte aligned rows)");
    if (batch > 0 && seq > 0)
      launch_attention_tc(dtype, qkv, ldqkv, ctx_out, batch, seq, hidden, heads, causal != 0, (cudaStream_t)stream);
  });
}

extern "C" dp_status dp_attention(const void* qkv, int32_t ldqkv, void* ctx_out, int32_t batch, int32_t seq,
                                  int32_t hidden, int32_t heads, int32_t causal, int32_t dtype, void* stream) {
  return guard([&] {
    check_dtype(dtype);
    DP_CHECK(qkv && ctx_out && ldqkv >= 3 * hidden, DP_ERR_INVALID, "bad arguments");
    launch_attention(dtype, qkv, ldqkv, ctx_out, batch, seq, hidden, heads, causal != 0, (cudaStream_t)stream);
  });
}
