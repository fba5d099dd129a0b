// linkprobe: measures the host-link and on-GPU rates that bound the cold-start path
// (SURVEY §7 step 0). Standalone; prints one JSON object. Not part of the product path.
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/linkprobe tools/linkprobe.cu
//
// What it measures (all device-timed with CUDA events on the issuing stream):
//   h2d_pinned[size]     cudaMemcpyAsync H2D from cudaHostAlloc(Portable|Mapped) memory
//   h2d_wc[size]         same from write-combined pinned memory
//   d2h_pinned[size]     D2H into pinned memory
//   zc_read[cfg]         SM zero-copy read of mapped host memory (16 B loads), sum to HBM
//   zc_copy              SM zero-copy host->HBM copy kernel (ld.v4 host / st.v4 HBM)
//   zc_gather            S random rows of H*2 bytes (the DHA embedding access pattern)
//   h2d_plus_zc          concurrent H2D + zero-copy read (link sharing)
//   small_copy_us        latency of a small H2D (3 KB) and of event record / stream wait
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdlib>
#include <cstdint>
#include <vector>
#include <algorithm>
#include <string>
#include <chrono>
#include <cstring>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { \
  fprintf(stderr, "CUDA %s at %s:%d: %s\n", #x, __FILE__, __LINE__, cudaGetErrorString(e)); exit(1);} } while (0)

__global__ void zc_read_kernel(const int4* __restrict__ src, size_t n16, int4* out) {
  int4 acc = make_int4(0, 0, 0, 0);
  size_t stride = (size_t)gridDim.x * blockDim.x;
  size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  for (; i + 3 * stride < n16; i += 4 * stride) {
    int4 a = src[i], b = src[i + stride], c = src[i + 2 * stride], d = src[i + 3 * stride];
    acc.x ^= a.x ^ b.x ^ c.x ^ d.x; acc.y ^= a.y ^ b.y ^ c.y ^ d.y;
    acc.z ^= a.z ^ b.z ^ c.z ^ d.z; acc.w ^= a.w ^ b.w ^ c.w ^ d.w;
  }
  for (; i < n16; i += stride) { int4 a = src[i]; acc.x ^= a.x; acc.y ^= a.y; acc.z ^= a.z; acc.w ^= a.w; }
  if ((acc.x ^ acc.y ^ acc.z ^ acc.w) == 0x7fffffff) out[0] = acc;
}

__global__ void zc_copy_kernel(const int4* __restrict__ src, int4* __restrict__ dst, size_t n16) {
  size_t stride = (size_t)gridDim.x * blockDim.x;
  size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  for (; i + 3 * stride < n16; i += 4 * stride) {
    int4 a = src[i], b = src[i + stride], c = src[i + 2 * stride], d = src[i + 3 * stride];
    dst[i] = a; dst[i + stride] = b; dst[i + 2 * stride] = c; dst[i + 3 * stride] = d;
  }
  for (; i < n16; i += stride) dst[i] = src[i];
}

// one warp per row; row_bytes multiple of 512
__global__ void zc_gather_kernel(const int4* __restrict__ table, const int* ids, int nrows, int row16,
                                 int4* __restrict__ out) {
  int warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
  if (warp >= nrows) return;
  const int4* r = table + (size_t)ids[warp] * row16;
  for (int c = lane; c < row16; c += 32) out[(size_t)warp * row16 + c] = r[c];
}

__global__ void spin_kernel(long long cycles) {
  long long t0 = clock64();
  while (clock64() - t0 < cycles) {}
}

static float time_ms(cudaStream_t s, cudaEvent_t a, cudaEvent_t b) {
  float ms; CK(cudaEventSynchronize(b)); CK(cudaEventElapsedTime(&ms, a, b)); return ms;
}

int main() {
  int dev = 0; CK(cudaSetDevice(dev));
  cudaDeviceProp p; CK(cudaGetDeviceProperties(&p, dev));
  cudaStream_t s, s2; CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  CK(cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking));
  cudaEvent_t e0, e1, e2, e3;
  CK(cudaEventCreate(&e0)); CK(cudaEventCreate(&e1)); CK(cudaEventCreate(&e2)); CK(cudaEventCreate(&e3));
  const size_t MAXB = 512ull << 20;
  void *hp, *hwc, *dp, *dp2;
  CK(cudaHostAlloc(&hp, MAXB, cudaHostAllocPortable | cudaHostAllocMapped));
  CK(cudaHostAlloc(&hwc, MAXB, cudaHostAllocPortable | cudaHostAllocMapped | cudaHostAllocWriteCombined));
  memset(hp, 1, MAXB); memset(hwc, 1, MAXB);
  CK(cudaMalloc(&dp, MAXB)); CK(cudaMalloc(&dp2, MAXB));
  int4* dout; CK(cudaMalloc(&dout, 64));
  printf("{\n \"gpu\": \"%s\", \"sms\": %d, \"pci_bus\": %d, \"can_map_host\": %d, \"unified_addr\": %d,\n",
         p.name, p.multiProcessorCount, p.pciBusID, p.canMapHostMemory, p.unifiedAddressing);
  int pageable = 0; cudaDeviceGetAttribute(&pageable, cudaDevAttrPageableMemoryAccess, dev);
  printf(" \"pageable_memory_access\": %d,\n", pageable);

  std::vector<size_t> sizes = {4096, 65536, 1 << 20, 4 << 20, 16 << 20, 64 << 20, 256 << 20, 512ull << 20};
  auto h2d = [&](void* src, const char* name, cudaMemcpyKind kind) {
    printf(" \"%s\": {", name);
    for (size_t i = 0; i < sizes.size(); ++i) {
      size_t n = sizes[i];
      int reps = n < (1 << 20) ? 200 : (n < (64 << 20) ? 20 : 5);
      for (int w = 0; w < 2; ++w)
        CK(kind == cudaMemcpyHostToDevice ? cudaMemcpyAsync(dp, src, n, kind, s) : cudaMemcpyAsync(src, dp, n, kind, s));
      CK(cudaStreamSynchronize(s));
      float best = 1e30f;
      for (int r = 0; r < reps; ++r) {
        CK(cudaEventRecord(e0, s));
        CK(kind == cudaMemcpyHostToDevice ? cudaMemcpyAsync(dp, src, n, kind, s) : cudaMemcpyAsync(src, dp, n, kind, s));
        CK(cudaEventRecord(e1, s));
        best = std::min(best, time_ms(s, e0, e1));
      }
      printf("%s\"%zu\": [%.4f, %.2f]", i ? ", " : "", n, best * 1e3f, n / (best * 1e-3) / 1e9);
    }
    printf("},\n");
  };
  h2d(hp, "h2d_pinned_us_gbs", cudaMemcpyHostToDevice);
  h2d(hwc, "h2d_wc_us_gbs", cudaMemcpyHostToDevice);
  h2d(hp, "d2h_pinned_us_gbs", cudaMemcpyDeviceToHost);

  // back-to-back many copies of one layer-sized chunk (as the load stream issues them)
  {
    const size_t chunk = 1181184;  // BERT-Base q/k/v weight+bias fp16
    const int nchunk = 100;
    CK(cudaEventRecord(e0, s));
    for (int i = 0; i < nchunk; ++i)
      CK(cudaMemcpyAsync((char*)dp + i * chunk, (char*)hp + i * chunk, chunk, cudaMemcpyHostToDevice, s));
    CK(cudaEventRecord(e1, s));
    float ms = time_ms(s, e0, e1);
    CK(cudaEventRecord(e0, s));
    for (int i = 0; i < nchunk; ++i) {
      CK(cudaMemcpyAsync((char*)dp + i * chunk, (char*)hp + i * chunk, chunk, cudaMemcpyHostToDevice, s));
      CK(cudaEventRecord(e2, s));
    }
    CK(cudaEventRecord(e1, s));
    float ms2 = time_ms(s, e0, e1);
    printf(" \"h2d_100x1.18MB_gbs\": %.2f, \"h2d_100x1.18MB_with_events_gbs\": %.2f,\n",
           nchunk * chunk / (ms * 1e-3) / 1e9, nchunk * chunk / (ms2 * 1e-3) / 1e9);
  }

  // zero-copy read sweep
  printf(" \"zc_read_gbs\": {");
  {
    size_t n = 256ull << 20; size_t n16 = n / 16;
    int blocks_list[] = {148, 296, 592, 1184, 2368};
    int threads_list[] = {256, 512, 1024};
    bool first = true;
    for (int b : blocks_list) for (int t : threads_list) {
      zc_read_kernel<<<b, t, 0, s>>>((const int4*)hp, n16, dout);
      CK(cudaStreamSynchronize(s));
      float best = 1e30f;
      for (int r = 0; r < 3; ++r) {
        CK(cudaEventRecord(e0, s)); zc_read_kernel<<<b, t, 0, s>>>((const int4*)hp, n16, dout);
        CK(cudaEventRecord(e1, s)); best = std::min(best, time_ms(s, e0, e1));
      }
      printf("%s\"%dx%d\": %.2f", first ? "" : ", ", b, t, n / (best * 1e-3) / 1e9); first = false;
    }
  }
  printf("},\n");
  // zero-copy read of write-combined memory
  {
    size_t n = 256ull << 20;
    float best = 1e30f;
    for (int r = 0; r < 3; ++r) {
      CK(cudaEventRecord(e0, s)); zc_read_kernel<<<1184, 512, 0, s>>>((const int4*)hwc, n / 16, dout);
      CK(cudaEventRecord(e1, s)); best = std::min(best, time_ms(s, e0, e1));
    }
    printf(" \"zc_read_wc_gbs\": %.2f,\n", n / (best * 1e-3) / 1e9);
  }
  // zero-copy host->HBM copy kernel
  {
    size_t n = 256ull << 20;
    printf(" \"zc_copy_gbs\": {");
    int cfg[][2] = {{148, 512}, {296, 512}, {592, 512}, {1184, 512}};
    for (int c = 0; c < 4; ++c) {
      float best = 1e30f;
      for (int r = 0; r < 3; ++r) {
        CK(cudaEventRecord(e0, s)); zc_copy_kernel<<<cfg[c][0], cfg[c][1], 0, s>>>((const int4*)hp, (int4*)dp, n / 16);
        CK(cudaEventRecord(e1, s)); best = std::min(best, time_ms(s, e0, e1));
      }
      printf("%s\"%dx%d\": %.2f", c ? ", " : "", cfg[c][0], cfg[c][1], n / (best * 1e-3) / 1e9);
    }
    printf("},\n");
  }
  // zero-copy gather: S rows of 1536 B (BERT-Base fp16 H=768) from a 47 MB table
  {
    int rows_list[] = {32, 128, 384, 1024, 8192};
    int* dids; CK(cudaMalloc(&dids, 8192 * sizeof(int)));
    std::vector<int> ids(8192); srand(1); for (auto& v : ids) v = rand() % 30522;
    CK(cudaMemcpy(dids, ids.data(), ids.size() * 4, cudaMemcpyHostToDevice));
    printf(" \"zc_gather_1536B_us_gbs\": {");
    for (int k = 0; k < 5; ++k) {
      int nr = rows_list[k];
      float best = 1e30f;
      for (int r = 0; r < 10; ++r) {
        CK(cudaEventRecord(e0, s));
        zc_gather_kernel<<<(nr * 32 + 255) / 256, 256, 0, s>>>((const int4*)hp, dids, nr, 1536 / 16, (int4*)dp);
        CK(cudaEventRecord(e1, s)); best = std::min(best, time_ms(s, e0, e1));
      }
      printf("%s\"%d\": [%.3f, %.2f]", k ? ", " : "", nr, best * 1e3, (double)nr * 1536 / (best * 1e-3) / 1e9);
    }
    printf("},\n");
  }
  // concurrent H2D (copy engine) + zero-copy read (SM) on two streams
  {
    size_t n = 256ull << 20;
    CK(cudaEventRecord(e0, s));
    CK(cudaMemcpyAsync(dp, hp, n, cudaMemcpyHostToDevice, s));
    CK(cudaEventRecord(e1, s));
    CK(cudaEventRecord(e2, s2));
    zc_read_kernel<<<1184, 512, 0, s2>>>((const int4*)((char*)hp + n), n / 16, dout);
    CK(cudaEventRecord(e3, s2));
    float a = time_ms(s, e0, e1), b = time_ms(s2, e2, e3);
    printf(" \"concurrent_h2d_and_zc\": {\"h2d_ms\": %.3f, \"zc_ms\": %.3f, \"h2d_gbs\": %.2f, \"zc_gbs\": %.2f},\n",
           a, b, n / (a * 1e-3) / 1e9, n / (b * 1e-3) / 1e9);
  }
  // two concurrent H2D copies on two streams (does a second copy engine add bandwidth?)
  {
    size_t n = 256ull << 20;
    CK(cudaDeviceSynchronize());
    CK(cudaEventRecord(e0, s));
    CK(cudaStreamWaitEvent(s2, e0));
    CK(cudaMemcpyAsync(dp, hp, n, cudaMemcpyHostToDevice, s));
    CK(cudaMemcpyAsync(dp2, (char*)hp + n, n, cudaMemcpyHostToDevice, s2));
    CK(cudaEventRecord(e2, s2));
    CK(cudaStreamWaitEvent(s, e2));
    CK(cudaEventRecord(e1, s));
    float a = time_ms(s, e0, e1);
    printf(" \"two_stream_h2d_gbs\": %.2f,\n", 2 * n / (a * 1e-3) / 1e9);
  }
  // overheads
  {
    CK(cudaDeviceSynchronize());
    spin_kernel<<<1, 1, 0, s>>>(2000000);  // keep the stream busy so we time only enqueue cost
    auto t0 = std::chrono::steady_clock::now();
    for (int i = 0; i < 1000; ++i) CK(cudaMemcpyAsync((char*)dp + i * 4096, (char*)hp + i * 4096, 3072, cudaMemcpyHostToDevice, s));
    auto t1 = std::chrono::steady_clock::now();
    for (int i = 0; i < 1000; ++i) CK(cudaEventRecord(e2, s));
    auto t2 = std::chrono::steady_clock::now();
    for (int i = 0; i < 1000; ++i) CK(cudaStreamWaitEvent(s2, e2));
    auto t3 = std::chrono::steady_clock::now();
    for (int i = 0; i < 1000; ++i) spin_kernel<<<1, 1, 0, s2>>>(0);
    auto t4 = std::chrono::steady_clock::now();
    CK(cudaDeviceSynchronize());
    auto us = [](auto a, auto b) { return std::chrono::duration<double, std::micro>(b - a).count() / 1000; };
    // device-side latency of a tiny H2D
    float best = 1e30f;
    for (int r = 0; r < 50; ++r) {
      CK(cudaEventRecord(e0, s)); CK(cudaMemcpyAsync(dp, hp, 3072, cudaMemcpyHostToDevice, s));
      CK(cudaEventRecord(e1, s)); best = std::min(best, time_ms(s, e0, e1));
    }
    float best100 = 1e30f;
    for (int r = 0; r < 5; ++r) {
      CK(cudaEventRecord(e0, s));
      for (int i = 0; i < 100; ++i) CK(cudaMemcpyAsync((char*)dp + i * 4096, (char*)hp + i * 4096, 3072, cudaMemcpyHostToDevice, s));
      CK(cudaEventRecord(e1, s)); best100 = std::min(best100, time_ms(s, e0, e1));
    }
    float kbest = 1e30f;
    for (int r = 0; r < 5; ++r) {
      CK(cudaEventRecord(e0, s));
      for (int i = 0; i < 100; ++i) spin_kernel<<<1, 32, 0, s>>>(0);
      CK(cudaEventRecord(e1, s)); kbest = std::min(kbest, time_ms(s, e0, e1));
    }
    printf(" \"host_enqueue_us\": {\"memcpy_async\": %.3f, \"event_record\": %.3f, \"stream_wait\": %.3f, \"launch\": %.3f},\n",
           us(t0, t1), us(t1, t2), us(t2, t3), us(t3, t4));
    printf(" \"device_us\": {\"h2d_3KB\": %.3f, \"h2d_3KB_x100_each\": %.3f, \"empty_kernel_x100_each\": %.3f}\n",
           best * 1e3, best100 * 10, kbest * 10);
  }
  printf("}\n");
  return 0;
}
