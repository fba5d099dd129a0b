// linkprobe2: per-copy overhead of back-to-back H2D DMAs as the load stream issues them,
// on 1 / 2 / 4 streams round-robin, with and without an event after each copy.  Decides
// the engine's chunking.  Standalone; prints JSON.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/linkprobe2 tools/linkprobe2.cu
#include <cuda_runtime.h>

#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <vector>

#define CK(x)                                                                                   \
  do {                                                                                          \
    cudaError_t e = (x);                                                                        \
    if (e != cudaSuccess) {                                                                     \
      fprintf(stderr, "CUDA %s: %s\n", #x, cudaGetErrorString(e));                              \
      exit(1);                                                                                  \
    }                                                                                           \
  } while (0)

int main() {
  CK(cudaSetDevice(0));
  const size_t TOTAL = 192ull << 20;
  void *hp, *dp;
  CK(cudaHostAlloc(&hp, TOTAL, cudaHostAllocPortable | cudaHostAllocMapped));
  memset(hp, 3, TOTAL);
  CK(cudaMalloc(&dp, TOTAL));
  cudaStream_t st[4], main_s;
  for (auto& s : st) CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  CK(cudaStreamCreateWithFlags(&main_s, cudaStreamNonBlocking));
  std::vector<cudaEvent_t> evs(4096);
  for (size_t i = 0; i < evs.size(); ++i) CK(cudaEventCreateWithFlags(&evs[i], cudaEventDisableTiming));
  cudaEvent_t t0, t1, fork;
  CK(cudaEventCreate(&t0));
  CK(cudaEventCreate(&t1));
  CK(cudaEventCreateWithFlags(&fork, cudaEventDisableTiming));
  printf("{\"total_bytes\": %zu, \"runs\": [\n", TOTAL);
  bool first = true;
  for (size_t chunk : {65536ul, 262144ul, 1ul << 20, 1181184ul, 4ul << 20, 16ul << 20, 64ul << 20, 192ul << 20}) {
    for (int ns : {1, 2, 3, 4}) {
      for (int with_ev : {0, 1}) {
        float best = 1e30f;
        for (int rep = 0; rep < 3; ++rep) {
          CK(cudaDeviceSynchronize());
          CK(cudaEventRecord(t0, main_s));
          CK(cudaEventRecord(fork, main_s));
          for (int i = 0; i < ns; ++i) CK(cudaStreamWaitEvent(st[i], fork, 0));
          size_t n = TOTAL / chunk;
          for (size_t c = 0; c < n; ++c) {
            cudaStream_t s = st[c % ns];
            CK(cudaMemcpyAsync((char*)dp + c * chunk, (char*)hp + c * chunk, chunk, cudaMemcpyHostToDevice, s));
            if (with_ev) CK(cudaEventRecord(evs[c % evs.size()], s));
          }
          for (int i = 0; i < ns; ++i) {
            CK(cudaEventRecord(evs[4095 - i], st[i]));
            CK(cudaStreamWaitEvent(main_s, evs[4095 - i], 0));
          }
          CK(cudaEventRecord(t1, main_s));
          CK(cudaEventSynchronize(t1));
          float ms;
          CK(cudaEventElapsedTime(&ms, t0, t1));
          if (ms < best) best = ms;
        }
        size_t n = TOTAL / chunk;
        printf("%s {\"chunk\": %zu, \"streams\": %d, \"events\": %d, \"ms\": %.4f, \"gbs\": %.2f, "
               "\"overhead_us_per_copy\": %.3f}",
               first ? "" : ",\n", chunk, ns, with_ev, best, (n * chunk) / (best * 1e-3) / 1e9,
               (best * 1e3 - (n * chunk) / 55.6e3) / n);
        first = false;
      }
    }
  }
  printf("\n]}\n");
  return 0;
}
