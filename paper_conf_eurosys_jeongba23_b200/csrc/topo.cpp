// Host-link topology for parallel transmission ("[the GPUs] share the PCIe
// switch ... contention", P:186 / P:227-229 "utilize GPUs attached to different PCIe switches").
//
// * NUMA: the node a GPU hangs off (sysfs numa_node of its PCI function), the CPUs of a node,
//   pinned host memory placed on a node (allocated and first-touched by a thread bound to that
//   node's CPUs), and the node a host page actually lives on (move_pages query);
// * concurrent H2D: k devices copying from pinned memory at the same time, per-device GB/s -- a
//   shared PCIe switch or root port shows up as a concurrent rate below the solo one;
// * secondary selection: given the solo rates and the pairwise concurrent matrix, pick the k-1
//   secondaries that keep the slowest link of the set fastest (greedy; R25), instead
//   of the fixed (primary + s) mod N.
#include <sched.h>
#include <sys/syscall.h>
#include <unistd.h>

#include <algorithm>
#include <cctype>
#include <cstring>
#include <fstream>
#include <sstream>
#include <thread>
#include <vector>

#include "common.h"

namespace dp {

int device_numa_node(int dev) {
  char bus[32] = {0};
  if (cudaDeviceGetPCIBusId(bus, sizeof(bus), dev) != cudaSuccess) {
    cudaGetLastError();
    return -1;
  }
  std::string id(bus);
  for (auto& ch : id) ch = (char)std::tolower((unsigned char)ch);
  std::ifstream f("/sys/bus/pci/devices/" + id + "/numa_node");
  int node = -1;
  if (f >> node) return node;
  return -1;
}

std::vector<int> node_cpus(int node) {
  std::vector<int> cpus;
  std::ifstream f("/sys/devices/system/node/node" + std::to_string(node) + "/cpulist");
  std::string list;
  if (!(f >> list)) return cpus;
  std::stringstream ss(list);
  std::string part;
  while (std::getline(ss, part, ',')) {
    const size_t dash = part.find('-');
    const int lo = std::atoi(part.substr(0, dash).c_str());
    const int hi = dash == std::string::npos ? lo : std::atoi(part.substr(dash + 1).c_str());
    for (int c = lo; c <= hi; ++c) cpus.push_back(c);
  }
  return cpus;
}

// Pinned, mapped, portable host memory whose pages live on `node` (< 0: wherever the caller
// runs): a thread bound to the node's CPUs allocates and first-touches it.
void* host_alloc_on_node(int64_t bytes, int node) {
  void* p = nullptr;
  cudaError_t err = cudaSuccess;
  auto body = [&] {
    if (node >= 0) {
      const auto cpus = node_cpus(node);
      if (!cpus.empty()) {
        cpu_set_t set;
        CPU_ZERO(&set);
        for (int c : cpus) CPU_SET(c, &set);
        sched_setaffinity(0, sizeof(set), &set);  // this thread only
      }
    }
    err = cudaHostAlloc(&p, bytes, cudaHostAllocPortable | cudaHostAllocMapped);
    if (err == cudaSuccess) std::memset(p, 0, bytes);  // first touch on this node
  };
  std::thread t(body);
  t.join();
  if (err != cudaSuccess) {
    cudaGetLastError();
    return nullptr;
  }
  return p;
}

// NUMA node of the page holding p (-1 if the kernel does not say).
int host_page_node(const void* p) {
  void* page = reinterpret_cast<void*>(reinterpret_cast<uintptr_t>(p) & ~uintptr_t(4095));
  int status = -1;
  const long r = syscall(SYS_move_pages, 0, 1UL, &page, nullptr, &status, 0);
  return (r == 0 && status >= 0) ? status : -1;
}

// Greedy secondary selection (R25).  pair[i * n + j] = device i's H2D GB/s while j
// copies at the same time.  The chosen set starts as {primary}; each step adds the candidate c
// that maximises min over s in the set of min(pair[c][s], pair[s][c]) (the slowest of the links
// that would now share time), ties broken by the same NUMA node as the primary (the arena's
// node), then by the higher solo rate, then by the lower index.
void select_secondaries(const double* solo, const double* pair, const int32_t* numa, int n, int primary, int k,
                        int32_t* out) {
  DP_CHECK(solo && pair && out, DP_ERR_INVALID, "NULL argument");
  DP_CHECK(n >= 1 && n <= 64 && primary >= 0 && primary < n && k >= 1 && k <= n, DP_ERR_INVALID,
           "bad n / primary / k");
  std::vector<int> chosen{primary};
  std::vector<char> used(n, 0);
  used[primary] = 1;
  for (int step = 1; step < k; ++step) {
    int best = -1;
    double best_score = -1.0;
    for (int c = 0; c < n; ++c) {
      if (used[c]) continue;
      double score = solo[c];
      for (int s : chosen) score = std::min(score, std::min(pair[c * n + s], pair[s * n + c]));
      auto better = [&] {
        if (best < 0 || score > best_score) return true;
        if (score < best_score) return false;
        const bool cl = numa && numa[c] == numa[primary], bl = numa && numa[best] == numa[primary];
        if (cl != bl) return cl;
        if (solo[c] != solo[best]) return solo[c] > solo[best];
        return c < best;
      };
      if (better()) {
        best = c;
        best_score = score;
      }
    }
    used[best] = 1;
    chosen.push_back(best);
    out[step - 1] = best;
  }
}

}  // namespace dp

using namespace dp;

extern "C" int32_t dp_device_numa_node(int32_t dev) { return device_numa_node(dev); }

extern "C" int32_t dp_host_numa_node(const void* p) { return p ? host_page_node(p) : -1; }

extern "C" dp_status dp_host_alloc_node(int64_t bytes, int32_t node, void** out) {
  return guard([&] {
    DP_CHECK(out && bytes > 0, DP_ERR_INVALID, "bad arguments");
    *out = host_alloc_on_node(bytes, node);
    DP_CHECK(*out, DP_ERR_OOM, "cudaHostAlloc failed");
  });
}

extern "C" dp_status dp_select_secondaries(const double* solo_gbs, const double* pair_gbs, const int32_t* numa,
                                           int32_t n, int32_t primary, int32_t k, int32_t* out) {
  return guard([&] { select_secondaries(solo_gbs, pair_gbs, numa, n, primary, k, out); });
}

extern "C" dp_status dp_measure_h2d_concurrent(const int32_t* devs, int32_t n, int64_t bytes, int32_t reps,
                                               double* gbs) {
  struct Dev {
    int d = -1;
    void* h = nullptr;
    void* b = nullptr;
    cudaStream_t s = nullptr;
    cudaEvent_t e0 = nullptr, e1 = nullptr;
    std::vector<float> ms;
  };
  std::vector<Dev> ds;
  int prev = 0;
  cudaGetDevice(&prev);
  dp_status st = guard([&] {
    DP_CHECK(devs && gbs && n >= 1 && n <= DP_MAX_DEVICES && bytes > 0 && reps >= 1, DP_ERR_INVALID, "bad arguments");
    ds.resize(n);
    for (int i = 0; i < n; ++i) {
      Dev& x = ds[i];
      x.d = devs[i];
      DP_CUDA(cudaSetDevice(x.d));
      x.h = host_alloc_on_node(bytes, device_numa_node(x.d));  // each source local to its GPU
      DP_CHECK(x.h, DP_ERR_OOM, "cudaHostAlloc failed");
      DP_CHECK(cudaMalloc(&x.b, bytes) == cudaSuccess, DP_ERR_OOM, "cudaMalloc failed");
      DP_CUDA(cudaStreamCreateWithFlags(&x.s, cudaStreamNonBlocking));
      DP_CUDA(cudaEventCreate(&x.e0));
      DP_CUDA(cudaEventCreate(&x.e1));
    }
    for (int r = 0; r <= reps; ++r) {  // rep 0 warms up; all devices' copies issued together
      for (auto& x : ds) {
        DP_CUDA(cudaSetDevice(x.d));
        DP_CUDA(cudaEventRecord(x.e0, x.s));
        DP_CUDA(cudaMemcpyAsync(x.b, x.h, bytes, cudaMemcpyHostToDevice, x.s));
        DP_CUDA(cudaEventRecord(x.e1, x.s));
      }
      for (auto& x : ds) {
        DP_CUDA(cudaSetDevice(x.d));
        DP_CUDA(cudaEventSynchronize(x.e1));
        float ms = 0;
        DP_CUDA(cudaEventElapsedTime(&ms, x.e0, x.e1));
        if (r > 0) x.ms.push_back(ms);
      }
    }
    for (int i = 0; i < n; ++i) {
      auto v = ds[i].ms;
      std::sort(v.begin(), v.end());
      gbs[i] = double(bytes) / (double(v[v.size() / 2]) * 1e-3) / 1e9;  // median rep
    }
  });
  for (auto& x : ds) {
    if (x.d < 0) continue;
    cudaSetDevice(x.d);
    if (x.e0) cudaEventDestroy(x.e0);
    if (x.e1) cudaEventDestroy(x.e1);
    if (x.s) cudaStreamDestroy(x.s);
    if (x.b) cudaFree(x.b);
    if (x.h) cudaFreeHost(x.h);
  }
  cudaSetDevice(prev);
  return st;
}
