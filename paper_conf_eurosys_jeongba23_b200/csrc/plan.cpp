// Planner and pipeline cost model (host-only, exact int64 arithmetic).
//
// PAPER.md §4.1 defines PerfDiff = Exe(DHA) - Exe(InMem) and the stall a
// loaded layer suffers when its load has not finished; §4.3.2 / Algorithm 1
// chooses DHA layers; §4.3.3 partitions the model equally across the GPUs
// used for parallel transmission and forces the later partitions to be loaded.  The
// readings taken where the paper is silent (re-simulation instead of re-profiling,
// strict "<" on line 9, line 13 verbatim, tie-breaks, partition rule) are DESIGN.md §3.
#include <algorithm>
#include <cstring>
#include <numeric>
#include <vector>

#include "common.h"

namespace dp {

struct Sim {
  int64_t latency = 0;
  std::vector<int64_t> stall;
  std::vector<int64_t> link_bytes;
};

static void check_cost(const dp_cost_table* c) {
  DP_CHECK(c && c->n >= 0, DP_ERR_INVALID, "cost table is NULL or n < 0");
  DP_CHECK(c->n == 0 || (c->bytes && c->load_ns && c->fwd_ns && c->exe_mem_ns && c->exe_dha_ns),
           DP_ERR_INVALID, "cost table has a NULL array");
}

// The pipeline model: loads on each link go back to back in forward order from t = 0;
// a slot-s (s >= 1) unit is forwarded over NVLink after it lands on the secondary and
// after the previous forward from that secondary; compute runs units in order, each
// starting when the previous one ended and its weights are available (DHA: at once).
// link_aware (our NEXT-row extension, R19): a DHA unit's reads occupy the primary
// link for dha_link_ns[i], in forward order with the loads.
static Sim simulate(const dp_cost_table* c, const int8_t* method, const int8_t* slot, int k, bool serial,
                    bool link_aware = false) {
  const int n = c->n;
  Sim r;
  r.stall.assign(n, 0);
  r.link_bytes.assign(std::max(k, 1), 0);
  std::vector<int64_t> link_t(std::max(k, 1), 0), fwd_t(std::max(k, 1), 0), ready(n, 0);
  const bool la = link_aware && c->dha_link_ns != nullptr;
  for (int i = 0; i < n; ++i) {
    if (method[i] == DP_DHA) {  // in host memory: usable immediately
      if (la) link_t[0] += c->dha_link_ns[i];
      continue;
    }
    const int s = slot ? slot[i] : 0;
    link_t[s] += c->load_ns[i];
    r.link_bytes[s] += c->bytes[i];
    if (s == 0) {
      ready[i] = link_t[0];
    } else {
      fwd_t[s] = std::max(fwd_t[s], link_t[s]) + c->fwd_ns[i];
      ready[i] = fwd_t[s];
    }
  }
  if (serial) {  // Baseline: execution begins after every load has completed
    int64_t all = 0;
    for (int i = 0; i < n; ++i) all = std::max(all, ready[i]);
    std::fill(ready.begin(), ready.end(), all);
  }
  int64_t t = 0;
  for (int i = 0; i < n; ++i) {
    const int64_t begin = std::max(t, ready[i]);
    r.stall[i] = begin - t;
    t = begin + (method[i] == DP_DHA ? c->exe_dha_ns[i] : c->exe_mem_ns[i]);
  }
  r.latency = t;
  return r;
}

// Algorithm 1, single link.  For every layer i whose stall is positive (line 2), visit
// the not-yet-DHA layers L_1..L_i by ascending PerfDiff (lines 3-6); stop when the
// remaining stall is below the candidate's PerfDiff (line 9); otherwise switch it to DHA
// (line 12) and deduct Load + PerfDiff (line 13) until the stall is gone (lines 16-18).
// Stalls are refreshed by re-simulating the current plan before each i (line 17).
// With `slot` (NEXT-row extension f1(ii), R20): stalls come from the PT arrival
// model with those slots and only slot-0 units are candidates (later partitions are loaded).
// keep_init: start from the DHA set already in `method` instead of all LOAD.
static void algorithm1(const dp_cost_table* c, int8_t* method, const int8_t* slot = nullptr, int k = 1,
                       bool keep_init = false) {
  const int n = c->n;
  std::vector<int64_t> pd(n);
  for (int i = 0; i < n; ++i) pd[i] = c->exe_dha_ns[i] - c->exe_mem_ns[i];
  if (!keep_init)
    for (int i = 0; i < n; ++i) method[i] = DP_LOAD;
  std::vector<int> cand;
  cand.reserve(n);
  for (int i = 0; i < n; ++i) {
    int64_t S = simulate(c, method, slot, k, false).stall[i];
    if (S <= 0) continue;
    cand.clear();
    for (int j = 0; j <= i; ++j)
      if (method[j] == DP_LOAD && (slot == nullptr || slot[j] == 0)) cand.push_back(j);
    std::stable_sort(cand.begin(), cand.end(), [&](int a, int b) { return pd[a] < pd[b]; });
    for (int j : cand) {
      if (S < pd[j]) break;
      method[j] = DP_DHA;
      S = S - c->load_ns[j] - pd[j];
      if (S <= 0) break;
    }
  }
}

// Link-aware Algorithm 1 (NEXT-row extension, not the paper's; R19): the same loop
// on the link-aware model; switching L_j frees only saved_j = Load_j - DhaLink_j of link
// time, so a candidate with saved_j <= 0 is skipped and line 13 deducts saved_j.
static void algorithm1_link(const dp_cost_table* c, int8_t* method, const int8_t* slot = nullptr, int k = 1,
                            bool keep_init = false) {
  const int n = c->n;
  std::vector<int64_t> pd(n);
  for (int i = 0; i < n; ++i) pd[i] = c->exe_dha_ns[i] - c->exe_mem_ns[i];
  if (!keep_init)
    for (int i = 0; i < n; ++i) method[i] = DP_LOAD;
  std::vector<int> cand;
  cand.reserve(n);
  for (int i = 0; i < n; ++i) {
    int64_t S = simulate(c, method, slot, k, false, true).stall[i];
    if (S <= 0) continue;
    cand.clear();
    for (int j = 0; j <= i; ++j)
      if (method[j] == DP_LOAD && (slot == nullptr || slot[j] == 0)) cand.push_back(j);
    std::stable_sort(cand.begin(), cand.end(), [&](int a, int b) { return pd[a] < pd[b]; });
    for (int j : cand) {
      if (S < pd[j]) break;
      const int64_t saved = c->load_ns[j] - (c->dha_link_ns ? c->dha_link_ns[j] : 0);
      if (saved <= 0) continue;
      method[j] = DP_DHA;
      S = S - saved - pd[j];
      if (S <= 0) break;
    }
  }
}

static bool link_mode(int mode) {
  return mode == DP_MODE_DHA_LINK || mode == DP_MODE_PT_DHA_LINK || mode == DP_MODE_PT_DHA_LINK_BAL ||
         mode == DP_MODE_PT_DHA_LINK_STRIPE;
}

// Striped PT assignment (NEXT-row extension, R22; not the paper's contiguous rule):
// each loaded unit, in forward order, goes to the link on which it reaches the primary first
// under the pipeline model, given the units already assigned -- arrival on link 0 = link_0 +
// Load_i, on link s >= 1 = max(link_s + Load_i, fwd_s) + Fwd_i; ties -> the lowest link.  DHA
// units stay in slot 0; on the link-aware model their reads occupy link 0 in forward order.
static void stripe(const dp_cost_table* c, const int8_t* method, int k, bool link_aware, int8_t* slot) {
  const int n = c->n;
  std::vector<int64_t> link(k, 0), fw(k, 0);
  const bool la = link_aware && c->dha_link_ns != nullptr;
  for (int i = 0; i < n; ++i) {
    slot[i] = 0;
    if (method[i] == DP_DHA) {
      if (la) link[0] += c->dha_link_ns[i];
      continue;
    }
    int best = 0;
    int64_t best_t = 0;
    for (int s = 0; s < k; ++s) {
      const int64_t t = s == 0 ? link[0] + c->load_ns[i] : std::max(link[s] + c->load_ns[i], fw[s]) + c->fwd_ns[i];
      if (s == 0 || t < best_t) {
        best = s;
        best_t = t;
      }
    }
    slot[i] = int8_t(best);
    link[best] += c->load_ns[i];
    if (best >= 1) fw[best] = best_t;
  }
}

static void partition(const int64_t* bytes, int n, int k, int8_t* part) {
  int64_t total = 0;
  for (int i = 0; i < n; ++i) total += bytes[i];
  int64_t off = 0;
  for (int i = 0; i < n; ++i) {
    int64_t p = total == 0 ? 0 : (int64_t(k) * off) / total;
    part[i] = int8_t(std::min<int64_t>(k - 1, p));
    off += bytes[i];
  }
}

static void generate(const dp_cost_table* c, int mode, int k, dp_plan* out) {
  check_cost(c);
  DP_CHECK(out && out->method && out->slot, DP_ERR_INVALID, "plan arrays are NULL");
  DP_CHECK(out->n == c->n, DP_ERR_INVALID, "plan.n != cost.n");
  DP_CHECK(k >= 1 && k <= DP_MAX_DEVICES, DP_ERR_INVALID, "k out of range");
  const int n = c->n;
  out->mode = mode;
  out->k = k;
  out->serial = 0;
  std::memset(out->slot, 0, n);
  switch (mode) {
    case DP_MODE_BASELINE:
      std::memset(out->method, DP_LOAD, n);
      out->serial = 1;
      out->k = 1;
      return;
    case DP_MODE_PIPESWITCH:
      std::memset(out->method, DP_LOAD, n);
      out->k = 1;
      return;
    case DP_MODE_GREEDY:
      for (int i = 0; i < n; ++i)
        out->method[i] = c->exe_dha_ns[i] < c->load_ns[i] + c->exe_mem_ns[i] ? DP_DHA : DP_LOAD;
      out->k = 1;
      return;
    case DP_MODE_DHA:
      algorithm1(c, out->method);
      out->k = 1;
      return;
    case DP_MODE_DHA_LINK:
      algorithm1_link(c, out->method);
      out->k = 1;
      return;
    case DP_MODE_PT:
    case DP_MODE_PT_DHA:
    case DP_MODE_PT_DHA_LINK: {
      if (mode == DP_MODE_PT_DHA)
        algorithm1(c, out->method);
      else if (mode == DP_MODE_PT_DHA_LINK)
        algorithm1_link(c, out->method);
      else
        std::memset(out->method, DP_LOAD, n);
      std::vector<int8_t> part(n);
      partition(c->bytes, n, k, part.data());
      for (int i = 0; i < n; ++i)
        if (part[i] >= 1) {  // later partitions are loaded (to the other GPUs)
          out->slot[i] = part[i];
          out->method[i] = DP_LOAD;
        }
      return;
    }
    case DP_MODE_PT_DHA_BAL:
    case DP_MODE_PT_DHA_LINK_BAL: {
      const bool link = mode == DP_MODE_PT_DHA_LINK_BAL;
      // NEXT-row extension f1(i)+(ii) (R20): Algorithm 1 on one link; the P3 rule
      // on the bytes that are transferred (DHA units count 0); Algorithm 1 continued (its DHA
      // set kept) under the PT arrival model on the slot-0 units
      // (a DHA unit that falls into a later partition is loaded there, so it leaves the DHA
      // set and the split is recomputed; the set only shrinks, so this terminates)
      if (link)
        algorithm1_link(c, out->method);
      else
        algorithm1(c, out->method);
      if (k == 1) return;  // one link: nothing to split
      std::vector<int64_t> tb(n);
      for (bool moved = true; moved;) {
        for (int i = 0; i < n; ++i) tb[i] = out->method[i] == DP_LOAD ? c->bytes[i] : 0;
        partition(tb.data(), n, k, out->slot);
        moved = false;
        for (int i = 0; i < n; ++i)
          if (out->method[i] == DP_DHA && out->slot[i] >= 1) {
            out->method[i] = DP_LOAD;
            moved = true;
          }
      }
      if (link)
        algorithm1_link(c, out->method, out->slot, k, true);
      else
        algorithm1(c, out->method, out->slot, k, true);
      return;
    }
    case DP_MODE_PT_DHA_STRIPE:
    case DP_MODE_PT_DHA_LINK_STRIPE: {
      // R22: (1) all units loaded, striped by earliest arrival; (2) Algorithm 1 (or its
      // link-aware form) under that PT arrival model on the slot-0 units; (3) the units still
      // loaded re-striped around the chosen DHA set.  k = 1 is exactly Algorithm 1.
      const bool link = mode == DP_MODE_PT_DHA_LINK_STRIPE;
      std::memset(out->method, DP_LOAD, n);
      stripe(c, out->method, k, link, out->slot);
      if (link)
        algorithm1_link(c, out->method, out->slot, k, true);
      else
        algorithm1(c, out->method, out->slot, k, true);
      stripe(c, out->method, k, link, out->slot);
      return;
    }
    default:
      fail(DP_ERR_INVALID, "unknown plan mode");
  }
}

}  // namespace dp

using namespace dp;

extern "C" dp_status dp_plan_generate(const dp_cost_table* cost, int32_t mode, int32_t k, dp_plan* out) {
  return guard([&] { generate(cost, mode, k, out); });
}

extern "C" dp_status dp_plan_simulate(const dp_cost_table* cost, const dp_plan* plan, int64_t* latency_ns,
                                      int64_t* stall_ns, int64_t* link_bytes) {
  return guard([&] {
    check_cost(cost);
    DP_CHECK(plan && plan->method && plan->slot && plan->n == cost->n, DP_ERR_INVALID, "bad plan");
    DP_CHECK(plan->k >= 1 && plan->k <= DP_MAX_DEVICES, DP_ERR_INVALID, "plan.k out of range");
    for (int i = 0; i < plan->n; ++i)
      DP_CHECK(plan->slot[i] >= 0 && plan->slot[i] < plan->k, DP_ERR_INVALID, "slot out of range");
    Sim r = simulate(cost, plan->method, plan->slot, plan->k, plan->serial != 0, link_mode(plan->mode));
    if (latency_ns) *latency_ns = r.latency;
    if (stall_ns) std::copy(r.stall.begin(), r.stall.end(), stall_ns);
    if (link_bytes) std::copy(r.link_bytes.begin(), r.link_bytes.begin() + plan->k, link_bytes);
  });
}

extern "C" dp_status dp_plan_partition(const int64_t* bytes, int32_t n, int32_t k, int8_t* part) {
  return guard([&] {
    DP_CHECK(n >= 0 && (n == 0 || (bytes && part)), DP_ERR_INVALID, "bad arguments");
    DP_CHECK(k >= 1 && k <= DP_MAX_DEVICES, DP_ERR_INVALID, "k out of range");
    partition(bytes, n, k, part);
  });
}

extern "C" dp_status dp_plan_exhaustive(const dp_cost_table* cost, const dp_plan* base, const int32_t* free_idx,
                                        int32_t nfree, dp_plan* out, int64_t* latency_ns) {
  return guard([&] {
    check_cost(cost);
    DP_CHECK(base && base->method && base->n == cost->n, DP_ERR_INVALID, "bad base plan");
    DP_CHECK(out && out->method && out->slot && out->n == cost->n, DP_ERR_INVALID, "bad out plan");
    DP_CHECK(nfree >= 0 && nfree <= 30 && (nfree == 0 || free_idx), DP_ERR_INVALID, "nfree out of range");
    const int n = cost->n, k = std::max(1, base->k);
    std::vector<int8_t> part(n, 0), m(base->method, base->method + n);
    if (k > 1) {
      if (base->mode == DP_MODE_PT_DHA_BAL || base->mode == DP_MODE_PT_DHA_LINK_BAL ||
          base->mode == DP_MODE_PT_DHA_STRIPE || base->mode == DP_MODE_PT_DHA_LINK_STRIPE) {  // its own split
        DP_CHECK(base->slot != nullptr, DP_ERR_INVALID, "bad base plan");
        std::copy(base->slot, base->slot + n, part.begin());
      } else {
        partition(cost->bytes, n, k, part.data());
      }
    }
    for (int i = 0; i < n; ++i)
      if (part[i] >= 1) m[i] = DP_LOAD;
    for (int b = 0; b < nfree; ++b) {
      DP_CHECK(free_idx[b] >= 0 && free_idx[b] < n, DP_ERR_INVALID, "free index out of range");
      // a unit of a PT partition (slot >= 1) must stay LOAD: freeing it could put DHA on a
      // secondary's slot, an infeasible plan whose under-counted latency would win
      DP_CHECK(part[free_idx[b]] == 0, DP_ERR_INVALID, "free index names a unit of a PT partition (slot >= 1)");
    }
    int64_t best = INT64_MAX;
    uint64_t best_v = 0;
    const uint64_t total = uint64_t(1) << nfree;
    for (uint64_t v = 0; v < total; ++v) {  // free_idx[0] is the most significant bit
      for (int b = 0; b < nfree; ++b) m[free_idx[b]] = int8_t((v >> (nfree - 1 - b)) & 1);
      int64_t lat = simulate(cost, m.data(), part.data(), k, false, link_mode(base->mode)).latency;
      if (lat < best) {
        best = lat;
        best_v = v;
      }
    }
    for (int b = 0; b < nfree; ++b) m[free_idx[b]] = int8_t((best_v >> (nfree - 1 - b)) & 1);
    std::copy(m.begin(), m.end(), out->method);
    std::copy(part.begin(), part.end(), out->slot);
    out->k = k;
    out->mode = base->mode;
    out->serial = 0;
    if (latency_ns) *latency_ns = best;
  });
}
