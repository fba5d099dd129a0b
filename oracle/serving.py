"""ORACLE (test infrastructure): discrete-event replay of the serving policy of §5.3.

P:322 "our execution engine is designed for each GPU to run one inference request at a
time"; "To evict an instance due to the lack of GPU memory, we select the least
recently used instance"; P:328 Poisson arrivals randomly distributed across instances.
Dispatch policy = DESIGN.md §3 R11: each request, in arrival order, goes to the GPU that
holds its instance (warm), else to the GPU that becomes free first (lowest index on ties)
where LRU instances are evicted until it fits the per-GPU budget (cold).  Each GPU serves
its requests in dispatch order; start = max(arrival, GPU free), finish = start + latency.

Written as an explicit event-driven simulation (a heap of arrivals and completions) so it
shares no structure with the library's replay loop.
"""
from __future__ import annotations

import heapq
from collections import OrderedDict

import numpy as np


def replay(arrival_ns, instance, *, ngpu, per_gpu_budget_bytes, cold_ns, warm_ns, resident_bytes,
           model_of_instance):
    n = len(arrival_ns)
    free_at = [0] * ngpu               # when each GPU finishes its last dispatched request
    cache = [OrderedDict() for _ in range(ngpu)]  # instance -> bytes, oldest first (LRU)
    used = [0] * ngpu
    home = {}
    out = {k: np.zeros(n, dtype=np.int64) for k in ("start_ns", "finish_ns", "gpu", "cold", "nevicted")}
    events = [(int(arrival_ns[r]), r) for r in range(n)]
    heapq.heapify(events)
    while events:
        t, r = heapq.heappop(events)
        i = int(instance[r])
        mdl = int(model_of_instance[i])
        if i in home:
            g = home[i]
            cache[g].move_to_end(i)
            cold, ev = 0, 0
        else:
            g = min(range(ngpu), key=lambda j: (free_at[j], j))
            need = int(resident_bytes[mdl])
            ev = 0
            while used[g] + need > per_gpu_budget_bytes:
                victim, vb = cache[g].popitem(last=False)
                used[g] -= vb
                del home[victim]
                ev += 1
            cache[g][i] = need
            used[g] += need
            home[i] = g
            cold = 1
        start = max(t, free_at[g])
        fin = start + int(cold_ns[mdl] if cold else warm_ns[mdl])
        free_at[g] = fin
        for k, v in (("start_ns", start), ("finish_ns", fin), ("gpu", g), ("cold", cold), ("nevicted", ev)):
            out[k][r] = v
    return out


def metrics(arrival_ns, res, slo_ns):
    lat = (res["finish_ns"] - np.asarray(arrival_ns)).astype(np.float64)
    return {"p99_ms": float(np.percentile(lat, 99) / 1e6), "mean_ms": float(lat.mean() / 1e6),
            "goodput": float(np.mean(lat <= slo_ns)), "cold_rate": float(np.mean(res["cold"]))}


def replay_online(arrival_ns, instance, *, ngpu, per_gpu_budget_bytes, resident_bytes, decide_ns, finish_ns):
    """The live (online) policy, R11-live, re-derived from what the live dispatcher had
    observed when it decided each request -- its decision time decide_ns[r] and the time it saw
    each request complete, finish_ns[q]: request q is complete at r's decision iff
    finish_ns[q] <= decide_ns[r].  In arrival order:
      * instance resident (or becoming resident) on g  -> warm on g;
      * else cold on the GPU with the fewest outstanding (decided, not complete) requests, lowest
        index on ties;
      * then, on that GPU, while its resident bytes exceed the budget, the least recently used
        resident instance other than this one with no outstanding request is evicted; if
        none can go the GPU runs over budget until a later decision on it can evict.
    resident_bytes is per INSTANCE (its plan's loaded units).  Returns gpu, cold, nevicted and
    `resident`: {gpu: sorted instances resident there after the last decision}."""
    n = len(arrival_ns)
    gpu = np.full(n, -1, dtype=np.int64)
    cold = np.zeros(n, dtype=np.int64)
    nev = np.zeros(n, dtype=np.int64)
    home = {}
    lru = [OrderedDict() for _ in range(ngpu)]  # instance -> bytes, least recently used first
    used = [0] * ngpu
    for r in range(n):
        t = decide_ns[r]
        live = [q for q in range(r) if finish_ns[q] > t]  # decided earlier, not observed complete
        i = int(instance[r])
        if i in home:
            g = home[i]
            lru[g].move_to_end(i)
        else:
            busy = [sum(1 for q in live if gpu[q] == x) for x in range(ngpu)]
            g = min(range(ngpu), key=lambda x: (busy[x], x))
            lru[g][i] = int(resident_bytes[i])
            used[g] += int(resident_bytes[i])
            home[i] = g
            cold[r] = 1
        pend = {int(instance[q]) for q in live}
        for v in list(lru[g].keys()):
            if used[g] <= per_gpu_budget_bytes:
                break
            if v == i or v in pend:
                continue
            used[g] -= lru[g].pop(v)
            del home[v]
            nev[r] += 1
        gpu[r] = g
    return {"gpu": gpu, "cold": cold, "nevicted": nev,
            "resident": {x: sorted(lru[x].keys()) for x in range(ngpu)}}
