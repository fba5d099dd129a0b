"""ORACLE (test infrastructure): DeepPlan's planner and its pipeline cost model.

Follows PAPER.md §4.1-4.3 step by step, with the readings of DESIGN.md §3 (SURVEY §8(c)
P1-P4, G2-G10).  Everything is exact int64 nanosecond arithmetic, so the product
planner (C++, behind the C-ABI) must match it bit-exactly.

Encodings: method LOAD = 0, DHA = 1; slot 0 = the primary GPU's own PCIe
link, slot s >= 1 = the s-th parallel-transmission partition.

Cost table (dict of int64 arrays, one entry per planning unit in forward order):
  bytes, load_ns (H2D on one link), fwd_ns (secondary -> primary over NVLink),
  exe_mem_ns (Exe(InMem)), exe_dha_ns (Exe(DHA); INF_NS = ineligible)  -- P:200-202.
"""
from __future__ import annotations

import heapq
import itertools

import numpy as np

LOAD, DHA = 0, 1
MODES = ("BASELINE", "PIPESWITCH", "GREEDY", "DHA", "PT", "PT_DHA")  # the paper's options
EXT_MODES = ("DHA_LINK", "PT_DHA_LINK", "PT_DHA_BAL", "PT_DHA_LINK_BAL",  # NEXT-row extensions, R19 / R20
             "PT_DHA_STRIPE", "PT_DHA_LINK_STRIPE")                              # R22
LINK_AWARE = {"DHA_LINK", "PT_DHA_LINK", "PT_DHA_LINK_BAL", "PT_DHA_LINK_STRIPE"}
INF_NS = 1 << 50


def _arr(cost, key):
    return [int(v) for v in np.asarray(cost[key], dtype=np.int64)]


# ------------------------------------------------------------------------------------
# P1: pipeline simulator.  P:162-170 (Fig.7/8): a loaded layer can start only after it
# is loaded ("the pipeline execution for L1 is stalled due to the dependency"); a DHA
# layer needs no load; loads go back to back in plan order on one link ("The load
# stream copies selected layers sequentially according to the plan").  PT:
# the secondary's partition goes over its own link, then is forwarded over NVLink "in
# the pipelined manner", one layer at a time after it lands.
# ------------------------------------------------------------------------------------

def simulate(cost, method, slot=None, k: int = 1, serial: bool = False, link_aware: bool = False):
    """Returns dict(latency, stall[n], avail[n], start[n], link_bytes[k]).

    serial=True is the "Baseline" option (Fig.1b): load every layer, then execute.
    link_aware=True is our NEXT-row extension (R19): a DHA unit's
    reads occupy the primary link for cost["dha_link_ns"][i], in forward order with the loads
    (the paper profiles Exe(DHA) in isolation and ignores that sharing, G11).
    """
    n = len(method)
    load, fwd = _arr(cost, "load_ns"), _arr(cost, "fwd_ns")
    exe_mem, exe_dha = _arr(cost, "exe_mem_ns"), _arr(cost, "exe_dha_ns")
    nbytes = _arr(cost, "bytes")
    dlink = _arr(cost, "dha_link_ns") if (link_aware and "dha_link_ns" in cost) else [0] * n
    slot = [0] * n if slot is None else [int(s) for s in slot]
    t_link = [0] * k
    t_fwd = [0] * k
    link_bytes = [0] * k
    avail = [0] * n
    for i in range(n):
        if method[i] == DHA:
            avail[i] = 0
            t_link[0] += dlink[i]
        elif slot[i] == 0:
            t_link[0] += load[i]
            avail[i] = t_link[0]
            link_bytes[0] += nbytes[i]
        else:
            s = slot[i]
            t_link[s] += load[i]
            t_fwd[s] = max(t_link[s], t_fwd[s]) + fwd[i]
            avail[i] = t_fwd[s]
            link_bytes[s] += nbytes[i]
    if serial:
        done = max(avail) if n else 0
        avail = [done] * n
    t = 0
    stall = [0] * n
    start = [0] * n
    for i in range(n):
        st = max(t, avail[i])
        stall[i] = st - t
        start[i] = st
        t = st + (exe_dha[i] if method[i] == DHA else exe_mem[i])
    return {"latency": t, "stall": stall, "avail": avail, "start": start, "link_bytes": link_bytes}


def simulate_events(cost, method, slot=None, k: int = 1, link_aware: bool = False):
    """An independent formulation of P1 as a discrete-event simulation with FIFO
    resources (one per PCIe link, one NVLink forwarder per secondary, one compute
    engine).  Used only to pin ``simulate``; returns (latency, stall[n]).  link_aware:
    DHA units' reads are jobs on link 0 too (forward order), gating nothing."""
    n = len(method)
    load, fwd = _arr(cost, "load_ns"), _arr(cost, "fwd_ns")
    exe_mem, exe_dha = _arr(cost, "exe_mem_ns"), _arr(cost, "exe_dha_ns")
    slot = [0] * n if slot is None else [int(s) for s in slot]
    dlink = _arr(cost, "dha_link_ns") if (link_aware and "dha_link_ns" in cost) else None
    if dlink is not None:
        load = [load[i] if method[i] == LOAD else dlink[i] for i in range(n)]
    # queues of pending jobs per resource, in forward order
    link_q = {s: [i for i in range(n) if (method[i] == LOAD or (dlink is not None and s == 0)) and slot[i] == s]
              for s in range(k)}
    busy_until = {("link", s): 0 for s in range(k)}
    busy_until.update({("nvl", s): 0 for s in range(1, k)})
    ready = [None] * n  # time unit i's weights are usable on the primary
    for i in range(n):
        if method[i] == DHA:
            ready[i] = 0
    ev = []  # (time, seq, kind, payload)
    seq = itertools.count()
    # start the first transfer on each link at t=0
    for s in range(k):
        if link_q[s]:
            i = link_q[s].pop(0)
            heapq.heappush(ev, (load[i], next(seq), "link_done", (s, i)))
    nvl_q = {s: [] for s in range(1, k)}
    nvl_busy = {s: False for s in range(1, k)}
    while ev:
        t, _, kind, (s, i) = heapq.heappop(ev)
        if kind == "link_done":
            if s == 0:
                if method[i] == LOAD:  # a DHA read completing gates nothing
                    ready[i] = t
            else:
                nvl_q[s].append(i)
                if not nvl_busy[s]:
                    j = nvl_q[s].pop(0)
                    nvl_busy[s] = True
                    heapq.heappush(ev, (t + fwd[j], next(seq), "nvl_done", (s, j)))
            if link_q[s]:
                j = link_q[s].pop(0)
                heapq.heappush(ev, (t + load[j], next(seq), "link_done", (s, j)))
        else:  # nvl_done
            ready[i] = t
            nvl_busy[s] = False
            if nvl_q[s]:
                j = nvl_q[s].pop(0)
                nvl_busy[s] = True
                heapq.heappush(ev, (t + fwd[j], next(seq), "nvl_done", (s, j)))
    t = 0
    stall = []
    for i in range(n):
        st = max(t, ready[i])
        stall.append(st - t)
        t = st + (exe_dha[i] if method[i] == DHA else exe_mem[i])
    return t, stall


# ------------------------------------------------------------------------------------
# P2: Algorithm 1 (prose P:225)
# ------------------------------------------------------------------------------------

def algorithm1(cost):
    """Returns method[n] chosen by Algorithm 1 on a single link (slot 0 everywhere)."""
    n = len(cost["load_ns"])
    load = _arr(cost, "load_ns")
    pd = [d - m for d, m in zip(_arr(cost, "exe_dha_ns"), _arr(cost, "exe_mem_ns"))]
    method = [LOAD] * n
    for i in range(n):                                   # line 1
        stall = simulate(cost, method)["stall"]          # reading G3: re-simulate each i
        S = stall[i]
        if not S > 0:                                    # line 2
            continue
        # Step 1 (lines 3-5): L_1..L_i not yet DHA, ascending PerfDiff, ties by index (G4)
        cand = sorted((j for j in range(i + 1) if method[j] == LOAD), key=lambda j: (pd[j], j))
        for j in cand:                                   # line 6
            if S < pd[j]:                                # line 9 (strict, G5)
                break
            method[j] = DHA                              # line 12
            S = S - load[j] - pd[j]                      # line 13, verbatim (G5)
            if S <= 0:                                   # lines 16-18 (G6)
                break                                    # line 17: re-simulated at next i
    return method


def algorithm1_link(cost, slot=None, k: int = 1, init=None):
    """NEXT-row extension (R19), not the paper's algorithm: the
    same loop as Algorithm 1 run on the link-aware simulator, where switching L_j to DHA frees
    only saved_j = Load_j - DhaLink_j of link time.  Line 9 still breaks on S < PerfDiff_j;
    a candidate with saved_j <= 0 is skipped (no link time freed: it cannot advance any later
    load); line 13 becomes S - saved_j - PerfDiff_j.  With DhaLink = 0 and every Load > 0
    this is exactly algorithm1.  ``slot``/``k``/``init``: the PT arrival model, slot-0
    candidates and a kept DHA set, as in algorithm1_slots (R20)."""
    n = len(cost["load_ns"])
    load = _arr(cost, "load_ns")
    dlink = _arr(cost, "dha_link_ns") if "dha_link_ns" in cost else [0] * n
    pd = [d - m for d, m in zip(_arr(cost, "exe_dha_ns"), _arr(cost, "exe_mem_ns"))]
    method = [LOAD] * n if init is None else list(init)
    for i in range(n):
        S = simulate(cost, method, slot, k, link_aware=True)["stall"][i]
        if not S > 0:
            continue
        cand = sorted((j for j in range(i + 1) if method[j] == LOAD and (slot is None or slot[j] == 0)),
                      key=lambda j: (pd[j], j))
        for j in cand:
            if S < pd[j]:
                break
            saved = load[j] - dlink[j]
            if saved <= 0:
                continue
            method[j] = DHA
            S = S - saved - pd[j]
            if S <= 0:
                break
    return method


def algorithm1_slots(cost, slot, k: int, init=None):
    """NEXT-row extension f1(ii) (R20), not the paper's algorithm: Algorithm 1 run
    under the PT arrival model -- stalls come from P1 with the given slots (a slot-s unit is
    ready when its NVLink forward ends) and the candidates are the slot-0 units L_1..L_i not
    yet DHA (the later partitions are loaded).  ``init``: DHA units kept from an
    earlier pass (default none).  With k = 1 and no init this is exactly algorithm1."""
    n = len(cost["load_ns"])
    load = _arr(cost, "load_ns")
    pd = [d - m for d, m in zip(_arr(cost, "exe_dha_ns"), _arr(cost, "exe_mem_ns"))]
    method = [LOAD] * n if init is None else list(init)
    for i in range(n):
        S = simulate(cost, method, slot, k)["stall"][i]
        if not S > 0:
            continue
        cand = sorted((j for j in range(i + 1) if method[j] == LOAD and slot[j] == 0), key=lambda j: (pd[j], j))
        for j in cand:
            if S < pd[j]:
                break
            method[j] = DHA
            S = S - load[j] - pd[j]
            if S <= 0:
                break
    return method


def greedy(cost):
    """The "initial approach" (Table 3): DHA iff Exe(DHA) < Load + Exe(InMem)."""
    load, em, ed = _arr(cost, "load_ns"), _arr(cost, "exe_mem_ns"), _arr(cost, "exe_dha_ns")
    return [DHA if ed[i] < load[i] + em[i] else LOAD for i in range(len(load))]


# ------------------------------------------------------------------------------------
# P3: transmission planning: "equally partition a given model into the
# number of GPUs"; "change the execution method for layers belonging to the second and
# later partitions to be loaded".  Reading G10: contiguous, by whole-model bytes.
# ------------------------------------------------------------------------------------

def partition(nbytes, k: int):
    T = int(sum(int(b) for b in nbytes))
    part = []
    off = 0
    for b in nbytes:
        part.append(0 if T == 0 else min(k - 1, (k * off) // T))
        off += int(b)
    return part


def partition_transferred(nbytes, method, k: int):
    """NEXT-row extension f1(i) (R20): the P3 rule applied to the bytes that are
    actually transferred -- a DHA unit counts 0 -- so the primary's link carries its share
    instead of idling behind DHA'd embeddings (BERT-Base k = 8: slot 0 = {word} under P3)."""
    return partition([int(b) if m == LOAD else 0 for b, m in zip(nbytes, method)], k)


def stripe(cost, method, k: int, link_aware: bool = False):
    """NEXT-row extension (R22), not the paper's rule: instead of contiguous equal
    partitions, every loaded unit, in forward order, goes to the link on which it
    would reach the primary first under the P1 model, given the units already assigned:
      arrival(0) = link[0] + Load_i;  arrival(s >= 1) = max(link[s] + Load_i, fwd[s]) + Fwd_i
    (ties -> the lowest slot).  The k links then deliver the model front to back together, so
    the compute can follow the arrivals instead of waiting for a whole later partition.
    DHA units stay in slot 0; on the link-aware model (R19) their reads occupy link 0 in
    forward order, as in the simulator.  Returns slot[n]."""
    n = len(cost["load_ns"])
    load, fwd = _arr(cost, "load_ns"), _arr(cost, "fwd_ns")
    dlink = _arr(cost, "dha_link_ns") if (link_aware and "dha_link_ns" in cost) else [0] * n
    link = [0] * k
    fw = [0] * k
    slot = [0] * n
    for i in range(n):
        if method[i] == DHA:
            link[0] += dlink[i]
            continue
        best, best_t = 0, None
        for s in range(k):
            t = link[0] + load[i] if s == 0 else max(link[s] + load[i], fw[s]) + fwd[i]
            if best_t is None or t < best_t:
                best, best_t = s, t
        slot[i] = best
        link[best] += load[i]
        if best >= 1:
            fw[best] = best_t
    return slot


def plan(cost, mode: str, k: int = 1):
    """Returns (method[n], slot[n], serial flag) for one of the five engine options
     plus the greedy comparison."""
    n = len(cost["load_ns"])
    if mode == "BASELINE":
        return [LOAD] * n, [0] * n, True
    if mode == "PIPESWITCH":
        return [LOAD] * n, [0] * n, False
    if mode == "GREEDY":
        return greedy(cost), [0] * n, False
    if mode == "DHA":
        return algorithm1(cost), [0] * n, False
    if mode == "DHA_LINK":
        return algorithm1_link(cost), [0] * n, False
    if mode in ("PT", "PT_DHA", "PT_DHA_LINK"):
        method = (algorithm1(cost) if mode == "PT_DHA" else
                  algorithm1_link(cost) if mode == "PT_DHA_LINK" else [LOAD] * n)
        part = partition(cost["bytes"], k)
        slot = [0] * n
        for i in range(n):
            if part[i] >= 1:
                slot[i] = part[i]
                method[i] = LOAD
        return method, slot, False
    if mode in ("PT_DHA_BAL", "PT_DHA_LINK_BAL"):
        # (1) Algorithm 1 on one link; (2) the P3 rule on the transferred bytes, where a DHA
        # unit that falls into a later partition is loaded there, so it is dropped from
        # the DHA set and the split recomputed until the set is stable (it only shrinks);
        # (3) Algorithm 1 continued under the PT arrival model on the slot-0 units (the DHA
        # set of (1)-(2) is kept, so partition 0 only sheds bytes)
        link = mode == "PT_DHA_LINK_BAL"
        method = algorithm1_link(cost) if link else algorithm1(cost)
        if k == 1:  # one link: nothing to split
            return method, [0] * n, False
        while True:
            slot = partition_transferred(cost["bytes"], method, k)
            moved = [i for i in range(n) if method[i] == DHA and slot[i] >= 1]
            if not moved:
                break
            for i in moved:
                method[i] = LOAD
        if link:
            return algorithm1_link(cost, slot, k, init=method), slot, False
        return algorithm1_slots(cost, slot, k, init=method), slot, False
    if mode in ("PT_DHA_STRIPE", "PT_DHA_LINK_STRIPE"):
        # R22: (1) every unit loaded, striped over the k links by earliest arrival; (2) Algorithm
        # 1 (or its link-aware form) under that PT arrival model, candidates the slot-0 units
        # (as R20 step 3); (3) the units still loaded re-striped around the chosen DHA set.
        # With k = 1 this is exactly Algorithm 1.  (Starting from the one-link DHA set instead
        # keeps DHA linears that only paid while one link carried everything.)
        link = mode == "PT_DHA_LINK_STRIPE"
        method = [LOAD] * n
        slot = stripe(cost, method, k, link)
        method = algorithm1_link(cost, slot, k, init=method) if link else algorithm1_slots(cost, slot, k, init=method)
        return method, stripe(cost, method, k, link), False
    raise ValueError(mode)


# ------------------------------------------------------------------------------------
# P4: exhaustive search over method vectors (partition fixed), vectorised.
# Ties -> lexicographically smallest method vector (LOAD=0 < DHA=1).
# ------------------------------------------------------------------------------------

def simulate_batch(cost, methods: np.ndarray, slot=None, k: int = 1, link_aware: bool = False) -> np.ndarray:
    """Vectorised P1 latency over P method vectors (methods: [P, n] of 0/1)."""
    P, n = methods.shape
    load = np.asarray(cost["load_ns"], dtype=np.int64)
    fwd = np.asarray(cost["fwd_ns"], dtype=np.int64)
    em = np.asarray(cost["exe_mem_ns"], dtype=np.int64)
    ed = np.asarray(cost["exe_dha_ns"], dtype=np.int64)
    dl = (np.asarray(cost["dha_link_ns"], dtype=np.int64) if (link_aware and "dha_link_ns" in cost)
          else np.zeros(n, dtype=np.int64))
    slot = np.zeros(n, dtype=np.int64) if slot is None else np.asarray(slot, dtype=np.int64)
    t_link = np.zeros((k, P), dtype=np.int64)
    t_fwd = np.zeros((k, P), dtype=np.int64)
    t = np.zeros(P, dtype=np.int64)
    for i in range(n):
        is_dha = methods[:, i] == DHA
        s = int(slot[i])
        t_link[s] = np.where(is_dha, t_link[s] + (dl[i] if s == 0 else 0), t_link[s] + load[i])
        if s == 0:
            avail = np.where(is_dha, 0, t_link[0])
        else:
            t_fwd[s] = np.where(is_dha, t_fwd[s], np.maximum(t_link[s], t_fwd[s]) + fwd[i])
            avail = np.where(is_dha, 0, t_fwd[s])
        t = np.maximum(t, avail) + np.where(is_dha, ed[i], em[i])
    return t


def exhaustive(cost, k: int = 1, free=None, base_method=None, chunk: int = 1 << 18, link_aware: bool = False,
               slot=None):
    """Optimal method vector under P1 with the P3 partition fixed (units with part >= 1
    are LOAD on their slot).  ``free``: indices allowed to vary (default: all part-0
    units); others keep ``base_method``.  ``slot``: a given partition instead of P3 (the
    PT_DHA_BAL plans).  Returns (latency, method, slot)."""
    n = len(cost["load_ns"])
    part = list(slot) if slot is not None else (partition(cost["bytes"], k) if k > 1 else [0] * n)
    slot = list(part)
    if free is None:
        free = [i for i in range(n) if part[i] == 0]
    if any(part[u] >= 1 for u in free):
        # a unit of a PT partition must stay LOAD (the secondaries only transmit)
        raise ValueError("free index names a unit of a PT partition (slot >= 1)")
    base = np.array([LOAD] * n if base_method is None else base_method, dtype=np.int8)
    for i in range(n):
        if part[i] >= 1:
            base[i] = LOAD
    m = len(free)
    best_lat, best_idx = None, None
    total = 1 << m
    for lo in range(0, total, chunk):
        idx = np.arange(lo, min(total, lo + chunk), dtype=np.int64)
        methods = np.repeat(base[None, :], len(idx), axis=0)
        for b, u in enumerate(free):  # free[0] is the most significant bit -> lexicographic
            methods[:, u] = (idx >> (m - 1 - b)) & 1
        lat = simulate_batch(cost, methods, slot, k, link_aware)
        j = int(np.argmin(lat))  # first minimum = lexicographically smallest
        if best_lat is None or lat[j] < best_lat:
            best_lat, best_idx = int(lat[j]), int(idx[j])
    method = base.copy()
    for b, u in enumerate(free):
        method[u] = (best_idx >> (m - 1 - b)) & 1
    return best_lat, [int(x) for x in method], slot


# ---------------------------------------------------------------------------------------
# Secondary selection for PT (R25; "utilize GPUs attached to
# different PCIe switches").  Not an algorithm of the paper -- the paper only says to prefer GPUs
# on other switches; this is the greedy reading on measured link rates.
# ---------------------------------------------------------------------------------------

def select_secondaries(solo, pair, primary: int, k: int, numa=None) -> list:
    """solo[i]: device i's H2D GB/s alone; pair[i][j]: device i's GB/s while j copies at the same
    time.  Start from {primary}; k-1 times add the device c whose worst concurrent link with the
    set, min over s in the set of min(pair[c][s], pair[s][c]) (capped by solo[c]), is largest.
    Ties: same NUMA node as the primary first, then higher solo rate, then lower index."""
    n = len(solo)
    chosen = [primary]
    out = []
    for _ in range(k - 1):
        best_key, best = None, None
        for c in range(n):
            if c in chosen:
                continue
            worst = solo[c]
            for s in chosen:
                worst = min(worst, pair[c][s], pair[s][c])
            same_node = numa is not None and numa[c] == numa[primary]
            key = (worst, same_node, solo[c], -c)  # larger is better
            if best_key is None or key > best_key:
                best_key, best = key, c
        chosen.append(best)
        out.append(best)
    return out
