"""Pins for the planner oracle (oracle/planner.py):

* hand-computed simulator examples (3-4 units) and an independent discrete-event
  formulation of the same pipeline model;
* exhaustive 2^n enumeration for n <= 8: optimum <= Algorithm 1 <= all-LOAD;
* Algorithm 1's final plan is never worse than PipeSwitch (all LOAD);
* special cases: no stalls -> no DHA; zero loads -> all LOAD; unit 0
  becomes DHA when PerfDiff_0 <= Load_0;
* Table 3b: GPT-2's first five layers, Initial = X X O O O, DeepPlan(DHA) =
  X O O O O on a GPT-2-like cost table;
* Fig.9 / Fig.10 narratives;
* partition closed form and BERT-Base k=8: slot 0 = {word} only.
"""
import itertools

import numpy as np
import pytest

import synth
from oracle import planner as P
from oracle import units as U

L, X = P.LOAD, P.DHA


def table(load, exe_mem, exe_dha, fwd=None, nbytes=None):
    n = len(load)
    return {"bytes": np.array(nbytes or [1] * n, dtype=np.int64),
            "load_ns": np.array(load, dtype=np.int64),
            "fwd_ns": np.array(fwd or [0] * n, dtype=np.int64),
            "exe_mem_ns": np.array(exe_mem, dtype=np.int64),
            "exe_dha_ns": np.array(exe_dha, dtype=np.int64)}


def test_simulate_hand_examples():
    c = table([10, 20, 5], [3, 4, 5], [8, 100, 100])
    r = P.simulate(c, [L, L, L])
    assert r["latency"] == 40 and r["stall"] == [10, 17, 1]
    r = P.simulate(c, [X, L, L])
    assert r["latency"] == 30 and r["stall"] == [0, 12, 1]
    # baseline: all loads (35) then all compute (12)
    assert P.simulate(c, [L, L, L], serial=True)["latency"] == 47
    # PT, k=2: link0 {0,1}, link1 {2,3} then NVLink forward (2 each)
    c4 = table([10, 10, 10, 10], [1, 1, 1, 1], [9, 9, 9, 9], fwd=[2, 2, 2, 2], nbytes=[5, 6, 7, 8])
    r = P.simulate(c4, [L] * 4, [0, 0, 1, 1], k=2)
    assert r["avail"] == [10, 20, 12, 22]
    assert r["latency"] == 23
    assert r["link_bytes"] == [11, 15]


@pytest.mark.parametrize("seed", range(200))
def test_simulate_matches_event_formulation(seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(1, 12))
    k = int(rng.integers(1, 5))
    c = synth.make_cost_table(n, seed)
    method = [int(v) for v in rng.integers(0, 2, n)]
    slot = [int(v) for v in rng.integers(0, k, n)]
    r = P.simulate(c, method, slot, k)
    lat, stall = P.simulate_events(c, method, slot, k)
    assert r["latency"] == lat and r["stall"] == stall


@pytest.mark.parametrize("seed", range(300))
def test_exhaustive_bounds(seed):
    rng = np.random.default_rng(1000 + seed)
    n = int(rng.integers(1, 9))
    c = synth.make_cost_table(n, 1000 + seed, p_inf=0.1)
    opt, m_opt, _ = P.exhaustive(c)
    a1 = P.simulate(c, P.algorithm1(c))["latency"]
    allload = P.simulate(c, [L] * n)["latency"]
    assert opt <= a1 <= allload
    assert P.simulate(c, m_opt)["latency"] == opt
    # brute force in plain python for the optimum and the tie rule
    best = None
    for v in itertools.product([0, 1], repeat=n):
        lat = P.simulate(c, list(v))["latency"]
        if best is None or lat < best[0]:
            best = (lat, list(v))
    assert best[0] == opt and best[1] == m_opt


@pytest.mark.parametrize("seed", range(40))
def test_exhaustive_pt_bounds(seed):
    rng = np.random.default_rng(5000 + seed)
    n = int(rng.integers(2, 9))
    k = int(rng.integers(2, 5))
    c = synth.make_cost_table(n, 5000 + seed)
    opt, _, slot = P.exhaustive(c, k=k)
    m, s, _ = P.plan(c, "PT_DHA", k)
    assert s == slot
    lat = P.simulate(c, m, s, k)["latency"]
    m2, s2, _ = P.plan(c, "PT", k)
    assert opt <= lat and opt <= P.simulate(c, m2, s2, k)["latency"]


def test_special_cases():
    # no stalls (every load hidden behind compute of the previous unit): no DHA
    c = table([0, 5, 5, 5], [10, 10, 10, 10], [1, 1, 1, 1])
    assert P.algorithm1(c) == [L, L, L, L]
    # all loads zero -> nothing stalls -> all LOAD
    c = table([0] * 5, [3] * 5, [0] * 5)
    assert P.algorithm1(c) == [L] * 5
    # the first unit's stall is its own load; PerfDiff_0 <= Load_0 -> DHA
    c = table([100, 1, 1], [1, 1, 1], [50, 1000, 1000])
    assert P.algorithm1(c)[0] == X
    # line 9 strict: PerfDiff exactly equal to the stall is accepted
    c = table([7], [1], [8])  # stall 7, pd 7
    assert P.algorithm1(c) == [X]
    c = table([6], [1], [8])  # stall 6 < pd 7 -> break
    assert P.algorithm1(c) == [L]
    # ineligible units (INF) are never chosen
    c = table([100, 100], [1, 1], [P.INF_NS, P.INF_NS])
    assert P.algorithm1(c) == [L, L]


def test_smallest_perfdiff_first():
    """'we choose the layer that shows the smallest PerfDiff first among the
    earlier layers' -- L_{n-2} is preferred over L_{n-1} when its PerfDiff is smaller."""
    # units 0,1 small loads hidden; unit 2 has a big load -> stall at 2
    c = table([1, 10, 100], [20, 20, 5], [25, 60, 10_000])
    m = P.algorithm1(c)
    # stall at unit 1 = 11-21<0 none; stall at 2 = 111-41 = 70; pd = [5, 40, ...]
    # sorted: unit0 (5): 70>=5 -> DHA, S = 70-1-5 = 64; unit1 (40): 64>=40 -> DHA
    assert m == [X, X, L]


def test_table3b_gpt2_pattern():
    """Table 3b: GPT-2 front five layers Emb, Emb, LN, FC, FC.
    Initial approach: X X O O O; DeepPlan (DHA): X O O O O.  Costs (us) are a GPT-2-like
    table: huge wte load, wte DHA gather slower than loading wpe, wpe DHA slightly
    cheaper than load+exe, LN DHA slower than load, FC DHA very slow."""
    c = table(load=[1400, 280, 5, 640, 215],
              exe_mem=[20, 20, 10, 150, 60],
              exe_dha=[700, 290, 600, 20_000, 7_000])
    assert P.greedy(c) == [X, X, L, L, L]
    assert P.algorithm1(c) == [X, L, L, L, L]


def test_fig10_narrative():
    """Fig.10: Alg.1 selects L1 and L4 for DHA; with two GPUs the PT step
    overrides L4 to be loaded to the other GPU."""
    c = table(load=[100, 10, 10, 60, 10, 10], exe_mem=[5, 5, 5, 5, 5, 5],
              exe_dha=[20, 200, 200, 30, 200, 200], nbytes=[1] * 6, fwd=[1] * 6)
    m = P.algorithm1(c)
    assert m == [X, L, L, X, L, L]
    m2, s2, _ = P.plan(c, "PT_DHA", 2)
    assert m2 == [X, L, L, L, L, L] and s2 == [0, 0, 0, 1, 1, 1]


def test_fig9_narrative():
    """Fig.9: L1 is chosen for DHA; L2-L4 are loaded to GPU-0 and L5-L7 to
    GPU-1, then forwarded; the PT plan removes the stalls of the latter partition."""
    c = table(load=[100] + [30] * 6, exe_mem=[5] + [20] * 6, exe_dha=[10] + [500] * 6,
              nbytes=[1] * 7, fwd=[5] * 7)
    m, s, _ = P.plan(c, "PT_DHA", 2)
    assert m == [X, L, L, L, L, L, L]
    assert s == [0, 0, 0, 0, 1, 1, 1]
    lat_pt = P.simulate(c, m, s, 2)["latency"]
    lat_dha = P.simulate(c, *P.plan(c, "DHA", 1)[:2])["latency"]
    lat_ps = P.simulate(c, [L] * 7)["latency"]
    assert lat_pt < lat_dha < lat_ps


def test_partition_closed_form():
    assert P.partition([1] * 7, 2) == [0, 0, 0, 0, 1, 1, 1]
    assert P.partition([5, 1, 1, 1], 2) == [0, 1, 1, 1]  # offsets 0,5,6,7: (2*5)//8 = 1
    assert P.partition([1, 1, 1, 1], 1) == [0, 0, 0, 0]
    # contiguous and non-decreasing, covers 0..k-1 when units are small
    nb = list(range(1, 50))
    for k in (2, 3, 4, 8):
        p = P.partition(nb, k)
        assert p == sorted(p) and p[0] == 0 and p[-1] == k - 1


def test_bert_base_k8_slot0_is_word_only():
    """BERT-Base k=8 -> slot 0 carries only `word` (DHA under PT_DHA)."""
    m = synth.SHAPES["bert_base"]
    p = P.partition(U.unit_bytes(m, "fp16"), 8)
    names = [u[0] for u in U.unit_params(m)]
    assert [names[i] for i in range(len(p)) if p[i] == 0] == ["word"]


def test_tiny_bert_exhaustive_2pow21():
    """Vectorised 2^21 exhaustive search on a tiny-BERT-shaped table (SURVEY (vi))."""
    m = synth.SHAPES["tiny_bert"]
    nb = U.unit_bytes(m, "fp16")
    n = len(nb)
    rng = np.random.default_rng(21)
    load = np.array([b // 55 for b in nb], dtype=np.int64)  # ~55 GB/s -> ns
    exe_mem = rng.integers(2000, 6000, n).astype(np.int64)
    exe_dha = exe_mem + load + rng.integers(-3000, 20000, n)
    c = {"bytes": np.array(nb, dtype=np.int64), "load_ns": load, "fwd_ns": np.zeros(n, np.int64),
         "exe_mem_ns": exe_mem, "exe_dha_ns": np.maximum(exe_dha, 0).astype(np.int64)}
    opt, mopt, _ = P.exhaustive(c)
    a1 = P.simulate(c, P.algorithm1(c))["latency"]
    assert opt <= a1 <= P.simulate(c, [L] * n)["latency"]
    assert P.simulate(c, mopt)["latency"] == opt
