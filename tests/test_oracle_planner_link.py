"""Pins for the link-aware planning extension (R19).

It is ours, not the paper's: DHA reads share the primary PCIe link with the DMA loads
(G11).  Pinned by: reduction to the paper's Algorithm 1 / P1 when DHA reads cost no link
time; an independent discrete-event formulation of the link-aware simulator; exhaustive
bounds (optimum <= link-aware Alg.1 <= all-LOAD) with a brute-force check of the optimum;
a hand example where a linear's DHA reads cost as much link time as loading it.
"""
import itertools

import numpy as np
import pytest

import synth
from oracle import planner as P

L, X = P.LOAD, P.DHA


@pytest.mark.parametrize("seed", range(150))
def test_link_aware_simulator_matches_event_formulation(seed):
    rng = np.random.default_rng(7000 + seed)
    n = int(rng.integers(1, 12))
    k = int(rng.integers(1, 4))
    c = synth.make_cost_table(n, 7000 + seed)
    method = [int(v) for v in rng.integers(0, 2, n)]
    slot = [int(v) for v in rng.integers(0, k, n)]
    slot = [0 if method[i] == X else slot[i] for i in range(n)]  # PT units are LOAD
    r = P.simulate(c, method, slot, k, link_aware=True)
    lat, stall = P.simulate_events(c, method, slot, k, link_aware=True)
    assert r["latency"] == lat and r["stall"] == stall


@pytest.mark.parametrize("seed", range(150))
def test_reduces_to_paper_without_link_cost(seed):
    c = synth.make_cost_table(int(np.random.default_rng(seed).integers(1, 30)), 8000 + seed, p_inf=0.05)
    c["load_ns"] = np.maximum(c["load_ns"], 1)  # zero-load units are the one degenerate difference
    c0 = dict(c, dha_link_ns=np.zeros_like(c["dha_link_ns"]))
    assert P.algorithm1_link(c0) == P.algorithm1(c0)
    m = P.algorithm1(c)
    assert P.simulate(c0, m, link_aware=True)["latency"] == P.simulate(c, m)["latency"]


@pytest.mark.parametrize("seed", range(200))
def test_link_aware_exhaustive_bounds(seed):
    rng = np.random.default_rng(9000 + seed)
    n = int(rng.integers(1, 9))
    c = synth.make_cost_table(n, 9000 + seed, p_inf=0.1)
    opt, m_opt, _ = P.exhaustive(c, link_aware=True)
    a1 = P.simulate(c, P.algorithm1_link(c), link_aware=True)["latency"]
    allload = P.simulate(c, [L] * n, link_aware=True)["latency"]
    assert opt <= a1 <= allload
    best = min((P.simulate(c, list(v), link_aware=True)["latency"], list(v))
               for v in itertools.product([0, 1], repeat=n))
    assert best == (opt, m_opt)


def test_linear_with_full_link_cost_is_not_chosen():
    """Unit 1 is linear-like: its DHA reads cost at least as much link time as loading it
    (equal: B200 K3 reads each byte once; larger: the V100 stock FC re-read its weights ~12x,
    Table 1).  The paper's Algorithm 1 (Exe(DHA) profiled alone, G11) moves it to
    DHA to cut unit 2's stall; the link-aware variant does not.  With re-reads the paper's
    plan is strictly slower under the link-aware model; with equal bytes it gains nothing."""
    for dlink1, strictly in ((50, False), (70, True)):
        c = {"bytes": np.array([1, 1, 1]), "load_ns": np.array([10, 50, 60]), "fwd_ns": np.zeros(3, np.int64),
             "exe_mem_ns": np.array([5, 5, 5]), "exe_dha_ns": np.array([12, 30, 900]),
             "dha_link_ns": np.array([1, dlink1, 60])}
        paper = P.algorithm1(c)
        ours = P.algorithm1_link(c)
        assert paper[1] == X and ours[1] == L
        a = P.simulate(c, ours, link_aware=True)["latency"]
        b = P.simulate(c, paper, link_aware=True)["latency"]
        assert (a < b) if strictly else (a == b)
