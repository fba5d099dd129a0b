"""The product planner (C++, behind the C-ABI) against the oracle planner: plans, simulated
latencies, stalls and per-link bytes must match bit-exactly (north_star: "Plans and
transferred weight bytes must match the oracle bit-exactly")."""
import numpy as np
import pytest

import synth
import paper_conf_eurosys_jeongba23_b200 as dp
from oracle import planner as P
from oracle import units as U


def _check_one(c, mode, k):
    om, osl, oser = P.plan(c, mode, k)
    p = dp.plan_generate(c, mode, k)
    assert list(p.method) == om, (mode, k)
    assert list(p.slot) == osl, (mode, k)
    assert p.serial == int(oser)
    lat, stall, link = dp.plan_simulate(c, p)
    r = P.simulate(c, om, osl, max(k, 1) if mode.startswith("PT") else 1, serial=oser,
                   link_aware=mode in P.LINK_AWARE)
    assert lat == r["latency"]
    assert list(stall) == r["stall"]
    assert list(link) == r["link_bytes"][:len(link)]


ALL_MODES = P.MODES + P.EXT_MODES


@pytest.mark.parametrize("block", range(20))
def test_random_tables_all_modes(block):
    """10^4 random integer tables (20 blocks x 500), the paper's modes and the link-aware
    extension."""
    rng = np.random.default_rng(block)
    for t in range(500):
        seed = block * 1000 + t
        n = int(rng.integers(1, 40))
        c = synth.make_cost_table(n, seed, max_ns=int(rng.integers(10, 100000)), p_inf=0.05)
        mode = ALL_MODES[t % len(ALL_MODES)]
        k = int(rng.integers(1, 9)) if mode.startswith("PT") else 1
        _check_one(c, mode, k)
        if t % 7 == 0:  # the paper's modes must not depend on dha_link_ns
            c2 = {kk: v for kk, v in c.items() if kk != "dha_link_ns"}
            if mode in P.MODES:
                _check_one(c2, mode, k)


@pytest.mark.parametrize("name", ["tiny_bert", "bert_base", "bert_large", "roberta_large", "gpt2_medium"])
def test_model_shaped_tables(name):
    m = synth.SHAPES[name]
    nb = np.array(U.unit_bytes(m, "fp16"), dtype=np.int64)
    rng = np.random.default_rng(7)
    load = nb * 1_000_000_000 // 55_000_000_000
    n = len(nb)
    exe = rng.integers(3_000, 30_000, n)
    c = {"bytes": nb, "load_ns": load, "fwd_ns": nb // 700, "exe_mem_ns": exe,
         "exe_dha_ns": exe + load + rng.integers(-5000, 40000, n)}
    c["exe_dha_ns"] = np.maximum(c["exe_dha_ns"], 0)
    c["dha_link_ns"] = load.copy()
    for mode in ALL_MODES:
        for k in ((1, 2, 4, 8) if mode.startswith("PT") else (1,)):
            _check_one(c, mode, k)


def test_partition_matches():
    rng = np.random.default_rng(3)
    for _ in range(500):
        n = int(rng.integers(1, 200))
        b = rng.integers(0, 1 << 26, n)
        k = int(rng.integers(1, 9))
        assert list(dp.plan_partition(b, k)) == P.partition(list(b), k)


@pytest.mark.parametrize("seed", range(60))
def test_exhaustive_matches(seed):
    rng = np.random.default_rng(900 + seed)
    n = int(rng.integers(1, 11))
    k = int(rng.integers(1, 4))
    c = synth.make_cost_table(n, 900 + seed)
    lat_o, m_o, slot_o = P.exhaustive(c, k=k)
    base = dp.plan_generate(c, "PT" if k > 1 else "PIPESWITCH", k)
    part = P.partition(list(c["bytes"]), k) if k > 1 else [0] * n
    free = [i for i in range(n) if part[i] == 0]
    lat, p = dp.plan_exhaustive(c, base, free)
    assert lat == lat_o and list(p.method) == m_o and list(p.slot) == slot_o


def test_exhaustive_rejects_pt_partition_units():
    """A unit of a PT partition (slot >= 1) must stay LOAD: freeing it in the
    exhaustive search is rejected by both planners instead of returning an infeasible plan
    whose under-counted latency wins."""
    c = synth.make_cost_table(8, 77)
    k = 3
    part = P.partition(list(c["bytes"]), k)
    bad = [i for i in range(8) if part[i] >= 1][:1]
    assert bad
    base = dp.plan_generate(c, "PT", k)
    with pytest.raises(dp.DeepPlanError):
        dp.plan_exhaustive(c, base, bad)
    with pytest.raises(ValueError):
        P.exhaustive(c, k=k, free=bad)
