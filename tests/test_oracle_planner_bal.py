"""NEXT-row extension f1(i)+(ii) (R20): PT_DHA_BAL -- the equal split
over the bytes that are actually transferred, then Algorithm 1 under the PT arrival model.

Pins (none of them re-derives the planner's own arithmetic):
  * k = 1 reduces to the paper's Algorithm 1 (DHA mode);
  * with no DHA unit chosen, the split is the paper's P3 partition (PT mode);
  * the split's parts are contiguous and each carries T'/k +- one unit of transferred bytes
    (the closed-form property of floor(k * offset / T'));
  * on BERT-Base at k = 8 (Table 1 byte counts) the busiest link carries about 1/8 of the
    transferred bytes (not the 1/7 the paper's rule leaves on the secondaries) -- the
    0.52 -> 0.39 ms figure SURVEY §8(f) f1 quotes at 55 GB/s;
  * the product planner and exhaustive search over a BAL plan match the oracle bit-exactly.
"""
import numpy as np
import pytest

import synth
import paper_conf_eurosys_jeongba23_b200 as dp
from oracle import planner as P
from oracle import units as U


def _model_table(name, seed=7):
    m = synth.SHAPES[name]
    nb = np.array(U.unit_bytes(m, "fp16"), dtype=np.int64)
    rng = np.random.default_rng(seed)
    load = nb * 1_000_000_000 // 55_000_000_000
    n = len(nb)
    exe = rng.integers(3_000, 30_000, n)
    # embeddings: DHA touches only the used rows -> far cheaper than their load
    ed = exe + load + rng.integers(-5000, 40000, n)
    ed[:2] = exe[:2] + 2000
    return {"bytes": nb, "load_ns": load, "fwd_ns": nb // 700, "exe_mem_ns": exe,
            "exe_dha_ns": np.maximum(ed, 0)}


@pytest.mark.parametrize("seed", range(200))
def test_k1_is_algorithm1(seed):
    c = synth.make_cost_table(int(np.random.default_rng(seed).integers(1, 30)), 9100 + seed)
    m, s, _ = P.plan(c, "PT_DHA_BAL", 1)
    assert m == P.algorithm1(c) and s == [0] * len(m)
    m, s, _ = P.plan(c, "PT_DHA_LINK_BAL", 1)
    assert m == P.algorithm1_link(c) and s == [0] * len(m)


@pytest.mark.parametrize("seed", range(100))
def test_no_dha_is_paper_partition(seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(1, 40))
    c = synth.make_cost_table(n, 9300 + seed)
    c["exe_dha_ns"] = np.full(n, synth.INF_NS, dtype=np.int64)  # DHA never pays
    k = int(rng.integers(2, 9))
    m, s, _ = P.plan(c, "PT_DHA_BAL", k)
    assert m == [P.LOAD] * n
    assert s == P.plan(c, "PT", k)[1]


@pytest.mark.parametrize("seed", range(300))
def test_transferred_split_is_balanced(seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(1, 120))
    b = rng.integers(0, 1 << 24, n)
    meth = (rng.random(n) < 0.3).astype(int).tolist()
    k = int(rng.integers(1, 9))
    part = P.partition_transferred(list(b), meth, k)
    tb = [int(x) if mm == P.LOAD else 0 for x, mm in zip(b, meth)]
    T = sum(tb)
    assert all(part[i] <= part[i + 1] for i in range(n - 1))  # contiguous
    if T == 0:
        assert part == [0] * n
        return
    big = max(tb)
    for p in range(k):
        sp = sum(t for t, q in zip(tb, part) if q == p)
        if p < k - 1 or any(q == p for q in part):
            assert abs(sp * k - T) <= k * big + 0, (p, sp, T / k, big)


@pytest.mark.parametrize("paper,bal", [("PT_DHA", "PT_DHA_BAL"), ("PT_DHA_LINK", "PT_DHA_LINK_BAL")])
def test_bert_base_k8_busiest_link(paper, bal):
    c = _model_table("bert_base")
    c["dha_link_ns"] = c["load_ns"].copy()
    c["dha_link_ns"][:2] = c["load_ns"][:2] * 128 // 30522  # embeddings: only the used rows
    k = 8
    mp, sp, _ = P.plan(c, paper, k)
    mb, sb, _ = P.plan(c, bal, k)
    la = bal in P.LINK_AWARE
    lp = P.simulate(c, mp, sp, k, link_aware=la)["link_bytes"]
    lb = P.simulate(c, mb, sb, k, link_aware=la)["link_bytes"]
    assert mb[0] == P.DHA and mp[0] == P.DHA  # the word embedding stays DHA
    # the split's total T' = final transferred bytes + bytes DHA'd afterwards (<= all DHA bytes)
    dha_bytes = sum(int(x) for x, mm in zip(c["bytes"], mb) if mm == P.DHA)
    biggest = max(int(x) for x, mm in zip(c["bytes"], mb) if mm == P.LOAD)
    assert max(lb) <= (sum(lb) + dha_bytes) / k + biggest
    assert all(mm == P.LOAD for mm, s in zip(mb, sb) if s >= 1)
    assert lp[0] < max(lp) / 4  # the paper's rule leaves the primary link nearly idle
    assert max(lb) < 0.9 * max(lp)
    # the product planner agrees bit for bit
    p = dp.plan_generate(c, bal, k)
    assert list(p.method) == mb and list(p.slot) == sb
    assert list(dp.plan_simulate(c, p)[2]) == lb[:k]


@pytest.mark.parametrize("seed", range(60))
def test_exhaustive_over_bal_plan_matches(seed):
    rng = np.random.default_rng(9500 + seed)
    n = int(rng.integers(1, 11))
    k = int(rng.integers(2, 5))
    c = synth.make_cost_table(n, 9500 + seed)
    base = dp.plan_generate(c, "PT_DHA_BAL", k)
    slot = list(base.slot)
    free = [i for i in range(n) if slot[i] == 0]
    lat_o, m_o, slot_o = P.exhaustive(c, k=k, slot=slot, free=free, base_method=list(base.method))
    lat, p = dp.plan_exhaustive(c, base, free)
    assert lat == lat_o and list(p.method) == m_o and list(p.slot) == slot_o
    # the optimum under the BAL partition is no worse than the BAL plan itself
    assert lat <= dp.plan_simulate(c, base)[0]
