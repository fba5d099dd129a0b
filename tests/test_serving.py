"""Serving harness (C++, dry-run replay through dp_serve_run) against the independent
event-driven oracle replay: identical GPU assignment, cold/warm decisions, eviction counts
and start/finish times on seeded Poisson traces.  Also pins the oracle on
hand-checkable cases (P:322 one request per GPU, P:338 LRU)."""
import numpy as np
import pytest

import synth
import paper_conf_eurosys_jeongba23_b200 as dp
from oracle import serving as OS


def _table(nmodels, rng):
    cold = rng.integers(5_000_000, 60_000_000, nmodels)
    warm = rng.integers(500_000, 5_000_000, nmodels)
    rb = rng.integers(100 << 20, 700 << 20, nmodels)
    return cold, warm, rb


@pytest.mark.parametrize("seed", range(12))
def test_dry_run_matches_oracle(seed):
    rng = np.random.default_rng(seed)
    ninst = int(rng.integers(5, 300))
    ngpu = int(rng.integers(1, 9))
    nmodels = 3
    cold, warm, rb = _table(nmodels, rng)
    moi = synth.instance_models(ninst, (4, 4, 1))
    arr, inst = synth.make_poisson_trace(int(rng.integers(50, 1500)), float(rng.integers(20, 400)), ninst, seed)
    budget = int(rb.max() * rng.integers(1, 30))
    kw = dict(ngpu=ngpu, per_gpu_budget_bytes=budget, cold_ns=cold, warm_ns=warm, resident_bytes=rb,
              model_of_instance=moi)
    got = dp.serve_run(arr, inst, dry_run=True, **kw)
    ref = OS.replay(arr, inst, **kw)
    for k in ref:
        assert np.array_equal(got[k], ref[k]), k


def test_oracle_hand_cases():
    # one GPU, two instances, budget for one: A cold, A warm, B cold (evicts A), A cold again
    arr = [0, 10, 20, 30]
    inst = [0, 0, 1, 0]
    r = OS.replay(arr, inst, ngpu=1, per_gpu_budget_bytes=100, cold_ns=[50], warm_ns=[5], resident_bytes=[100],
                  model_of_instance=[0, 0])
    assert list(r["cold"]) == [1, 0, 1, 1]
    assert list(r["nevicted"]) == [0, 0, 1, 1]
    assert list(r["start_ns"]) == [0, 50, 55, 105]  # one request at a time
    assert list(r["finish_ns"]) == [50, 55, 105, 155]
    # two GPUs: a cold request goes to the GPU that frees up first
    r = OS.replay([0, 1, 2], [0, 1, 2], ngpu=2, per_gpu_budget_bytes=1000, cold_ns=[50], warm_ns=[5],
                  resident_bytes=[10], model_of_instance=[0, 0, 0])
    assert list(r["gpu"]) == [0, 1, 0] and list(r["start_ns"]) == [0, 1, 50]
    # LRU: with budget 2, touching A makes B the victim
    r = OS.replay([0, 100, 200, 300, 400], [0, 1, 0, 2, 1], ngpu=1, per_gpu_budget_bytes=20, cold_ns=[10],
                  warm_ns=[1], resident_bytes=[10], model_of_instance=[0, 0, 0])
    assert list(r["cold"]) == [1, 1, 0, 1, 1]  # C evicts B (LRU), B must reload


def test_metrics():
    r = {"finish_ns": np.array([10, 30, 200]), "cold": np.array([1, 0, 1])}
    m = OS.metrics([0, 0, 0], r, slo_ns=100)
    assert m["goodput"] == pytest.approx(2 / 3) and m["cold_rate"] == pytest.approx(2 / 3)


def test_maf_like_trace_properties():
    """The synthetic MAF-like trace: deterministic per seed, mean rate
    near the requested one, heavy-tailed popularity (hot sustained instances), and burstier
    than Poisson (index of dispersion of per-second counts > 1)."""
    arr, inst = synth.make_maf_like_trace(60.0, 150.0, 200, seed=3, spikes_per_min=0)
    arr2, inst2 = synth.make_maf_like_trace(60.0, 150.0, 200, seed=3, spikes_per_min=0)
    assert np.array_equal(arr, arr2) and np.array_equal(inst, inst2)
    assert np.all(np.diff(arr) >= 0) and arr[0] >= 0 and arr[-1] < 60e9
    assert abs(len(arr) / 60.0 - 150.0) < 0.1 * 150.0
    counts = np.bincount(inst, minlength=200)
    top = np.sort(counts)[::-1]
    assert top[:20].sum() > 0.5 * len(arr)  # the hottest 10% of instances carry most requests
    per_s = np.bincount((arr // 1_000_000_000).astype(np.int64), minlength=60)
    assert per_s.var() / per_s.mean() > 3.0  # rate swings: far from Poisson (dispersion 1)
    # spikes add load on a few instances for a short time
    arr_s, inst_s = synth.make_maf_like_trace(60.0, 150.0, 200, seed=3, spikes_per_min=10)
    assert len(arr_s) > len(arr)


@pytest.mark.parametrize("seed", range(4))
def test_dry_run_matches_oracle_maf_like(seed):
    rng = np.random.default_rng(100 + seed)
    ninst = int(rng.integers(50, 300))
    ngpu = int(rng.integers(1, 9))
    cold, warm, rb = _table(3, rng)
    moi = synth.instance_models(ninst, (4, 4, 1))
    arr, inst = synth.make_maf_like_trace(8.0, float(rng.integers(50, 300)), ninst, seed=seed)
    budget = int(rb.max() * rng.integers(1, 30))
    kw = dict(ngpu=ngpu, per_gpu_budget_bytes=budget, cold_ns=cold, warm_ns=warm, resident_bytes=rb,
              model_of_instance=moi)
    got = dp.serve_run(arr, inst, dry_run=True, **kw)
    ref = OS.replay(arr, inst, **kw)
    for k in ref:
        assert np.array_equal(got[k], ref[k]), k


def test_online_replay_hand_cases():
    """R11-live on hand-checkable observations (the live dispatcher's decide / finish stamps)."""
    # one GPU, budget for one instance: A cold; B arrives while A still runs -> A has work, so it
    # cannot be evicted: B goes over budget; C arrives after both finished -> evicts A and B (LRU)
    r = OS.replay_online([0, 1, 50], [0, 1, 2], ngpu=1, per_gpu_budget_bytes=10, resident_bytes=[10, 10, 10],
                         decide_ns=[0, 1, 50], finish_ns=[20, 40, 60])
    assert list(r["cold"]) == [1, 1, 1] and list(r["nevicted"]) == [0, 0, 2]
    # two GPUs: the second cold request goes to the GPU with fewer outstanding requests
    r = OS.replay_online([0, 1, 2, 100], [0, 1, 2, 0], ngpu=2, per_gpu_budget_bytes=100,
                         resident_bytes=[10, 10, 10], decide_ns=[0, 1, 2, 100], finish_ns=[50, 2, 60, 110])
    assert list(r["gpu"]) == [0, 1, 1, 0] and list(r["cold"]) == [1, 1, 1, 0]
    # a completion observed exactly at the decision time counts as complete
    r = OS.replay_online([0, 5], [0, 1], ngpu=2, per_gpu_budget_bytes=100, resident_bytes=[1, 1],
                         decide_ns=[0, 5], finish_ns=[5, 9])
    assert list(r["gpu"]) == [0, 0]
