"""Secondary selection for parallel transmission on measured link rates (R25; P:148
PCIe-switch contention, P:186 / P:227-229 "GPUs attached to different PCIe switches"): the C++
selector (dp_select_secondaries) equals the oracle's on random matrices, and both pick GPUs on
other switches on constructed topologies."""
import itertools

import numpy as np
import pytest

import paper_conf_eurosys_jeongba23_b200 as dp
from oracle import planner as P


def switch_topology(groups, solo=55.0):
    """GPUs in the same group share a PCIe switch: two at once get half the link each."""
    n = sum(len(g) for g in groups)
    grp = {d: i for i, g in enumerate(groups) for d in g}
    pair = np.full((n, n), solo)
    for i in range(n):
        for j in range(n):
            if i != j and grp[i] == grp[j]:
                pair[i][j] = solo / 2
    return [solo] * n, pair


def test_prefers_other_switches():
    solo, pair = switch_topology([[0, 1], [2, 3], [4, 5], [6, 7]])
    assert P.select_secondaries(solo, pair, 0, 2) == [2]
    assert P.select_secondaries(solo, pair, 0, 4) == [2, 4, 6]
    # equally fast other switches: the NUMA tie-break takes the primary's node first
    numa = [0, 0, 0, 0, 1, 1, 1, 1]
    assert P.select_secondaries(solo, pair, 5, 4, numa) == [6, 0, 2]
    # more links than switches: the fifth must share a switch
    sec = P.select_secondaries(solo, pair, 0, 5)
    assert sec[:3] == [2, 4, 6] and sec[3] in (1, 3, 5, 7)
    assert dp.select_secondaries(solo, pair, 0, 4) == [2, 4, 6]
    assert dp.select_secondaries(solo, pair, 5, 4, numa) == [6, 0, 2]


def test_bottleneck_is_maximised_brute_force():
    """Each greedy step picks a device maximising the set's worst concurrent link (checked by
    enumerating every candidate)."""
    rng = np.random.default_rng(0)
    for _ in range(50):
        n = int(rng.integers(2, 9))
        solo = rng.uniform(20, 60, n)
        pair = np.minimum(solo[:, None], rng.uniform(10, 60, (n, n)))
        prim = int(rng.integers(0, n))
        k = int(rng.integers(1, n + 1))
        sec = P.select_secondaries(list(solo), pair.tolist(), prim, k)
        chosen = [prim]
        for c in sec:
            def worst(x):
                return min([solo[x]] + [min(pair[x][s], pair[s][x]) for s in chosen])
            cand = [x for x in range(n) if x not in chosen]
            assert worst(c) == max(worst(x) for x in cand)
            chosen.append(c)
        assert len(set(chosen)) == k


@pytest.mark.parametrize("seed", range(40))
def test_cpp_matches_oracle(seed):
    rng = np.random.default_rng(100 + seed)
    n = int(rng.integers(1, 9))
    solo = np.round(rng.uniform(20, 60, n), 1)  # rounded: ties happen
    pair = np.minimum(solo[:, None], np.round(rng.uniform(10, 60, (n, n)), 0))
    numa = rng.integers(0, 2, n)
    for prim, k in itertools.product(range(n), range(1, n + 1)):
        assert dp.select_secondaries(solo, pair, prim, k, numa) == \
            P.select_secondaries(list(solo), pair.tolist(), prim, k, list(numa))


@pytest.mark.gpu
def test_numa_queries_on_this_host():
    p = dp.host_alloc_node(1 << 20, 0)
    try:
        assert dp.host_numa_node(p) in (0, -1)
    finally:
        dp.host_free(p)


@pytest.mark.gpu
def test_weight_arena_is_on_the_serving_gpus_numa_node():
    import synth
    m = synth.SHAPES["tiny_bert"]
    ctx = dp.Context([0])
    model = dp.Model(ctx, m, synth.make_weights(m, seed=0))
    node = dp.device_numa_node(0)
    page = model.arena().ctypes.data
    got = dp.host_numa_node(page)
    if node >= 0 and got >= 0:
        assert got == node
    model.close()
    ctx.close()
    # the concurrent probe on one device equals a solo measurement in kind (GB/s of a PCIe link)
    gbs = dp.measure_h2d_concurrent([0], 64 << 20, 3)
    assert 5.0 < gbs[0] < 200.0
