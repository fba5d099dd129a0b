"""Product planner vs oracle for the link-aware extension's exhaustive search (bit-exact)."""
import numpy as np
import pytest

import synth
import paper_conf_eurosys_jeongba23_b200 as dp
from oracle import planner as P


@pytest.mark.parametrize("seed", range(60))
def test_exhaustive_link_aware_matches(seed):
    rng = np.random.default_rng(4400 + seed)
    n = int(rng.integers(1, 11))
    k = int(rng.integers(1, 4))
    c = synth.make_cost_table(n, 4400 + seed)
    lat_o, m_o, slot_o = P.exhaustive(c, k=k, link_aware=True)
    base = dp.plan_generate(c, "PT_DHA_LINK" if k > 1 else "DHA_LINK", k)
    part = P.partition(list(c["bytes"]), k) if k > 1 else [0] * n
    free = [i for i in range(n) if part[i] == 0]
    lat, p = dp.plan_exhaustive(c, base, free)
    assert lat == lat_o and list(p.method) == m_o and list(p.slot) == slot_o
