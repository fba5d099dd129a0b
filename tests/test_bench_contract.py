"""The committed bench lines (profiles/r0*_bench_*.json) keep the bench.py JSON contract.

CPU-only: reads the JSON lines bench.py printed on the B200 box and checks the keys the driver
and the judge read (metric/value/unit, roofline, cpu_baseline, clocks, e2e, gpu_launches) and
the arithmetic that ties them together (frac = achieved / peak, value = ms_per_step).
"""
import glob
import json
import os

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
LINES = sorted(glob.glob(os.path.join(ROOT, "profiles", "r0*_bench_*.json")))
BAD_REASONS = {"hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown"}


def _load(p):
    with open(p) as f:
        return json.loads(f.read().strip().splitlines()[-1])


def test_there_are_bench_lines():
    assert LINES, "no committed bench lines under profiles/"


@pytest.mark.parametrize("path", LINES, ids=[os.path.basename(p) for p in LINES])
def test_bench_line_contract(path):
    d = _load(path)
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
              "scaling", "dtype", "data", "config"):
        assert k in d, k
    assert d["unit"] == "ms" and d["higher_is_better"] is False
    assert d["warmup"] >= 3 and d["steps"] >= 1 and d["n_gpus"] >= 1
    assert d["value"] == pytest.approx(d["ms_per_step"])
    assert d["value"] > 0
    assert "workload" in d["config"]
    if "roofline" in d:
        r = d["roofline"]
        assert r["bound"] in ("hbm", "tensor", "alu", "pcie")
        assert r["frac"] == pytest.approx(r["achieved"] / r["peak"], rel=2e-3)
        assert 0 < r["frac"] <= 1.05
    if "clocks" in d:
        assert not BAD_REASONS & set(d["clocks"]["reasons"])
        assert d["clocks"]["sm_mhz"] >= 0.9 * d["clocks"]["sm_max_mhz"]
    if "e2e" in d:
        e = d["e2e"]
        assert e["unit"] == d["unit"]
        # end to end includes the id upload and the output readback: never faster than the device time
        assert e["value"] >= d["value"] * 0.999
        if d.get("impl") == "reference":  # the host-only oracle moves nothing over the link
            assert e["h2d_bytes_per_step"] == 0 and e["d2h_bytes_per_step"] == 0
        else:
            assert e["h2d_bytes_per_step"] > 0 and e["d2h_bytes_per_step"] > 0
    if d.get("cpu_baseline") is not None:
        c = d["cpu_baseline"]
        assert c["kind"] == "oracle" and c["cores"] >= 1 and c["value"] > 0 and c["sample"]
    if "gpu_launches" in d:
        assert d["gpu_launches"] > 0
    if d.get("check") is not None:  # round 2: the bench checks its own output against the oracle
        c = d["check"]
        err = c["max_rel_err"] if c.get("tol_kind") == "relative" else c["max_abs_err"]
        assert c["ok"] and err <= c["tol"] + 1e-12


@pytest.mark.parametrize("path", [p for p in LINES if "_k1_" in p or "default" in p],
                         ids=lambda p: os.path.basename(p))
def test_k1_cold_start_is_host_link_bound(path):
    """At k = 1 the step moves the non-DHA weight bytes over one link: it cannot beat that bound
    (beyond timing noise) and the measured step should sit close to it."""
    d = _load(path)
    pr = d["path_roofline"]
    assert d["value"] >= 0.97 * pr["R_algorithmic_ms"]
    assert d["value"] <= 1.25 * pr["bound_ms"]
    assert d["roofline"]["bound"] == "pcie"
