"""bench.py's N > 1 path on a one-GPU box (GPU): two ranks under torch.distributed.run, both on
device 0 (DP_BENCH_ONE_GPU=1, gloo process group), PT slot 1 served by rank 1 over the CUDA
IPC transports (sm / ce).  Checks the whole multi-rank control flow -- plan broadcast, IPC
exchange, timed region with barriers, max-over-ranks, e2e, the warm measurement after the
secondaries leave -- ends in one valid JSON line with the per-link bytes of the plan."""
import json
import os
import socket
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


@pytest.mark.parametrize("transport", ["sm", "ce"])
def test_bench_two_ranks_one_gpu(transport):
    env = dict(os.environ, DP_BENCH_ONE_GPU="1")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2", "--master-addr",
           "127.0.0.1", "--master-port", str(_port()), os.path.join(ROOT, "bench.py"), "--gpus", "2", "--steps", "3",
           "--warmup", "3", "--model", "tiny_bert", "--seq", "32", "--quick", "--no-cpu-baseline",
           "--profile-iters", "2", "--pt-transport", transport]
    r = subprocess.run(cmd, cwd=ROOT, env=env, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["value"] > 0 and d["config"]["pt_transport"] == transport
    assert d["e2e"]["value"] > 0
    links = d["links"]
    assert len(links["h2d_solo_gbs"]) == 2 and len(links["pair_gbs"]) == 2 and links["slot_ranks"] == [1]
    assert [p["rank"] for p in d["pcie_rx"]] == [0, 1]


def test_bench_spawns_its_own_ranks():
    """`python bench.py --gpus 2` without a launcher (no WORLD_SIZE) re-launches itself under
    torch.distributed.run; the line carries the output check against the oracle."""
    env = {k: v for k, v in os.environ.items() if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK")}
    env["DP_BENCH_ONE_GPU"] = "1"
    cmd = [sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2", "--steps", "3", "--warmup", "3", "--model",
           "tiny_bert", "--seq", "32", "--quick", "--profile-iters", "2", "--pt-transport", "ce"]
    r = subprocess.run(cmd, cwd=ROOT, env=env, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["check"]["ok"] and d["cpu_baseline"]["kind"] == "oracle"
