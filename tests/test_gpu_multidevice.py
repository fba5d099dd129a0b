"""Parallel transmission across real peers.  These tests need
>= 2 GPUs and skip on a one-GPU box (the one-GPU loopback and two-processes-on-one-GPU variants
of the same paths are in test_gpu_forward / test_gpu_pt_forward / test_gpu_bench_multirank).

* single process, Context([0, 1]): every transport -- dma (secondary H2D into its staging ring +
  cudaMemcpyPeerAsync over NVLink), sm (the forwarder kernel on the secondary storing through the
  peer mapping), ce (the secondary's copy engine straight into the primary's slot) -- gives the
  fp64 oracle's outputs, bit-identical across transports, and the bytes each link carried equal
  the oracle simulator's link_bytes;
* two processes (one per GPU) through bench.py --gpus 2 (it spawns its own ranks): the NCCL
  send/recv gather (dma) and the IPC transports run end to end and the bench's own output check
  against the oracle passes.
"""
import json
import os
import subprocess
import sys

import numpy as np
import pytest

import synth
from oracle import forward as F
from oracle import planner as OP
from oracle import units as OU

torch = pytest.importorskip("torch")
pytestmark = [pytest.mark.gpu,
              pytest.mark.skipif(not torch.cuda.is_available() or torch.cuda.device_count() < 2,
                                 reason="needs >= 2 GPUs")]

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def dp():
    import paper_conf_eurosys_jeongba23_b200 as m
    return m


def fake_cost(m, dtype="fp16"):
    nb = np.array(OU.unit_bytes(m, dtype), dtype=np.int64)
    n = len(nb)
    rng = np.random.default_rng(0)
    load = nb * 1000 // 55_000 + 4000
    exe = rng.integers(3000, 9000, n)
    return {"bytes": nb, "load_ns": load, "fwd_ns": nb // 700, "exe_mem_ns": exe, "exe_dha_ns": exe + load}


@pytest.mark.parametrize("name,S", [("tiny_bert", 32), ("bert_base", 128), ("gpt2", 256)])
@pytest.mark.parametrize("mode", ["PT", "PT_DHA_STRIPE"])
def test_single_process_transports_across_peers(name, S, mode):
    m = synth.SHAPES[name]
    w = synth.make_weights(m, seed=1, dtype="fp16")
    ids = synth.make_ids(m, 1, S, seed=2)
    ref, ref_pool = F.forward(m, w, ids, "fp16")
    ndev = min(torch.cuda.device_count(), 4)
    c = dp().Context(list(range(ndev)))
    model = dp().Model(c, m, w, "fp16")
    cost = fake_cost(m)
    plan = dp().plan_generate(cost, mode, ndev)
    om, osl, ser = OP.plan(cost, mode, ndev)
    link = OP.simulate(cost, om, osl, ndev, ser)["link_bytes"]
    outs = []
    for transport in ("dma", "sm", "ce"):
        c.set_opts(pt_transport=transport)
        out = torch.empty(S, m.hidden, dtype=torch.float16, device="cuda:0")
        pool = torch.empty(1, m.hidden, dtype=torch.float16, device="cuda:0") if m.family != "gpt2" else None
        st = model.infer_cold(plan, 0, torch.from_numpy(ids).cuda(0), out, pool,
                              secondaries=list(range(1, ndev)))
        for d in range(ndev):
            torch.cuda.synchronize(d)
        model.evict(0)
        assert np.abs(out.double().cpu().numpy() - ref.reshape(S, -1)).max() <= 1e-2, transport
        assert st["h2d_bytes"][:ndev] == link and st["nvlink_bytes"][1:ndev] == link[1:], transport
        outs.append(out.clone())
    assert torch.equal(outs[0], outs[1]) and torch.equal(outs[0], outs[2])
    model.close()
    c.close()


@pytest.mark.parametrize("transport", ["dma", "ce", "sm"])
def test_bench_two_processes(transport):
    cmd = [sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2", "--steps", "3", "--warmup", "3", "--quick",
           "--pt-transport", transport]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=900, cwd=ROOT,
                       env={k: v for k, v in os.environ.items() if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK")})
    assert r.returncode == 0, r.stderr[-3000:]
    line = json.loads([x for x in r.stdout.splitlines() if x.startswith("{")][-1])
    assert line["n_gpus"] == 2 and line["check"]["ok"], line.get("check")
    assert line["links"]["slot_ranks"] == [1]
    assert len(line["pcie_rx"]) == 2
