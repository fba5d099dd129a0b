"""SM-driven PT forwarder (the design alternative of PAPER.md P:182) on the GPU.

* the forwarder kernel (dp_pt_forward) moves every byte of host-mapped memory into HBM
  exactly, for sizes spanning the 16-byte vector path, a sub-vector tail, one CTA, several
  waves and a grid-stride loop;
* a cold start whose PT slots use the forwarder (opts.pt_transport = "sm") gives the same
  outputs, bit for bit, as the copy-engine + staging-ring path (same kernels, same weights) and
  the fp64 oracle's within the north_star tolerance; the bytes over each link and over NVLink
  equal the oracle simulator's link_bytes bit-exactly;
* event gating holds under fault injection (slow forwarders, NaN-poisoned slots) and in
  CUDA-graph replay;
* the copy-engine variant (pt_transport = "ce": one DMA per piece straight into the primary's
  slot, no staging ring) satisfies the same checks;
* across processes (CUDA IPC, no NCCL): rank 1 forwards its slot into rank 0's HBM through
  the IPC mapping and releases done words that rank 0's execution stream acquires.  Both
  ranks run on this one GPU (loopback across processes) -- the protocol (go / done epochs,
  last-CTA release, waits before the first kernel of a piece) is exactly the multi-GPU one.
"""
import ctypes
import os
import socket

import numpy as np
import pytest

import synth
from oracle import forward as F
from oracle import planner as OP

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

DT = {"fp16": torch.float16, "bf16": torch.bfloat16}


def dp():
    import paper_conf_eurosys_jeongba23_b200 as m
    return m


def f64(t):
    return t.float().cpu().numpy().astype(np.float64)


def fake_cost(m, dtype, seed=0):
    from oracle import units as OU
    nb = np.array(OU.unit_bytes(m, dtype), dtype=np.int64)
    rng = np.random.default_rng(seed)
    n = len(nb)
    load = nb * 1000 // 55_000 + 4000
    exe = rng.integers(3000, 9000, n)
    kinds = [u[1] for u in OU.unit_params(m)]
    dha = np.where(np.array(kinds) == "emb", exe + 2000, exe + load + rng.integers(-6000, 6000, n))
    return {"bytes": nb, "load_ns": load, "fwd_ns": nb // 700, "exe_mem_ns": exe, "exe_dha_ns": np.maximum(dha, 0)}


@pytest.mark.parametrize("nbytes", [1, 15, 16, 17, 4096 + 3, 16 * 1024 + 16, (1 << 20) + 9, (37 << 20) + 5])
def test_forwarder_copies_every_byte(nbytes):
    rng = np.random.default_rng(nbytes)
    src = dp().host_alloc(nbytes + 64)
    try:
        data = rng.integers(0, 256, nbytes + 64, dtype=np.uint8)
        ctypes.memmove(src, data.ctypes.data, nbytes + 64)
        dst = torch.full((nbytes + 64,), 0xAB, dtype=torch.uint8, device="cuda")
        dp().pt_forward(src, dst.data_ptr() + 16, nbytes)
        torch.cuda.synchronize()
        got = dst.cpu().numpy()
        assert np.array_equal(got[16:16 + nbytes], data[:nbytes])
        assert np.all(got[:16] == 0xAB) and np.all(got[16 + nbytes:] == 0xAB)  # nothing outside
    finally:
        dp().host_free(src)


def test_forwarder_rejects_misaligned():
    src = dp().host_alloc(256)
    try:
        dst = torch.empty(256, dtype=torch.uint8, device="cuda")
        with pytest.raises(dp().DeepPlanError):
            dp().pt_forward(src + 4, dst.data_ptr(), 64)
    finally:
        dp().host_free(src)


def _run(model, plan, ids_np, dtype, k):
    H = model.shape.hidden
    B, S = ids_np.shape
    ids = torch.from_numpy(ids_np).cuda()
    out = torch.empty(B * S, H, dtype=DT[dtype], device="cuda")
    pool = torch.empty(B, H, dtype=DT[dtype], device="cuda") if model.shape.family != "gpt2" else None
    st = model.infer_cold(plan, 0, ids, out, pool, secondaries=[0] * (k - 1))
    torch.cuda.synchronize()
    model.evict(0)
    return out, pool, st


@pytest.mark.parametrize("name,B,S", [("tiny_bert", 2, 77), ("tiny_gpt2", 1, 70), ("tiny_roberta", 2, 50),
                                      ("bert_base", 1, 128)])
@pytest.mark.parametrize("mode,k", [("PT", 2), ("PT_DHA", 3), ("PT_DHA_LINK_BAL", 4), ("PT_DHA_LINK_STRIPE", 8)])
@pytest.mark.parametrize("transport", ["sm", "ce"])
def test_sm_transport_equals_dma_and_oracle(name, B, S, mode, k, transport):
    m = synth.SHAPES[name]
    dtype = "fp16"
    w = synth.make_weights(m, seed=21, dtype=dtype)
    ids = synth.make_ids(m, B, S, seed=22)
    ref, ref_pool = F.forward(m, w, ids, dtype)
    c = dp().Context([0])
    model = dp().Model(c, m, w, dtype)
    cost = fake_cost(m, dtype, seed=5)
    plan = dp().plan_generate(cost, mode, k)
    c.set_opts(pt_transport="dma")
    a, pa, sa = _run(model, plan, ids, dtype, k)
    c.set_opts(pt_transport=transport)
    b, pb, sb = _run(model, plan, ids, dtype, k)
    assert torch.equal(a, b)
    if pa is not None:
        assert torch.equal(pa, pb)
    assert np.abs(f64(b) - ref.reshape(B * S, -1)).max() <= 1e-2
    om, osl, ser = OP.plan(cost, mode, k)
    link = OP.simulate(cost, om, osl, k, ser)["link_bytes"]
    assert sb["h2d_bytes"][:k] == link and sa["h2d_bytes"][:k] == link
    assert sb["nvlink_bytes"][1:k] == link[1:]
    if transport == "sm":
        assert sb["n_copies"] < sa["n_copies"] or sum(link[1:]) == 0  # PT pieces need no DMA
    else:
        assert sb["n_copies"] <= sa["n_copies"]  # one DMA per piece instead of DMA + peer copy
    model.close()
    c.close()


@pytest.mark.parametrize("use_graph", [0, 1])
@pytest.mark.parametrize("transport", ["sm", "ce"])
def test_sm_transport_event_gating_and_graph(use_graph, transport):
    """Forwarders stalled 200 us before every piece + slots poisoned with NaN on eviction:
    a kernel that ran before its piece landed would read NaN.  Repeated (graph) replays must
    equal the undelayed eager run bit for bit."""
    m = synth.SHAPES["tiny_bert"]
    dtype = "fp16"
    w = synth.make_weights(m, seed=23, dtype=dtype, recipe="scaled")
    ids = synth.make_ids(m, 1, 32, seed=24)
    c = dp().Context([0])
    model = dp().Model(c, m, w, dtype)
    plan = dp().plan_generate(fake_cost(m, dtype, seed=2), "PT_DHA", 3)
    c.set_opts(pt_transport=transport, chunk_bytes=4096, debug_poison=1)
    base, pbase, _ = _run(model, plan, ids, dtype, 3)
    c.set_opts(debug_delay_us=200, use_graph=use_graph)
    for _ in range(3):
        out, pool, _ = _run(model, plan, ids, dtype, 3)
        assert torch.isfinite(out).all()
        assert torch.equal(out, base) and torch.equal(pool, pbase)
    model.close()
    c.close()


# ---------------------------------------------------------------------------------------
# Across processes (CUDA IPC mailboxes; both ranks on this one GPU)
# ---------------------------------------------------------------------------------------

def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _ipc_worker(rank, world, port, name, mode, S, delay_us, transport, q, graph=0):
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import paper_conf_eurosys_jeongba23_b200 as D
        torch.cuda.set_device(0)
        m = synth.SHAPES[name]
        dtype = "fp16"
        w = synth.make_weights(m, seed=31, dtype=dtype)
        c = D.Context([0])
        c.peer_init_ipc(rank, world)
        c.set_opts(pt_transport=transport, debug_poison=1, chunk_bytes=1 << 20, use_graph=graph,
                   debug_delay_us=delay_us if rank > 0 else 0)
        model = D.Model(c, m, w, dtype)
        blocks = [None] * world
        dist.all_gather_object(blocks, model.ipc_export())
        model.ipc_import(blocks)
        cost = fake_cost(m, dtype, seed=7)
        plan = D.plan_generate(cost, mode, world)
        ids_np = synth.make_ids(m, 1, S, seed=32)
        outs, stats = [], []
        ids = torch.from_numpy(ids_np).cuda()
        out = torch.empty(S, m.hidden, dtype=torch.float16, device="cuda")  # fixed: graphs replay
        for _ in range(3):  # three epochs: go / done words are never reset
            if rank == 0:
                out.fill_(0)
                st = model.infer_cold(plan, 0, ids, out, None)
                torch.cuda.synchronize()
                outs.append(out.cpu())
                model.evict(0)
            else:
                st = model.infer_cold_raw(plan, 0, None, 1, S, None, None, None)
                torch.cuda.synchronize()
            stats.append((list(st["h2d_bytes"]), list(st["nvlink_bytes"])))
        if rank == 0:
            ref, _ = F.forward(m, w, ids_np, dtype)
            err = float(np.abs(outs[0].double().numpy() - ref.reshape(S, -1)).max())
            same = all(torch.equal(outs[0], o) for o in outs[1:])
            finite = all(bool(torch.isfinite(o).all()) for o in outs)
            om, osl, ser = OP.plan(cost, mode, world)
            link = OP.simulate(cost, om, osl, world, ser)["link_bytes"]
            q.put((rank, {"err": err, "same": same, "finite": finite, "stats": stats, "link": link}))
        else:
            q.put((rank, {"stats": stats}))
        dist.barrier()
        model.close()
        c.close()
    except Exception as e:  # pragma: no cover - reported to the parent
        q.put((rank, {"error": repr(e)}))
        raise
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("name,mode,S,delay", [("tiny_bert", "PT", 32, 0), ("tiny_gpt2", "PT_DHA", 40, 300),
                                               ("bert_base", "PT_DHA_BAL", 128, 0),
                                               ("bert_base", "PT_DHA_LINK_STRIPE", 128, 0)])
@pytest.mark.parametrize("transport,graph", [("sm", 0), ("ce", 0), ("ce", 1), ("sm", 1)])
def test_sm_transport_across_processes(name, mode, S, delay, transport, graph):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_ipc_worker, args=(r, 2, port, name, mode, S, delay, transport, q, graph)) for r in range(2)]
    for p in procs:
        p.start()
    res = {}
    try:
        for _ in range(2):
            r, d = q.get(timeout=300)
            res[r] = d
    finally:
        for p in procs:
            p.join(timeout=60)
            if p.is_alive():
                p.kill()
    assert "error" not in res[0] and "error" not in res[1], res
    r0, r1 = res[0], res[1]
    assert r0["finite"] and r0["same"]
    assert r0["err"] <= 1e-2
    link = r0["link"]
    for h2d, nvl in r1["stats"]:  # the secondary's reads over its own link = slot 1's bytes
        assert h2d[1] == link[1] and nvl[1] == link[1]
    for h2d, nvl in r0["stats"]:
        assert h2d[0] == link[0] and nvl[1] == link[1]


@pytest.mark.parametrize("name,S", [("tiny_bert", 77), ("tiny_gpt2", 70), ("bert_base", 128)])
@pytest.mark.parametrize("transport", ["sm", "ce"])
def test_one_hop_transports_bf16_striped(name, S, transport):
    """bf16 storage, the striped plan (R22) over 4 loopback links: one-hop transports equal the
    DMA path bit for bit and stay within the bf16 tolerance (R15) of the oracle: 1e-2 + the
    representation error of bf16 activations (the oracle with bf16 roundings where the kernels
    round) of the exact oracle."""
    m = synth.SHAPES[name]
    dtype = "bf16"
    w = synth.make_weights(m, seed=61, dtype=dtype)
    ids = synth.make_ids(m, 1, S, seed=62)
    ref, _ = F.forward(m, w, ids, dtype)
    emul, _ = F.forward(m, w, ids, dtype, act_round=dtype)  # bf16 representation error (R15)
    rep = float(np.abs(emul - ref).max())
    c = dp().Context([0])
    model = dp().Model(c, m, w, dtype)
    plan = dp().plan_generate(fake_cost(m, dtype, seed=9), "PT_DHA_LINK_STRIPE", 4)
    c.set_opts(pt_transport="dma")
    a, _, sa = _run(model, plan, ids, dtype, 4)
    c.set_opts(pt_transport=transport)
    b, _, sb = _run(model, plan, ids, dtype, 4)
    assert torch.equal(a, b)
    r = ref.reshape(S, -1)
    assert np.abs(f64(b) - r).max() <= 1e-2 + rep
    assert sa["h2d_bytes"] == sb["h2d_bytes"] and sa["nvlink_bytes"] == sb["nvlink_bytes"]
    model.close()
    c.close()
