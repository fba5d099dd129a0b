"""Multi-process parallel transmission, host side, on CPU (gloo, world size 2).

Each rank derives the plan (PT_DHA, k = 2) from the same cost table with the product
planner and the transfer schedule of slot 1 with dp_transfer_schedule -- rank 1 as the
sender (its own PCIe link), rank 0 as the receiver (the NVLink gather).  The data path is
emulated with gloo send/recv of the arena bytes, piece by piece, in schedule order: the
primary must end up with exactly the slot-1 units' bytes at their arena offsets, and the
number of bytes gathered must equal the oracle simulator's link_bytes[1] bit-exactly.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import synth


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _cost(name):
    import paper_conf_eurosys_jeongba23_b200._lib as L
    m = synth.SHAPES[name]
    nb = L.config_units(m)
    n = len(nb)
    rng = np.random.default_rng(4)
    exe = rng.integers(3000, 9000, n)
    load = nb * 1000 // 55_000 + 4000
    return m, {"bytes": nb, "load_ns": load, "fwd_ns": nb // 700, "exe_mem_ns": exe,
               "exe_dha_ns": exe + rng.integers(0, 3000, n)}


def _worker(rank, world, port, name, chunk, q, mode="PT_DHA"):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import paper_conf_eurosys_jeongba23_b200._lib as L
        m, cost = _cost(name)
        plan = L.plan_generate(cost, mode, world)
        # every rank derives the identical plan
        mine = torch.from_numpy(plan.method.astype(np.int64))
        other = mine.clone()
        dist.broadcast(other, src=0)
        assert torch.equal(mine, other)
        off, nb, fu, lu = L.transfer_schedule(m, plan, 1, chunk)
        units = L.config_units(m)
        total = int(sum(units)) + 256 * len(units)
        arena = (np.arange(total, dtype=np.int64) * 2654435761 % 251).astype(np.uint8)  # synthetic bytes
        if rank == 1:  # secondary: serve slot 1 = rank (0 + 1) % 2
            for o, b in zip(off, nb):
                dist.send(torch.from_numpy(arena[o:o + b].copy()), dst=0)
        else:
            dest = np.zeros(total, dtype=np.uint8)
            got = 0
            for o, b in zip(off, nb):
                buf = torch.empty(int(b), dtype=torch.uint8)
                dist.recv(buf, src=1)
                dest[o:o + b] = buf.numpy()
                got += int(b)
            q.put(("ok", got, dest.tobytes(), [int(x) for x in plan.method], [int(x) for x in plan.slot]))
    except Exception as e:  # pragma: no cover
        q.put(("err", repr(e)))
        raise
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("name,chunk,mode", [("tiny_bert", 4096, "PT_DHA"), ("tiny_gpt2", 1 << 20, "PT_DHA"),
                                             ("bert_base", 4 << 20, "PT_DHA"),
                                             ("bert_base", 4 << 20, "PT_DHA_LINK_STRIPE"),
                                             ("tiny_gpt2", 1 << 20, "PT_DHA_STRIPE")])
def test_pt_gather_schedule_gloo(name, chunk, mode):
    from oracle import planner as OP
    from oracle import units as OU
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, name, chunk, q, mode)) for r in range(2)]
    for p in procs:
        p.start()
    res = q.get(timeout=300)
    for p in procs:
        p.join(timeout=60)
    assert res[0] == "ok", res
    _, got, dest, method, slot = res
    m, cost = _cost(name)
    om, osl, _ = OP.plan(cost, mode, 2)
    assert method == om and slot == osl
    link = OP.simulate(cost, om, osl, 2, link_aware=mode in OP.LINK_AWARE)["link_bytes"]
    assert got == link[1]
    # the bytes of every slot-1 unit arrived at its arena offset, nothing else was written
    import paper_conf_eurosys_jeongba23_b200._lib as L
    units = L.config_units(m)
    total = int(sum(units)) + 256 * len(units)
    arena = (np.arange(total, dtype=np.int64) * 2654435761 % 251).astype(np.uint8)
    dest = np.frombuffer(dest, dtype=np.uint8)
    off = 0
    covered = np.zeros(total, dtype=bool)
    for u, b in enumerate(units):
        off = (off + 255) & ~255
        if slot[u] == 1:
            assert np.array_equal(dest[off:off + b], arena[off:off + b]), u
            covered[off:off + b] = True
        off += int(b)
    assert not dest[~covered].any()
    assert sum(b for u, b in enumerate(units) if slot[u] == 1) == got
    assert OU.model_bytes(m) == int(sum(units))
