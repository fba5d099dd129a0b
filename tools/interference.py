"""Concurrent cold starts (Table 4 "(2)"): two models cold-start at the
same time and share the host links they use.

* >= 2 GPUs: model A on primary 0 and model B on primary 1, each with parallel transmission over
  both GPUs (k = 2, A borrows GPU 1's link, B borrows GPU 0's): every PCIe link carries two cold
  starts at once -- the paper's 2-GPU interference experiment;
* 1 GPU (fallback): A and B on GPU 0 from two contexts (independent load / execution streams),
  k = 1: both cold starts share the one link.
Each model is timed alone and concurrently (device events on its execution stream, L2 flushed,
evicted between runs, median of --reps); prints one JSON line.

python tools/interference.py [--model bert_base] [--seq 128] [--mode PT_DHA_LINK_STRIPE] [--reps 10]
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import paper_conf_eurosys_jeongba23_b200 as dp
import synth


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--model", default="bert_base")
    ap.add_argument("--seq", type=int, default=128)
    ap.add_argument("--mode", default=None)
    ap.add_argument("--reps", type=int, default=10)
    ap.add_argument("--transport", default="ce", choices=["dma", "sm", "ce"])
    a = ap.parse_args()
    ngpu = torch.cuda.device_count()
    two = ngpu >= 2
    m = synth.SHAPES[a.model]
    w = synth.make_weights(m, seed=0)
    ids_np = synth.make_ids(m, 1, a.seq, seed=1)
    if two:
        ctx = dp.Context([0, 1])
        ctx.set_opts(use_graph=0, pt_transport=a.transport)
        ctxs = [ctx, ctx]
        prim, secs = [0, 1], [[1], [0]]
        mode, k = a.mode or "PT_DHA_LINK_STRIPE", 2
    else:
        ctxs = [dp.Context([0]), dp.Context([0])]
        for c in ctxs:
            c.set_opts(use_graph=1)
        prim, secs = [0, 0], [[], []]
        mode, k = a.mode or "DHA_LINK", 1
    models = [dp.Model(ctxs[i], m, w) for i in range(2)]
    cost = models[0].profile(0, 1, a.seq, 5)
    plan = dp.plan_generate(cost, mode, k)
    streams, bufs = [], []
    for i in range(2):
        with torch.cuda.device(prim[i]):
            streams.append(torch.cuda.Stream())
            ids = torch.from_numpy(ids_np).cuda()
            out = torch.empty(a.seq, m.hidden, dtype=torch.float16, device="cuda")
            pool = torch.empty(1, m.hidden, dtype=torch.float16, device="cuda") if m.family != "gpt2" else None
            flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
            bufs.append((ids, out, pool, flush))

    def once(which):
        evs = []
        for i in range(2):
            if models[i].is_resident(prim[i]):
                models[i].evict(prim[i])
            bufs[i][3].fill_(1)
        for d in set(prim):
            torch.cuda.synchronize(d)
        for i in which:
            with torch.cuda.device(prim[i]):
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(streams[i])
                ids, out, pool, _ = bufs[i]
                models[i].infer_cold(plan, prim[i], ids, out, pool, secondaries=secs[i], stream=streams[i])
                e1.record(streams[i])
                evs.append((i, e0, e1))
        for d in set(prim):
            torch.cuda.synchronize(d)
        return {i: e0.elapsed_time(e1) for i, e0, e1 in evs}

    for _ in range(3):
        once([0, 1])
    solo = {0: [], 1: []}
    conc = {0: [], 1: []}
    for _ in range(a.reps):
        for i in (0, 1):
            solo[i].append(once([i])[i])
        r = once([0, 1])
        for i in (0, 1):
            conc[i].append(r[i])
    res = {"model": a.model, "seq": a.seq, "mode": mode, "k": k, "gpus": 2 if two else 1,
           "setup": ("A on GPU 0, B on GPU 1, each PT over both links" if two else
                     "A and B on GPU 0 from two contexts, sharing its link"),
           "transport": a.transport if two else None}
    for i, nm in ((0, "A"), (1, "B")):
        s, c = float(np.median(solo[i])), float(np.median(conc[i]))
        res[nm] = {"solo_ms": round(s, 4), "concurrent_ms": round(c, 4), "slowdown": round(c / s, 3)}
    print(json.dumps(res), flush=True)
    for i in range(2):
        if models[i].is_resident(prim[i]):
            models[i].evict(prim[i])
        models[i].close()
    for c in {id(c): c for c in ctxs}.values():
        c.close()


if __name__ == "__main__":
    main()
