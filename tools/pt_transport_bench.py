"""PT transports on ONE GPU, in loopback: every slot is served by the same device,
so all k "links" are the same PCIe link -- this measures the MECHANISM cost of each transport
(copy-engine DMA into a staging ring + peer copy, the SM forwarder kernel, a direct DMA into
the slot), not the multi-link speedup.  Cold-start latency (CUDA-graph replay, L2 flushed,
device-timed with CUDA events), the k = 1 plan beside it.
python tools/pt_transport_bench.py [model] [seq] [steps]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import paper_conf_eurosys_jeongba23_b200 as dp
import synth

name = sys.argv[1] if len(sys.argv) > 1 else "bert_base"
S = int(sys.argv[2]) if len(sys.argv) > 2 else 128
steps = int(sys.argv[3]) if len(sys.argv) > 3 else 10
m = synth.SHAPES[name]
w = synth.make_weights(m, seed=0, dtype="fp16")
ids = torch.from_numpy(synth.make_ids(m, 1, S, seed=1)).cuda()
ctx = dp.Context([0])
model = dp.Model(ctx, m, w, "fp16")
cost = model.profile(0, 1, S, 5)
out = torch.empty(S, m.hidden, dtype=torch.float16, device="cuda")
pooled = torch.empty(1, m.hidden, dtype=torch.float16, device="cuda") if m.family != "gpt2" else None
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
stream = torch.cuda.Stream()
res = []
ref = None
bad = []
cases = [tuple(c.split("/")) for c in os.environ.get("DP_PT_CASES", "").split(",") if c] or \
    [("PIPESWITCH", "1"), ("PT", "2"), ("PT", "4"), ("PT_DHA_LINK_BAL", "4")]
for mode, k in ((m_, int(k_)) for m_, k_ in cases):
    plan = dp.plan_generate(cost, mode, k)
    for tr in (("dma",) if k == 1 else ("dma", "sm", "ce")):
        ctx.set_opts(pt_transport=tr, use_graph=1)
        ts = []
        for i in range(steps + 3):
            if model.is_resident(0):
                model.evict(0)
            flush.fill_(i)
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            with torch.cuda.stream(stream):
                e0.record(stream)
                st = model.infer_cold(plan, 0, ids, out, pooled, secondaries=[0] * (k - 1), stream=stream)
                e1.record(stream)
            torch.cuda.synchronize()
            if i >= 3:
                ts.append(e0.elapsed_time(e1))
            if ref is None:
                ref = out.clone()
            if not torch.equal(out, ref):  # same kernels, same weights: must be bit-identical
                wo = torch.empty_like(out)
                model.infer_warm(0, ids, wo, pooled)
                torch.cuda.synchronize()
                bad.append({"mode": mode, "k": k, "transport": tr, "iter": i, "rows": int((out != ref).any(1).sum()),
                            "finite": bool(torch.isfinite(out).all()), "warm_ok": bool(torch.equal(wo, ref))})
                print(json.dumps({"MISMATCH": bad[-1]}), flush=True)
        res.append({"model": name, "seq": S, "mode": mode, "k": k, "transport": tr,
                    "ms_mean": round(float(np.mean(ts)), 4), "ms_min": round(float(np.min(ts)), 4),
                    "h2d_bytes": st["h2d_bytes"][:k], "nvlink_bytes": st["nvlink_bytes"][:k],
                    "copies": st["n_copies"]})
        print(json.dumps(res[-1]), flush=True)
print(json.dumps({"mismatches": len(bad)}), flush=True)
model.evict(0) if model.is_resident(0) else None
model.close()
ctx.close()
