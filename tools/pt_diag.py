"""Diagnose a PT-transport mismatch: cold starts per transport vs the PIPESWITCH output, and
after each mismatching cold start a warm run (are the slots corrupted, or was it transient?);
then warm runs beside the forwarder noise kernel (is the forward itself contention-safe?).
python tools/pt_diag.py model seq"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import paper_conf_eurosys_jeongba23_b200 as dp
import synth

name, S = sys.argv[1], int(sys.argv[2])
m = synth.SHAPES[name]
w = synth.make_weights(m, seed=0, dtype="fp16")
ids = torch.from_numpy(synth.make_ids(m, 1, S, seed=1)).cuda()
ctx = dp.Context([0])
model = dp.Model(ctx, m, w, "fp16")
cost = model.profile(0, 1, S, 3)
out = torch.empty(S, m.hidden, dtype=torch.float16, device="cuda")
wout = torch.empty_like(out)
pooled = torch.empty(1, m.hidden, dtype=torch.float16, device="cuda")


def run(mode, k, tr, graph, reps=6):
    plan = dp.plan_generate(cost, mode, k)
    ctx.set_opts(pt_transport=tr, use_graph=graph)
    rows = []
    for i in range(reps):
        if model.is_resident(0):
            model.evict(0)
        model.infer_cold(plan, 0, ids, out, pooled, secondaries=[0] * (k - 1))
        torch.cuda.synchronize()
        row = {"cold_mismatch": int((out != ref).sum()) if ref is not None else 0}
        if row["cold_mismatch"]:
            model.infer_warm(0, ids, wout, pooled)
            torch.cuda.synchronize()
            row["warm_mismatch_after"] = int((wout != ref).sum())
            bad = (out != ref).any(dim=1).nonzero().flatten()
            row["bad_rows"] = [int(bad[0]), int(bad[-1]), int(bad.numel())]
        rows.append(row)
    return rows


ref = None
run("PIPESWITCH", 1, "dma", 0, 1)
ref = out.clone()
for args in [("PT", 2, "sm", 0), ("PT", 2, "sm", 1), ("PT", 4, "sm", 0), ("PT_DHA_LINK_BAL", 4, "sm", 0),
             ("PT", 2, "ce", 0), ("PT", 2, "dma", 0)]:
    print(json.dumps({"args": args, "runs": run(*args)}), flush=True)

# warm forward beside the forwarder noise
if model.is_resident(0):
    model.evict(0)
ctx.set_opts(pt_transport="dma", use_graph=0)
model.infer_cold(dp.plan_generate(cost, "PIPESWITCH", 1), 0, ids, out, pooled)
torch.cuda.synchronize()
src = torch.empty(256 << 20, dtype=torch.uint8).pin_memory()
dst = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
side, main = torch.cuda.Stream(), torch.cuda.Stream()
bad = 0
for i in range(100):
    with torch.cuda.stream(side):
        dp.pt_forward(src, dst, 128 << 20, stream=side)
    with torch.cuda.stream(main):
        model.infer_warm(0, ids, wout, pooled, stream=main)
    torch.cuda.synchronize()
    bad += int(not torch.equal(wout, ref))
print(json.dumps({"warm_beside_noise_mismatches": bad, "of": 100}), flush=True)
