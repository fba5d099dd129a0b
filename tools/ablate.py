"""Where the warm forward's time goes in the chain: the same warm forward (graph replay, L2
flushed) with whole kernel families skipped (DP_ABLATE bit mask: 1 attention, 2 LayerNorm,
4 resident GEMM, 8 skinny/GEMV), each in its own process.  Outputs are garbage; the time a
family's removal saves is its share of the chained forward (PDL overlap included).
python tools/ablate.py [model:seq ...]

Needs the instrumented library (the release build compiles DP_ABLATE out):
    DP_NVCC_EXTRA=-DDP_INSTRUMENT python paper_conf_eurosys_jeongba23_b200/build.py"""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
specs = sys.argv[1:] or ["bert_base:128"]
CHILD = r'''
import json, sys
sys.path.insert(0, ROOT)
import numpy as np, torch
import paper_conf_eurosys_jeongba23_b200 as dp, synth
name, S = SPEC.split(":"); S = int(S)
m = synth.SHAPES[name]
ctx = dp.Context([0]); model = dp.Model(ctx, m, synth.make_weights(m, seed=0))
ids = torch.from_numpy(synth.make_ids(m, 1, S)).cuda()
out = torch.empty(S, m.hidden, dtype=torch.float16, device="cuda")
pool = torch.empty(1, m.hidden, dtype=torch.float16, device="cuda") if m.family != "gpt2" else None
model.infer_cold(dp._lib.PlanArrays(model.n, np.zeros(model.n, np.int8), None, 1, 1), 0, ids, out, pool)
torch.cuda.synchronize()
ctx.set_opts(use_graph=1)
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
ts = []
for i in range(35):
    flush.fill_(i)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record(); st = model.infer_warm(0, ids, out, pool); e1.record()
    torch.cuda.synchronize()
    if i >= 5: ts.append(e0.elapsed_time(e1))
print(json.dumps({"warm_ms": round(float(np.median(ts)), 4)}))
'''
for spec in specs:
    child = CHILD.replace("ROOT", repr(ROOT)).replace("SPEC", repr(spec))
    for mask, what in ((0, "all"), (1, "no attention"), (2, "no LayerNorm"), (4, "no GEMM"), (8, "no skinny/GEMV"),
                       (1 | 2, "no attention, no LN"), (1 | 2 | 8, "GEMMs only"), (1 | 4 | 8, "LN only"),
                       (2 | 4 | 8, "attention only"), (15, "embedding only")):
        env = dict(os.environ, DP_ABLATE=str(mask))
        r = subprocess.run([sys.executable, "-c", child], env=env, capture_output=True, text=True, timeout=600)
        res = json.loads(r.stdout.strip().splitlines()[-1]) if r.returncode == 0 else {"error": r.stderr[-400:]}
        print(json.dumps({"model": spec, "mask": mask, "kept": what, **res}), flush=True)
