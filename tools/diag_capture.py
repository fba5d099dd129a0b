import sys, os, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_eurosys_jeongba23_b200 as dp, synth
m = synth.SHAPES["tiny_bert"]; w = synth.make_weights(m, seed=2)
c = dp.Context([0]); c.set_opts(use_graph=1)
base = dp.Model(c, m, w); models = [base.clone() for _ in range(4)]
n = base.n
plan = dp._lib.PlanArrays(n, np.zeros(n, np.int8), None, 1, 1)
ids = torch.from_numpy(synth.make_ids(m, 1, 32)).cuda()
out = torch.empty(32, m.hidden, dtype=torch.float16, device="cuda"); pool = torch.empty(1, m.hidden, dtype=torch.float16, device="cuda")
def t(fn):
    torch.cuda.synchronize(); a = time.perf_counter(); fn(); torch.cuda.synchronize(); return round((time.perf_counter() - a) * 1e3, 3)
for rep in range(3):
    for i, mm in enumerate(models):
        tc = t(lambda: mm.infer_cold(plan, 0, ids, out, pool))
        tw = t(lambda: mm.infer_warm(0, ids, out, pool))
        print(rep, i, "cold_ms", tc, "warm_ms", tw, "pool", c.pool_stats(0), flush=True)
    for mm in models:
        te = t(lambda: mm.evict(0))
        print("evict_ms", te)
c.set_opts(use_graph=0)
for i, mm in enumerate(models):
    print("eager cold", t(lambda: mm.infer_cold(plan, 0, ids, out, pool)), "warm", t(lambda: mm.infer_warm(0, ids, out, pool)))
    mm.evict(0)
