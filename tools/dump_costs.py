"""Profile models on this GPU (dp_profile, median of 10, L2 flushed) and dump the cost tables
(bytes, load_ns, fwd_ns, exe_mem_ns, exe_dha_ns, dha_link_ns) as JSON, for offline planning /
pipeline-model studies (tools/pt_piece_model.py).
python tools/dump_costs.py [model:seq ...] > profiles/r01_cost_tables.json"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np

import paper_conf_eurosys_jeongba23_b200 as dp
import synth

specs = sys.argv[1:] or ["bert_base:128", "bert_large:384", "roberta_large:384", "gpt2_medium:1024"]
ctx = dp.Context([0])
res = {"h2d_gbs": dp.measure_h2d(0)}
for spec in specs:
    name, S = spec.split(":")[0], int(spec.split(":")[1])
    m = synth.SHAPES[name]
    model = dp.Model(ctx, m, synth.make_weights(m, seed=0))
    cost = model.profile(0, 1, S, 10)
    res[spec] = {k: [int(x) for x in np.asarray(v)] for k, v in cost.items()}
    model.close()
ctx.close()
print(json.dumps(res))
