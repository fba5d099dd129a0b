"""GPT-2 tied LM head (dp_lm_head) through the C-ABI vs the fp64 oracle.

* head kernel: logits from the GPU's own last-position hidden rows == oracle.lm_head on the
  same rows within fp32-accumulation error (the forward itself is pinned by
  test_gpu_forward / test_gpu_persist);
* the same kernel reads wte from HBM (resident, wte loaded) or in place from pinned host
  memory (not resident / wte DHA): bit-identical logits;
* errors: BERT -> DP_ERR_UNSUPPORTED.
"""
import numpy as np
import pytest

import synth
from oracle import forward as F

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


def dp():
    import paper_conf_eurosys_jeongba23_b200 as m
    return m


@pytest.mark.parametrize("name,B,S", [("tiny_gpt2", 2, 40), ("tiny_gpt2", 3, 17), ("gpt2", 2, 64)])
def test_lm_head_last_position(name, B, S):
    m = synth.SHAPES[name]
    dtype = "fp16"
    w = synth.make_weights(m, seed=13, dtype=dtype)
    ids = synth.make_ids(m, B, S, seed=14)
    ctx = dp().Context([0])
    model = dp().Model(ctx, m, w, dtype)
    n = model.n
    plan = dp()._lib.PlanArrays(n, np.zeros(n, np.int8), np.zeros(n, np.int8), 1, 1)  # all loaded
    ids_t = torch.from_numpy(ids).cuda()
    out = torch.empty(B * S, m.hidden, dtype=torch.float16, device="cuda")
    model.infer_cold(plan, 0, ids_t, out, None)
    torch.cuda.synchronize()
    last = out[S - 1::S]  # the last position of every sequence (rows S*H apart)
    logits_hbm = torch.empty(B, m.vocab, dtype=torch.float32, device="cuda")
    model.lm_head(0, out[S - 1:], logits_hbm, rows=B, ld_hidden=S * m.hidden)
    torch.cuda.synchronize()
    hid = last.double().cpu().numpy()
    ref = F.lm_head(m, w, hid, dtype)
    bound = 1e-5 * np.abs(hid) @ np.abs(synth.storage_to_f64(w["wte.weight"], dtype)).T + 1e-6
    assert np.all(np.abs(logits_hbm.double().cpu().numpy() - ref) <= bound)
    # the forward's hidden rows themselves vs the oracle (north_star tolerance)
    xr, _ = F.forward(m, w, ids, dtype)
    assert np.abs(hid - xr[:, -1]).max() <= 1e-2
    # wte read in place from host memory after eviction: the same kernel, bit-identical
    model.evict(0)
    logits_host = torch.empty_like(logits_hbm)
    model.lm_head(0, out[S - 1:], logits_host, rows=B, ld_hidden=S * m.hidden)
    torch.cuda.synchronize()
    assert torch.equal(logits_hbm, logits_host)
    model.close()
    ctx.close()


def test_lm_head_rejects_bert():
    m = synth.SHAPES["tiny_bert"]
    ctx = dp().Context([0])
    model = dp().Model(ctx, m, synth.make_weights(m, seed=1), "fp16")
    x = torch.zeros(1, m.hidden, dtype=torch.float16, device="cuda")
    y = torch.zeros(1, m.vocab, dtype=torch.float32, device="cuda")
    with pytest.raises(dp().DeepPlanError):
        model.lm_head(0, x, y)
    model.close()
    ctx.close()
