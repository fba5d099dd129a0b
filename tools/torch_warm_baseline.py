"""Library baseline for the warm forward (the T_warm term of the path roofline): the same model,
weights and input run by transformers + PyTorch on the B200 (fp16, SDPA attention, cuBLAS
GEMMs), captured in a CUDA graph and replayed; L2 flushed between runs; CUDA events on the
replay stream; median of N.  Also checks the library output against ours (max-abs).
Tool only (never imported by the product path).
python tools/torch_warm_baseline.py [model:seq ...]   (default bert_base:128 bert_large:384 gpt2:256)"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import paper_conf_eurosys_jeongba23_b200 as dp
import synth

specs = sys.argv[1:] or ["bert_base:128", "bert_large:384", "gpt2:256"]
N = int(os.environ.get("DP_N", "30"))
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")


def hf_model(m, weights):
    from transformers import BertConfig, BertModel, GPT2Config, GPT2Model, RobertaConfig, RobertaModel
    if m.family in ("bert", "roberta"):
        C, M = (BertConfig, BertModel) if m.family == "bert" else (RobertaConfig, RobertaModel)
        kw = dict(pad_token_id=m.pad_idx) if m.family == "roberta" else {}
        cfg = C(vocab_size=m.vocab, hidden_size=m.hidden, num_hidden_layers=m.layers, num_attention_heads=m.heads,
                intermediate_size=m.ffn, max_position_embeddings=m.max_pos, type_vocab_size=m.type_vocab,
                layer_norm_eps=m.ln_eps, hidden_act="gelu", attn_implementation="sdpa", **kw)
        model = M(cfg)
    else:
        cfg = GPT2Config(vocab_size=m.vocab, n_embd=m.hidden, n_layer=m.layers, n_head=m.heads, n_positions=m.max_pos,
                         n_inner=m.ffn, activation_function="gelu_new", layer_norm_epsilon=m.ln_eps,
                         resid_pdrop=0.0, embd_pdrop=0.0, attn_pdrop=0.0, attn_implementation="sdpa")
        model = GPT2Model(cfg)
    sd = {k: torch.from_numpy(np.asarray(v).view(np.float16).astype(np.float32)) for k, v in weights.items()}
    model.load_state_dict(sd, strict=False)
    return model.half().cuda().eval()


def timed(fn):
    s = torch.cuda.current_stream()
    ts = []
    for i in range(N + 5):
        flush.fill_(i & 0xFF)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record(s)
        fn()
        e1.record(s)
        torch.cuda.synchronize()
        if i >= 5:
            ts.append(e0.elapsed_time(e1))
    return float(np.median(ts))


ctx = dp.Context([0])
ctx.set_opts(use_graph=1)
for spec in specs:
    name, S = spec.split(":")[0], int(spec.split(":")[1])
    m = synth.SHAPES[name]
    w = synth.make_weights(m, seed=0)
    ids_np = synth.make_ids(m, 1, S)
    ids = torch.from_numpy(ids_np).cuda()
    # ours: all units resident, warm graph replay
    model = dp.Model(ctx, m, w)
    out = torch.empty(S, m.hidden, dtype=torch.float16, device="cuda")
    pool = torch.empty(1, m.hidden, dtype=torch.float16, device="cuda") if m.family != "gpt2" else None
    plan = dp._lib.PlanArrays(model.n, np.zeros(model.n, np.int8), None, 1, 1)
    model.infer_cold(plan, 0, ids, out, pool)
    torch.cuda.synchronize()
    ours = timed(lambda: model.infer_warm(0, ids, out, pool))
    # library: transformers fp16 on cuBLAS / SDPA, one CUDA graph
    hf = hf_model(m, w)
    ids_l = ids.long()
    with torch.no_grad():
        for _ in range(3):
            hf(input_ids=ids_l)
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g):
            o = hf(input_ids=ids_l).last_hidden_state
    lib = timed(g.replay)
    diff = float((o.reshape(S, -1).float() - out.float()).abs().max())
    print(json.dumps({"model": name, "seq": S, "ours_warm_ms": round(ours, 4), "torch_cublas_graph_ms": round(lib, 4),
                      "speedup": round(lib / ours, 3), "max_abs_diff": diff, "l2_flushed": True}), flush=True)
    model.close()
    del hf, g
ctx.close()
