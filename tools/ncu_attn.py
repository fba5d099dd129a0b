"""Launch one attention core (for ncu): python tools/ncu_attn.py S H heads causal [tc]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import paper_conf_eurosys_jeongba23_b200 as dp

S, H, heads, causal = (int(v) for v in sys.argv[1:5])
tc = len(sys.argv) > 5 and sys.argv[5] == "tc"
qkv = torch.randn(S, 3 * H, device="cuda").half()
o = torch.empty(S, H, device="cuda").half()
(dp.attention_tc if tc else dp.attention)(qkv, 3 * H, o, 1, S, H, heads, causal)
torch.cuda.synchronize()
