"""Launch the tcgen05 GEMM once per forced tile configuration (for ncu: -k regex:gemm_tc).
python tools/ncu_gemm_cfgs.py M,N,K,bn [M,N,K,bn ...]"""
import math
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import paper_conf_eurosys_jeongba23_b200 as dp

for spec in sys.argv[1:]:
    M, N, K, bn = (int(v) for v in spec.split(","))
    x = torch.randn(M, K, device="cuda").half()
    w = (torch.randn(N, K, device="cuda") / math.sqrt(K)).half()
    y = torch.empty(M, N, device="cuda").half()
    dp.gemm_tc(x, K, w, None, None, 0, y, N, M, N, K, bn=bn)
    torch.cuda.synchronize()
