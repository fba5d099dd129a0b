import math, sys, torch
sys.path.insert(0, '.')
import paper_conf_eurosys_jeongba23_b200 as dp
M,N,K = 128,3072,768
torch.manual_seed(M+N+K)
x = torch.randn(M, K, device="cuda").half()
w = (torch.randn(N, K, device="cuda") / math.sqrt(K)).half()
b = torch.randn(N, device="cuda").half()
r = torch.randn(M, N, device="cuda").half()
y = torch.empty(M, N, device="cuda").half()
ref = (x.float() @ w.float().T + b.float() + r.float())
src = torch.empty(32 << 20, dtype=torch.uint8).pin_memory(); dst = torch.empty(32<<20, dtype=torch.uint8, device="cuda")
side, main = torch.cuda.Stream(), torch.cuda.Stream()
outs = []
for i in range(6):
    if i >= 3:
        with torch.cuda.stream(side):
            dp.pt_forward(src, dst, 16 << 20, stream=side)
    with torch.cuda.stream(main):
        dp.linear(x, K, w, b, r, N, y, N, M, N, K, path=0, stream=main)
    torch.cuda.synchronize()
    err = (y.float() - ref).abs()
    print(i, "maxerr", err.max().item(), "nan", torch.isnan(y).sum().item(), "bad rows", (err.max(1).values > 0.05).nonzero().flatten()[:10].tolist(), "bad cols", (err.max(0).values>0.05).nonzero().flatten()[:10].tolist(), flush=True)
    outs.append(y.clone())
print("equal consecutive", [torch.equal(outs[i], outs[i+1]) for i in range(5)])
