"""Run RGSQR on BASELINE config 2 (65536 x 4096) `steps` times (for ncu launch lists)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_hpdc_zhangbw20_b200 as rg

m = int(os.environ.get("RG_M", 65536)); n = int(os.environ.get("RG_N", 4096))
steps = int(sys.argv[1]) if len(sys.argv) > 1 else 1
h = rg.Handle(0)
A = torch.randn(n, m, device="cuda").t()
Q = torch.empty(n, m, device="cuda").t(); R = torch.empty(n, n, device="cuda").t()
o = rg.make_opts(sync=False)
for _ in range(steps):
    rg.rgsqr_factor(A, Q=Q, R=R, handle=h, opts=o, check=False)
torch.cuda.synchronize()
print("launches per call", h.last_launches())
