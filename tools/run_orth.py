"""One orthogonalize call at BASELINE config 4 after warm-ups (for ncu; development tool)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_hpdc_zhangbw20_b200 as rg
reps = int(sys.argv[1]) if len(sys.argv) > 1 else 2
m, n = 2097152, 256
h = rg.Handle(0)
A0 = torch.randn(n, m, device="cuda").t()
A = A0.clone()
R = torch.zeros(n, n, device="cuda").t()
for _ in range(reps):
    A.copy_(A0)
    rg.orthogonalize(A, R, orth_tol=1e-5, max_passes=3, handle=h)
torch.cuda.synchronize()
