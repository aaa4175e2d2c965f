"""One call each of ls_solve_refined (config 3 shape), orthogonalize (config 4) and lowrank_approx
(config 5) after warm-ups, eagerly (RGSQR_NO_GRAPH=1 recommended) -- for ncu (development tool)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_hpdc_zhangbw20_b200 as rg
which = sys.argv[1] if len(sys.argv) > 1 else "all"
h = rg.Handle(0)
if which in ("all", "ls"):
    m, n = 131072, 1024
    A = torch.randn(n, m, device="cuda").t()
    b = torch.randn(m, device="cuda")
    for _ in range(2):
        rg.ls_solve_refined(A, b, handle=h)
    del A
if which in ("all", "orth"):
    m, n = 2097152, 256
    A0 = torch.randn(n, m, device="cuda").t()
    A = A0.clone()
    for _ in range(2):
        A.copy_(A0)
        rg.orthogonalize(A, None, orth_tol=1e-5, max_passes=3, handle=h)
    del A, A0
if which in ("all", "lowrank"):
    m = 32768
    A = torch.randn(m, m, device="cuda").t()
    for _ in range(2):
        rg.lowrank_approx(A, 512, oversample=16, power_iters=1, seed=7, handle=h)
torch.cuda.synchronize()
