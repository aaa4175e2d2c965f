"""Profile classes of one ls_solve_refined call at BASELINE config 3 (development tool)."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import synth
import paper_conf_hpdc_zhangbw20_b200 as rg
m, n = 131072, 1024
A = synth.svd_matrix(m, n, "geometric", 1e4, seed=synth.SEED_BASE + 2)
b = synth.rhs(A, seed=synth.SEED_BASE + 2, consistent=False)
Ad = torch.from_numpy(np.ascontiguousarray(A.T.astype(np.float32))).cuda().t()
bd = torch.from_numpy(b.astype(np.float32)).cuda()
x = torch.zeros(n, dtype=torch.float64, device="cuda")
h = rg.Handle(0)
for _ in range(2):
    rg.ls_solve_refined(Ad, bd, x, handle=h)
torch.cuda.synchronize()
h.profile(True); h.profile_reset()
t0 = time.perf_counter()
_, it, rel, st = rg.ls_solve_refined(Ad, bd, x, handle=h)
torch.cuda.synchronize()
print("wall ms", (time.perf_counter() - t0) * 1e3, "iters", it, "relres", rel)
for c in ("update", "proj", "panel", "scale", "cgls", "other"):
    try:
        print(c, h.profile_get(c))
    except Exception as e:
        print(c, e)
