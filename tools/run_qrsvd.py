"""Time / check lowrank_qrsvd at the Table 4 size (524288 x 1024, arithmetic, kappa 1e6) (development tool)."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_hpdc_zhangbw20_b200 as rg
import synth
m = int(os.environ.get("RG_M", 524288)); n = int(os.environ.get("RG_N", 1024))
At, s = synth.svd_matrix_device(m, n, "arithmetic", 1e6, seed=4)
A = At.t()
h = rg.Handle(0)
for r in (16, 64, 128, 256, 512):
    torch.cuda.synchronize(); t0 = time.perf_counter()
    U, S, V = rg.lowrank_qrsvd(A, r, handle=h)
    torch.cuda.synchronize(); dt = time.perf_counter() - t0
    Ad = A.double()
    err = (torch.linalg.norm(Ad - (U.double() * S.double()) @ V.double().t()) / torch.linalg.norm(Ad)).item()
    opt = float(np.sqrt(np.sum(s[r:] ** 2) / np.sum(s ** 2)))
    print(f"r={r}: {dt*1e3:.1f} ms err {err:.4e} opt {opt:.4e} S0 {S[0].item():.6f} S[-1] {S[-1].item():.6f} vs {s[r-1]:.6f}")
