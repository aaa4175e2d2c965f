"""Scratch: RGSQR accuracy for ill-conditioned inputs (two-pass CholQR panels)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import oracle, synth
import paper_conf_hpdc_zhangbw20_b200 as rg

def dev(A):
    return torch.from_numpy(np.ascontiguousarray(np.asarray(A, dtype=np.float32).T)).cuda().t()

for (m, n, kappa) in [(8192, 32, 100.0), (8192, 64, 100.0), (8192, 256, 100.0), (65536, 32, 100.0), (8192, 32, 1e4)]:
    A = synth.svd_matrix(m, n, "geometric", kappa, seed=31).astype(np.float32)
    for panel in ("auto", "mgs"):
        Q, R = rg.rgsqr_factor(dev(A), opts=rg.make_opts(panel=panel))
        torch.cuda.synchronize()
        Q = Q.cpu().numpy().astype(np.float64); R = R.cpu().numpy().astype(np.float64)
        A64 = A.astype(np.float64)
        Qo, Ro, _ = oracle.householder(A64)
        print(f"m={m} n={n} k={kappa:g} {panel}: be={oracle.backward_error(A64,Q,R):.2e} orth={oracle.orthogonality(Q):.2e} dR={np.linalg.norm(R-Ro)/np.linalg.norm(Ro):.2e}", flush=True)
