"""Scratch diagnostics: rgsqr_factor vs the oracle over a ladder of shapes (prints, no asserts)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import oracle, synth
import paper_conf_hpdc_zhangbw20_b200 as rg

def dev(A):
    return torch.from_numpy(np.ascontiguousarray(np.asarray(A, dtype=np.float32).T)).cuda().t()

for (m, n) in [(64, 8), (256, 32), (1000, 32), (5000, 32), (128, 64), (1024, 64), (1024, 128), (4096, 256), (3000, 200), (8192, 512)]:
    A = synth.gaussian(m, n, seed=m + n).astype(np.float32)
    try:
        Q, R = rg.rgsqr_factor(dev(A))
        torch.cuda.synchronize()
        Q = Q.cpu().numpy().astype(np.float64); R = R.cpu().numpy().astype(np.float64)
        A64 = A.astype(np.float64)
        Qo, Ro, _ = oracle.householder(A64)
        be = oracle.backward_error(A64, Q, R); orth = oracle.orthogonality(Q)
        dr = np.linalg.norm(R - Ro) / np.linalg.norm(Ro)
        # where is R wrong?
        bad = np.argwhere(np.abs(R - Ro) > 1e-2 * np.abs(Ro).max())
        print(f"m={m} n={n} be={be:.3e} orth={orth:.3e} dR={dr:.3e} nbad={len(bad)} first={bad[:4].tolist()}", flush=True)
    except Exception as e:
        print(f"m={m} n={n} EXC {e}", flush=True)
