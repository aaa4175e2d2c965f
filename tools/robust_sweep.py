"""Robustness sweep (development tool): tall orthogonalize over n / m / kappa / alignment and the
default LS preconditioner over kappa and right-hand sides, against the fp64 oracle."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import oracle, synth
import paper_conf_hpdc_zhangbw20_b200 as rg

def dev(A):
    return torch.from_numpy(np.ascontiguousarray(np.asarray(A, dtype=np.float32).T)).cuda().t()

bad = 0
os.environ["RGSQR_TALL"] = "1"
for (m, n, kind, kap) in [(70000, 16, "gauss", 1), (70001, 100, "geometric", 1e2), (100003, 255, "gauss", 1),
                          (131072, 256, "geometric", 1e3), (40000, 256, "cluster", 1e2), (65536, 200, "arithmetic", 10),
                          (90000, 64, "geometric", 1e5)]:
    A = (synth.gaussian(m, n, seed=m + n) if kind == "gauss" else synth.svd_matrix(m, n, kind, kap, seed=m + n)).astype(np.float32)
    Ad = dev(A)
    R = torch.zeros(n, n, device="cuda").t()
    try:
        Q, R, p, est = rg.orthogonalize(Ad, R, orth_tol=1e-5, max_passes=3)
    except Exception as e:
        print("FAIL", m, n, kind, kap, e); bad += 1; continue
    Qn = Q.cpu().numpy().astype(np.float64); Rn = R.cpu().numpy().astype(np.float64)
    orth = oracle.orthogonality(Qn); be = oracle.backward_error(A.astype(np.float64), Qn, Rn)
    ok = orth <= 1e-5 and be <= 5e-3 and abs(est - orth) <= 0.5 * orth + 1e-7
    bad += not ok
    print(f"{'ok  ' if ok else 'FAIL'} orth {m}x{n} {kind} k={kap:g}: passes {p} orth {orth:.2e} est {est:.2e} be {be:.2e}", flush=True)
os.environ["RGSQR_TALL"] = "auto"
for (m, n, kind, kap, cons) in [(20000, 256, "geometric", 1e2, False), (20000, 256, "geometric", 1e4, True),
                                (30000, 512, "arithmetic", 1e4, False), (12000, 100, "cluster", 1e3, False),
                                (50000, 64, "geometric", 1e6, True)]:
    A = synth.svd_matrix(m, n, kind, kap, seed=m).astype(np.float32)
    b = synth.rhs(A.astype(np.float64), seed=m, consistent=cons).astype(np.float32)
    x = torch.zeros(n, dtype=torch.float64, device="cuda")
    _, it, rel, st = rg.ls_solve_refined(dev(A), torch.from_numpy(b).cuda(), x, maxit=200)
    xs, _ = oracle.ls_qr(A.astype(np.float64), b.astype(np.float64))
    fe = np.linalg.norm(x.cpu().numpy() - xs) / np.linalg.norm(xs)
    ok = st == 0 and (fe <= 1e-5 or kap > 1e4)
    bad += not ok
    print(f"{'ok  ' if ok else 'FAIL'} ls {m}x{n} {kind} k={kap:g} consistent={cons}: iters {it} status {st} fe {fe:.2e}", flush=True)
print("failures", bad)
