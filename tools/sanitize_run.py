"""Small calls through every kernel family, for compute-sanitizer (development tool)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_hpdc_zhangbw20_b200 as rg
import synth
which = sys.argv[1] if len(sys.argv) > 1 else "all"
def dev(A):
    return torch.from_numpy(np.ascontiguousarray(np.asarray(A, dtype=np.float32).T)).cuda().t()
h = rg.Handle(0)
o = rg.make_opts()
if which in ("all", "factor"):
    A = synth.gaussian(4096, 256, seed=1).astype(np.float32)      # leaf + tcgen05 K1/K2 (w = 128)
    rg.rgsqr_factor(dev(A), handle=h, opts=rg.make_opts(sync=True))
    A = synth.gaussian(20000, 96, seed=2).astype(np.float32)      # fused CholQR panels
    rg.rgsqr_factor(dev(A), handle=h)
    rg.rgsqr_factor(dev(A), handle=h, opts=rg.make_opts(panel="mgs"))
if which in ("all", "apps"):
    A = synth.svd_matrix(8192, 128, "geometric", 1e3, seed=3).astype(np.float32)
    rg.orthogonalize(dev(A), None, orth_tol=1e-5, max_passes=3, handle=h)
    b = synth.rhs(A.astype(np.float64), seed=3, consistent=False).astype(np.float32)
    rg.ls_solve_refined(dev(A), torch.from_numpy(b).cuda(), handle=h)
    rg.ls_solve_refined(dev(A), torch.from_numpy(b).cuda(), handle=h, opts=rg.make_opts(solver="lsqr"))
    L, _ = synth.lowrank_matrix(2048, 512, 128, "geometric", 1e4, seed=4)
    rg.lowrank_approx(dev(L), 64, oversample=16, power_iters=1, seed=5, handle=h)
if which in ("all", "tall"):
    # tall CholQR passes (tall.cu): TMA-fed Gram (aligned ld), register-fed Gram (ld % 4 != 0),
    # reduce / symmetrise, Cholesky (general + first-order), apply; kappa fallback
    os.environ["RGSQR_TALL"] = "1"
    A = synth.gaussian(20000, 256, seed=6).astype(np.float32)
    rg.orthogonalize(dev(A), None, orth_tol=0.0, max_passes=2, handle=h)
    A = synth.svd_matrix(9001, 200, "geometric", 1e2, seed=7).astype(np.float32)
    rg.orthogonalize(dev(A), None, orth_tol=1e-5, max_passes=3, handle=h)
    A = synth.svd_matrix(12000, 96, "geometric", 1e4, seed=8).astype(np.float32)
    rg.orthogonalize(dev(A), None, orth_tol=1e-5, max_passes=3, handle=h)
    os.environ["RGSQR_TALL"] = "0"
if which in ("all", "pair"):
    # cluster-pair K2 with TMA multicast (h = 768 at the top level) and 192-wide general GEMMs
    A = synth.gaussian(4096, 1536, seed=9).astype(np.float32)
    rg.rgsqr_factor(dev(A), handle=h)
    L, _ = synth.lowrank_matrix(2048, 1024, 256, "geometric", 1e4, seed=10)
    rg.lowrank_approx(dev(L), 256, oversample=16, power_iters=1, seed=5, handle=h)
torch.cuda.synchronize()
print("ok", which)
