"""Scratch diagnostic: virtual-rank row-sharded factorization vs single GPU (prints only)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_hpdc_zhangbw20_b200 as rg
import synth, oracle

def dev(A):
    return torch.from_numpy(np.ascontiguousarray(np.asarray(A, dtype=np.float32).T)).cuda().t()

def run(P, m, n, **kw):
    A = synth.gaussian(m, n, seed=5).astype(np.float32)
    g = rg.VGroup(P)
    ss = [torch.cuda.Stream() for _ in range(P)]
    hs = [rg.Handle(0, stream=s.cuda_stream) for s in ss]
    for r, h in enumerate(hs):
        h.set_vcomm(g, r)
    c = np.linspace(0, m, P + 1).astype(int)
    bl = [dev(A[c[r]:c[r+1]]) for r in range(P)]
    Qs = [torch.zeros(n, c[r+1]-c[r], device="cuda").t() for r in range(P)]
    Rs = [torch.zeros(n, n, device="cuda").t() for r in range(P)]
    o = rg.make_opts(**kw)
    torch.cuda.synchronize()
    rg.run_ranks([lambda r=r: rg.rgsqr_factor(bl[r], Q=Qs[r], R=Rs[r], handle=hs[r], opts=o) for r in range(P)])
    torch.cuda.synchronize()
    Q = np.vstack([q.cpu().numpy() for q in Qs]).astype(np.float64)
    R = Rs[0].cpu().numpy().astype(np.float64)
    _, Ro, _ = oracle.householder(A.astype(np.float64))
    print(f"P={P} m={m} n={n} {kw}: be {oracle.backward_error(A.astype(np.float64), Q, R):.3e} "
          f"orth {oracle.orthogonality(Q):.3e} dr {np.linalg.norm(R-Ro)/np.linalg.norm(Ro):.3e} "
          f"Rdiag {np.diag(R)[:4]} oracle {np.diag(Ro)[:4]} same-R {np.array_equal(Rs[0].cpu().numpy(), Rs[-1].cpu().numpy())}")
    for h in hs: h.close()
    g.close()

for P in (1, 2):
    for n in (32, 64, 160):
        for panel in ("auto", "mgs"):
            try:
                run(P, 6000, n, panel=panel)
            except Exception as e:
                print("ERR", P, n, panel, e)
