import os, sys, time
sys.path.insert(0, "/root/repo")
import numpy as np, torch
import synth, oracle
import paper_conf_hpdc_zhangbw20_b200 as rg
m, n = 131072, 1024
A = synth.svd_matrix(m, n, "geometric", 1e4, seed=synth.SEED_BASE + 2)
b = synth.rhs(A, seed=synth.SEED_BASE + 2, consistent=False)
A32 = A.astype(np.float32); b32 = b.astype(np.float32)
Ad = torch.from_numpy(np.ascontiguousarray(A32.T)).cuda().t()
bd = torch.from_numpy(b32).cuda()
# fp32-problem solution via normal equations in fp64 (QR of the fp32 A)
Q, R = np.linalg.qr(A32.astype(np.float64))
xs = np.linalg.solve(R, Q.T @ b32.astype(np.float64))
h = rg.Handle(0)
for reo, split in ((1, 0), (0, 1), (1, 1), (0, 0)):
    for solver in ("cgls",):
        o = rg.make_opts(reortho=reo, solver=solver, split=bool(split))
        x = torch.zeros(n, dtype=torch.float64, device="cuda")
        for _ in range(2):
            rg.ls_solve_refined(Ad, bd, x, handle=h, opts=o)
        torch.cuda.synchronize()
        ts = []
        for _ in range(5):
            torch.cuda.synchronize(); t0 = time.perf_counter()
            _, it, rel, st = rg.ls_solve_refined(Ad, bd, x, handle=h, opts=o)
            torch.cuda.synchronize(); ts.append(time.perf_counter() - t0)
        xv = x.cpu().numpy()
        print(f"reortho={reo} split={split} {solver}: {min(ts)*1e3:.2f} ms iters {it} relres {rel:.2e} fe {np.linalg.norm(xv-xs)/np.linalg.norm(xs):.2e} st {st}", flush=True)
