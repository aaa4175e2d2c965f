"""Compare the 64-column CholQR2 leaf level against the 32-column panels + K1/K2 (development tool)."""
import os
import subprocess
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np

if len(sys.argv) > 1 and sys.argv[1] == "child":
    import torch
    import oracle
    import synth
    import paper_conf_hpdc_zhangbw20_b200 as rg
    for (m, n, kappa) in [(8192, 128, 1e4), (65536, 256, 1e2), (4096, 128, 1e6), (3000, 96, 1e5)]:
        A = synth.svd_matrix(m, n, "geometric", kappa, seed=5).astype(np.float32)
        Ad = torch.from_numpy(np.ascontiguousarray(A.T)).cuda().t()
        for reo in (0, 1):
            Q, R = rg.rgsqr_factor(Ad, opts=rg.make_opts(reortho=reo))
            torch.cuda.synchronize()
            Qn = Q.cpu().numpy().astype(np.float64)
            Rn = R.cpu().numpy().astype(np.float64)
            be = oracle.backward_error(A.astype(np.float64), Qn, Rn)
            orth = oracle.orthogonality(Qn)
            b = synth.rhs(A.astype(np.float64), seed=5, consistent=True).astype(np.float32)
            _, it, rel, st = rg.ls_solve_refined(Ad, torch.from_numpy(b).cuda(), opts=rg.make_opts(reortho=reo), maxit=400)
            print(f"  m={m} n={n} kappa={kappa:.0e} reortho={reo}: be={be:.2e} orth={orth:.2e} cgls_iters={it} st={st}")
else:
    for env in ({}, {"RGSQR_NO_PAIR": "1"}):
        print("env", env, flush=True)
        e = dict(os.environ)
        e.update(env)
        subprocess.run([sys.executable, __file__, "child"], env=e, check=False)
