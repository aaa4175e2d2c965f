"""Tall CholQR pass (csrc/tall.cu) on the GPU: orthogonalize with RGSQR_TALL forced on / off,
accuracy against the fp64 oracle on small shapes and the config-4 timing.

    python tools/tall_check.py [--big]
"""
import os
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import oracle  # noqa: E402
import synth  # noqa: E402
import paper_conf_hpdc_zhangbw20_b200 as rg  # noqa: E402


def dev(A):
    return torch.from_numpy(np.ascontiguousarray(A.T)).cuda().t()


def run(A, tall, passes=3, tol=1e-5):
    os.environ["RGSQR_TALL"] = "1" if tall else "0"
    Ad = dev(A)
    n = A.shape[1]
    R = torch.zeros(n, n, device="cuda").t()
    Q, R, p, est = rg.orthogonalize(Ad, R, orth_tol=tol, max_passes=passes)
    torch.cuda.synchronize()
    return Q.cpu().numpy().astype(np.float64), R.cpu().numpy().astype(np.float64), p, est


def small():
    for (m, n, kind, kap) in [(20000, 256, "gauss", 1), (9001, 200, "geometric", 1e2), (4099, 64, "gauss", 1),
                              (30000, 256, "geometric", 1e4), (777, 130, "gauss", 1)]:
        A = (synth.gaussian(m, n, seed=3) if kind == "gauss" else synth.svd_matrix(m, n, kind, kap, seed=3)).astype(
            np.float32)
        for tall in (True, False):
            Q, R, p, est = run(A, tall)
            A64 = A.astype(np.float64)
            be = oracle.backward_error(A64, Q, R)
            orth = oracle.orthogonality(Q)
            Qo, Ro, _ = oracle.householder(A64)
            dq = np.linalg.norm(Q - Qo) / np.linalg.norm(Qo)
            dr = np.linalg.norm(R - Ro) / np.linalg.norm(Ro)
            print(f"{m}x{n} {kind} k={kap:g} tall={tall}: passes {p} est {est:.2e} orth {orth:.2e} be {be:.2e} "
                  f"dq {dq:.2e} dr {dr:.2e}", flush=True)


def big():
    m, n = 2097152, 256
    A = torch.randn(n, m, device="cuda", generator=torch.Generator("cuda").manual_seed(5)).t()
    A0 = A.clone()
    for tall in (True, False):
        os.environ["RGSQR_TALL"] = "1" if tall else "0"
        h = rg.Handle() if hasattr(rg, "Handle") else None
        ts = []
        for it in range(4):
            A.copy_(A0)
            torch.cuda.synchronize()
            t = time.perf_counter()
            _, _, p, est = rg.orthogonalize(A, None, orth_tol=1e-5, max_passes=3)
            torch.cuda.synchronize()
            ts.append(time.perf_counter() - t)
        print(f"config 4 tall={tall}: {min(ts) * 1e3:.2f} ms (wall, incl. syncs), passes {p}, est {est:.2e}", flush=True)


if __name__ == "__main__":
    small()
    if "--big" in sys.argv:
        big()
