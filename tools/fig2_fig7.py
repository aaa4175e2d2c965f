"""B200 analogues of the paper's Figure 7 (tensor cores in panel / update, section 4.1.2,
P:L392-395) and Figure 2 (cutoff B of the recursion with eq 7).

Figure 7: rgsqr_factor timed (graph replay, CUDA events) in three configurations --
  1. 16-bit tensor cores in panel AND update: the default (leaf Gram / apply on split-fp16
     mma.sync for well-conditioned panels, K1 / K2 on tcgen05),
  2. tensor cores in the update only: RGSQR_LEAF_FP64_GRAM=1 (panel Gram on fp64 DMMA, FFMA apply),
  3. no 16-bit tensor cores: RGSQR_NO_TC=1 (K1 / K2 as fp32 SIMT GEMMs, the Table 3 SGEMM rows).
Figure 2 / eq 7: the base case of the recursion B in {8, 16, 32} (panels of nb columns,
RGSQR_NO_LEAF=1) and 64 (the leaf kernel, default); measured total vs the eq 7 prediction built
from that run's own per-op rates (RGSQR_PROF_OPS=1: K1 / K2 per width, the panel rate).

    python tools/fig2_fig7.py [m n] > profiles/<round>_fig2_fig7.md
Each configuration runs in its own process (the switches are read once per process).
"""
import collections
import json
import os
import re
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def child(m, n, nb, prof):
    import numpy as np
    import torch
    import paper_conf_hpdc_zhangbw20_b200 as rg
    h = rg.Handle(0)
    gen = torch.Generator(device="cuda").manual_seed(20200625)
    A = torch.randn(n, m, generator=gen, device="cuda").t()
    Q = torch.empty(n, m, device="cuda").t()
    R = torch.empty(n, n, device="cuda").t()
    o = rg.make_opts(sync=False, nb=nb)
    for _ in range(3):
        rg.rgsqr_factor(A, Q=Q, R=R, handle=h, opts=o, check=False)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    reps = 5
    e0.record()
    for _ in range(reps):
        rg.rgsqr_factor(A, Q=Q, R=R, handle=h, opts=o, check=False)
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / reps
    # accuracy (Hutchinson probes on the device, fp64, check only)
    g = torch.Generator(device="cuda").manual_seed(99)
    G = torch.randn(n, 8, generator=g, device="cuda", dtype=torch.float64)
    A64, Q64, R64 = A.double(), Q.double(), R.double()
    be = (torch.linalg.norm(A64 @ G - Q64 @ (R64 @ G)) / torch.linalg.norm(A64 @ G)).item()
    orth = (torch.linalg.norm(G - Q64.t() @ (Q64 @ G)) / 8 ** 0.5).item()
    del A64, Q64, R64
    print("RESULT " + json.dumps({"ms": ms, "be": be, "orth": orth}))
    if prof:
        h.profile(True)
        h.profile_reset()
        rg.rgsqr_factor(A, Q=Q, R=R, handle=h, opts=o, check=False)
        torch.cuda.synchronize()


def run(m, n, nb, env_extra, prof=False):
    env = dict(os.environ, _F27_CHILD="1", **env_extra)
    if prof:
        env["RGSQR_PROF_OPS"] = "1"
    p = subprocess.run([sys.executable, __file__, str(m), str(n), str(nb), "1" if prof else "0"], env=env,
                       capture_output=True, text=True)
    if p.returncode != 0:
        raise RuntimeError(p.stdout[-2000:] + p.stderr[-2000:])
    res = json.loads(re.search(r"RESULT (\{.*\})", p.stdout).group(1))
    ops = collections.defaultdict(lambda: [0, 0.0])
    names = {0: "K2", 1: "K1", 2: "panel", 3: "scale", 5: "other"}
    for line in p.stderr.splitlines():
        mm = re.match(r"\[rgsqr op\] cls (\d+) w (\d+) us ([\d.]+)", line)
        if mm:
            c = names.get(int(mm.group(1)), mm.group(1))
            w = int(mm.group(2)) if c in ("K1", "K2") else 0
            ops[(c, w)][0] += 1
            ops[(c, w)][1] += float(mm.group(3))
    return res, ops


def eq7(m, n, B, ops):
    """S_RGSQRF(m, n) = 2 / (1/S(m, n/2) + 1/S_TC-GEMM(m, n/2)), S(m, B) = panel rate (eq 7)."""
    s_gemm = {}
    for (c, w), (cnt, us) in ops.items():
        if c == "K1" and ("K2", w) in ops:
            c2, u2 = ops[("K2", w)]
            s_gemm[w] = 2.0 * m * w * w * (cnt + c2) / ((us + u2) * 1e-6) / 1e12
    pc, pu = ops[("panel", 0)]
    s_panel = 2.0 * m * B * B * pc / (pu * 1e-6) / 1e12 if pu else float("nan")

    def S(nn):
        if nn <= B:
            return s_panel
        g = s_gemm.get(nn // 2)
        if g is None:
            return S(nn // 2)
        return 2.0 / (1.0 / S(nn // 2) + 1.0 / g)

    return S(n), s_panel, s_gemm


def main():
    if os.environ.get("_F27_CHILD"):
        child(int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3]), sys.argv[4] == "1")
        return
    m = int(sys.argv[1]) if len(sys.argv) > 1 else 65536
    n = int(sys.argv[2]) if len(sys.argv) > 2 else 4096
    fl = 2.0 * m * n * n - 2.0 * n ** 3 / 3.0
    print(f"# Figure 7 / Figure 2 analogues on B200: RGSQR of {m} x {n} N(0,1) fp32\n")
    print("Times: CUDA events around 5 graph-replayed `rgsqr_factor` calls after 3 warm-ups (one process per")
    print("configuration).  TFLOP/s with the 2mn^2 - 2n^3/3 convention.  be / orth: 8 fp64 Hutchinson probes.\n")
    print("## Figure 7: tensor cores in the panel and in the update (P:L392-395)\n")
    print("| configuration | ms | TFLOP/s | backward error | orthogonality (F) |")
    print("|---|---|---|---|---|")
    for label, env in (("16-bit TC in panel + update (default)", {}),
                       ("TC in update only (RGSQR_LEAF_FP64_GRAM=1)", {"RGSQR_LEAF_FP64_GRAM": "1"}),
                       ("no 16-bit TC (RGSQR_NO_TC=1: fp32 SIMT K1/K2)", {"RGSQR_NO_TC": "1"})):
        r, _ = run(m, n, 32, env)
        print(f"| {label} | {r['ms']:.2f} | {fl / (r['ms'] * 1e-3) / 1e12:.1f} | {r['be']:.2e} | {r['orth']:.2e} |")
    print("\n## Figure 2 / eq 7: the cutoff B of the recursion (P:L205-219)\n")
    print("eq 7 is evaluated with the same run's per-op rates (`RGSQR_PROF_OPS=1`: eager launches, so the")
    print("per-op rates include launch latency and eq 7 is a lower bound on the graph-replayed rate).\n")
    print("| B (base case) | measured ms | measured TFLOP/s (2mn^2) | eq 7 TFLOP/s (2mn^2) | panel TFLOP/s (2mB^2) | be | orth |")
    print("|---|---|---|---|---|---|---|")
    best = None
    for B, nb, env in ((8, 8, {"RGSQR_NO_LEAF": "1"}), (16, 16, {"RGSQR_NO_LEAF": "1"}),
                       (32, 32, {"RGSQR_NO_LEAF": "1"}), (64, 32, {})):
        r, ops = run(m, n, nb, env, prof=True)
        pred, s_panel, _ = eq7(m, n, B, ops)
        meas = 2.0 * m * n * n / (r["ms"] * 1e-3) / 1e12
        print(f"| {B}{' (leaf kernel, default)' if B == 64 else ''} | {r['ms']:.2f} | {meas:.1f} | {pred:.1f} | "
              f"{s_panel:.2f} | {r['be']:.2e} | {r['orth']:.2e} |")
        if best is None or r["ms"] < best[1]:
            best = (B, r["ms"])
    print(f"\nFastest measured base case: B = {best[0]} ({best[1]:.2f} ms).")


if __name__ == "__main__":
    main()
