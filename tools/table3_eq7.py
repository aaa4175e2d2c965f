"""B200 analogue of the paper's Table 3 and performance model eq 7.

PAPER.md P:L161-173 (Table 3: TC-GEMM TFLOPS for k = 128 ... 16384 at m = 32768, shapes
A^T B (k x m times m x k) and A B (m x k times k x k)) and P:L213-219 (eq 7:
S(m, n) = 2 / (1 / S(m, n/2) + 1 / S_TC-GEMM(m, n/2)) for n > B, S = S_panel at n = B).

On B200 the two GEMM shapes are exactly this library's K1 (R12 = Q1^T A2, h = w = k) and K2
(A2 -= Q1 R12) at recursion width k, so one RGSQR call on the paper's Figure 2 matrix
(32768 x 16384) with per-op CUDA events (RGSQR_PROF_OPS=1) measures every row of the table:
K1 and K2 rates per width, the leaf (panel) rate, and the measured total to compare with eq 7.

    python tools/table3_eq7.py [m n] > profiles/<round>_table3_eq7.md
"""
import collections
import os
import re
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def child(m, n):
    import torch
    import paper_conf_hpdc_zhangbw20_b200 as rg
    h = rg.Handle(0)
    A = torch.randn(n, m, device="cuda").t()
    Q = torch.empty(n, m, device="cuda").t()
    R = torch.empty(n, n, device="cuda").t()
    o = rg.make_opts(sync=False)
    for _ in range(2):
        rg.rgsqr_factor(A, Q=Q, R=R, handle=h, opts=o, check=False)
    torch.cuda.synchronize()
    # timed call without per-op events (graph replay)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    rg.rgsqr_factor(A, Q=Q, R=R, handle=h, opts=o, check=False)
    e1.record()
    torch.cuda.synchronize()
    print(f"TOTAL_MS {e0.elapsed_time(e1):.4f}")
    h.profile(True)
    h.profile_reset()
    rg.rgsqr_factor(A, Q=Q, R=R, handle=h, opts=o, check=False)
    torch.cuda.synchronize()


def main():
    m = int(sys.argv[1]) if len(sys.argv) > 1 else 32768
    n = int(sys.argv[2]) if len(sys.argv) > 2 else 16384
    if os.environ.get("_T3_CHILD"):
        child(m, n)
        return
    env = dict(os.environ, RGSQR_PROF_OPS="1", _T3_CHILD="1")
    p = subprocess.run([sys.executable, __file__, str(m), str(n)], env=env, capture_output=True, text=True)
    if p.returncode != 0:
        print(p.stdout, p.stderr[-3000:])
        sys.exit(p.returncode)
    total_ms = float(re.search(r"TOTAL_MS ([\d.]+)", p.stdout).group(1))
    names = {0: "K2", 1: "K1", 2: "panel", 3: "scale", 5: "other"}
    agg = collections.defaultdict(lambda: [0, 0.0])   # (class, w) -> [count, us]
    for line in p.stderr.splitlines():
        mm = re.match(r"\[rgsqr op\] cls (\d+) w (\d+) us ([\d.]+)", line)
        if mm:
            k = (names.get(int(mm.group(1)), mm.group(1)), int(mm.group(2)))
            agg[k][0] += 1
            agg[k][1] += float(mm.group(3))
    widths = sorted({w for (c, w) in agg if c in ("K1", "K2")}, reverse=True)
    print(f"# Table 3 / eq 7 on B200: RGSQR of {m} x {n} (fp16 tensor-core K1/K2, 64-column leaf)\n")
    print("Per-op CUDA events (`RGSQR_PROF_OPS=1`, no graph: each op includes its launch latency, which")
    print("dominates the narrow levels).  K1 = R12 = Q1^T A2 (Table 3 columns 2-3 shape, k x m times m x k),")
    print("K2 = A2 -= Q1 R12 (columns 4-5 shape, m x k times k x k), flops 2 m k^2 each.\n")
    print("| k (= w) | K1 calls | K1 TFLOP/s | K2 calls | K2 TFLOP/s | K1+K2 TFLOP/s | paper V100 TC-GEMM (cols 2 / 4) |")
    print("|---|---|---|---|---|---|---|")
    paper = {128: (8.45, 4.44), 256: (30.17, 11.39), 512: (56.48, 58.05), 1024: (72.39, 77.58),
             2048: (93.53, 87.29), 4096: (97.82, 92.72), 8192: (92.75, 92.20), 16384: (82.32, 83.40)}
    s_gemm = {}
    for w in widths:
        c1, u1 = agg[("K1", w)]
        c2, u2 = agg[("K2", w)]
        f = 2.0 * m * w * w
        t1 = f * c1 / (u1 * 1e-6) / 1e12 if u1 else float("nan")
        t2 = f * c2 / (u2 * 1e-6) / 1e12 if u2 else float("nan")
        tb = f * (c1 + c2) / ((u1 + u2) * 1e-6) / 1e12 if (u1 + u2) else float("nan")
        s_gemm[w] = tb
        pv = paper.get(w)
        print(f"| {w} | {c1} | {t1:.1f} | {c2} | {t2:.1f} | {tb:.1f} | {pv[0]:.2f} / {pv[1]:.2f} |" if pv else
              f"| {w} | {c1} | {t1:.1f} | {c2} | {t2:.1f} | {tb:.1f} | - |")
    pc, pu = agg[("panel", 0)]
    B = 64
    panel_flops = 2.0 * m * B * B * pc   # eq 5 base case T = 2 m n^2 per panel
    s_panel = panel_flops / (pu * 1e-6) / 1e12
    print(f"\nLeaf (64-column panel, Table 3 column 6 analogue): {pc} calls, {pu / pc:.1f} us each, "
          f"{s_panel:.2f} TFLOP/s (2 m B^2 per leaf; paper V100 SGEQRF at k = 128: 0.10)\n")

    # eq 7 with the measured rates; widths are the recursion's h = n / 2^i (n power of two)
    def S(nn):
        if nn <= B:
            return s_panel
        g = s_gemm.get(nn // 2)
        if g is None or g != g:
            return S(nn // 2)
        return 2.0 / (1.0 / S(nn // 2) + 1.0 / g)

    pred = S(n)
    flops_alg = 2.0 * m * n * n - 2.0 * n ** 3 / 3.0
    flops_rec = 2.0 * m * n * n
    meas = flops_rec / (total_ms * 1e-3) / 1e12
    print(f"eq 7 prediction S_RGSQRF({m}, {n}) from the measured K1/K2/leaf rates: {pred:.1f} TFLOP/s "
          f"(2 m n^2 convention of eq 5) -> {flops_rec / pred / 1e9:.2f} ms")
    print(f"measured (graph replay, one call): {total_ms:.3f} ms = {meas:.1f} TFLOP/s (2 m n^2), "
          f"{flops_alg / (total_ms * 1e-3) / 1e12:.1f} TFLOP/s (2mn^2 - 2n^3/3)")
    print("\nThe per-op events include launch latency (no graph), so eq 7 built from them is a lower bound on")
    print("the graph-replayed rate; the paper's Figure 2 analogue is the sweep over B (here fixed at 64).")


if __name__ == "__main__":
    main()
