"""Summarise an ncu launch list (--metrics gpu__time_duration.sum --csv) of `bench.py` for one
rgsqr_factor call: per-kernel-class time, share of the step, top launches (development tool)."""
import collections
import csv
import sys


def load(path):
    rows = list(csv.reader(open(path)))
    hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
    h = rows[hi]
    ik, iv, iid = h.index("Kernel Name"), h.index("Metric Value"), h.index("ID")
    return [(int(r[iid]), r[ik], float(r[iv].replace(",", ""))) for r in rows[hi + 1:] if len(r) > iv]


def short(name):
    n = name.split("(")[0].replace("void ", "")
    return n.replace("rg::", "")


def klass(n):
    if "leaf_kernel" in n:
        return "leaf (64-col CholQR2 panel + folded K1/K2 of w=64)"
    if "gemm_tc_kernel" in n:
        return "gemm (K1 proj / K2 update, tcgen05)"
    if "proj_reduce" in n or "proj_finish" in n:
        return "K1 split-K reduce"
    if n.startswith("cq_") or "panel" in n:
        return "panel (CholQR2 / MGS guard)"
    if "colnorm" in n or "scale" in n:
        return "column scaling"
    return "other"


def main(path, call_index):
    ks = load(path)
    starts = [i for i, (_, n, _) in enumerate(ks) if "colnorm_partial" in n]
    a = starts[call_index]
    b = starts[call_index + 1] if call_index + 1 < len(starts) else len(ks)
    step = [k for k in ks[a:b] if "rg::" in k[1]]   # librgsqr kernels only
    tot = sum(t for _, _, t in step)
    by = collections.defaultdict(lambda: [0, 0.0])
    for _, n, t in step:
        c = klass(short(n))
        by[c][0] += 1
        by[c][1] += t
    print(f"# ncu launch list, one rgsqr_factor call (launches {a}..{b - 1} of {path.split('/')[-1]})")
    print(f"# {len(step)} launches, sum of kernel durations {tot / 1e6:.3f} ms (serialised, cold-cache under ncu)\n")
    print("| class | launches | ms | share |")
    print("|---|---|---|---|")
    for c, (cnt, t) in sorted(by.items(), key=lambda x: -x[1][1]):
        print(f"| {c} | {cnt} | {t / 1e6:.3f} | {t / tot:.3f} |")
    print("\n| top launches | us |")
    print("|---|---|")
    for _, n, t in sorted(step, key=lambda x: -x[2])[:12]:
        print(f"| {short(n)} | {t / 1e3:.1f} |")
    return step


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 3)
