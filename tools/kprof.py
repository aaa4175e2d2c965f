"""Kernel-level time breakdown (CUPTI via torch.profiler) of one call (development tool).

    python tools/kprof.py factor|orth|lowrank|ls

Shapes: BASELINE configs 2 / 4 / 5 / 3.  Prints the kernels sorted by total device time.
"""
import os
import sys
import collections

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from torch.profiler import profile, ProfilerActivity

import paper_conf_hpdc_zhangbw20_b200 as rg

call = sys.argv[1] if len(sys.argv) > 1 else "factor"
h = rg.Handle(0)
if call == "factor":
    m, n = 65536, 4096
elif call == "orth":
    m, n = 2097152, 256
elif call == "lowrank":
    m = n = 32768
else:
    m, n = 131072, 1024
A = torch.randn(n, m, device="cuda").t()
A0 = A.clone() if call in ("orth",) else None
Q = torch.empty(n, m, device="cuda").t() if call == "factor" else None
R = torch.empty(n, n, device="cuda").t()
b = torch.randn(m, device="cuda")
x = torch.zeros(n, dtype=torch.float64, device="cuda")


def run():
    if call == "factor":
        rg.rgsqr_factor(A, Q=Q, R=R, handle=h, opts=rg.make_opts(sync=False), check=False)
    elif call == "orth":
        A.copy_(A0)
        rg.orthogonalize(A, R, orth_tol=1e-5, max_passes=3, handle=h)
    elif call == "lowrank":
        rg.lowrank_approx(A, 512, oversample=16, power_iters=1, seed=7, handle=h)
    else:
        rg.ls_solve_refined(A, b, x, handle=h)


for _ in range(3):
    run()
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
run()
e1.record()
torch.cuda.synchronize()
print(f"{call}: {e0.elapsed_time(e1):.3f} ms (events, no profiler)")
with profile(activities=[ProfilerActivity.CUDA]) as prof:
    run()
    torch.cuda.synchronize()
agg = collections.defaultdict(lambda: [0, 0.0])
for ev in prof.events():
    if ev.device_type == torch.autograd.DeviceType.CUDA:
        k = ev.name[:90]
        agg[k][0] += 1
        agg[k][1] += ev.device_time_total if hasattr(ev, "device_time_total") else ev.cuda_time_total
tot = sum(v[1] for v in agg.values())
print(f"kernel time sum {tot / 1e3:.3f} ms")
for k, (c, us) in sorted(agg.items(), key=lambda kv: -kv[1][1])[:25]:
    print(f"{us / 1e3:9.3f} ms {c:5d}x  {k}")
