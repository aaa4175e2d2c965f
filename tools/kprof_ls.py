"""CUPTI kernel breakdown of ls_solve_refined at BASELINE config 3 (kappa 1e4 geometric) (development tool)."""
import os, sys, collections, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from torch.profiler import profile, ProfilerActivity
import synth
import paper_conf_hpdc_zhangbw20_b200 as rg
m, n = 131072, 1024
A = synth.svd_matrix(m, n, "geometric", 1e4, seed=synth.SEED_BASE + 2)
b = synth.rhs(A, seed=synth.SEED_BASE + 2, consistent=False)
Ad = torch.from_numpy(np.ascontiguousarray(A.T.astype(np.float32))).cuda().t()
bd = torch.from_numpy(b.astype(np.float32)).cuda()
x = torch.zeros(n, dtype=torch.float64, device="cuda")
h = rg.Handle(0)
for _ in range(2):
    rg.ls_solve_refined(Ad, bd, x, handle=h)
torch.cuda.synchronize()
t0 = time.perf_counter(); _, it, _, _ = rg.ls_solve_refined(Ad, bd, x, handle=h); torch.cuda.synchronize()
print(f"ls: {(time.perf_counter() - t0) * 1e3:.2f} ms wall, {it} iterations")
with profile(activities=[ProfilerActivity.CUDA]) as prof:
    rg.ls_solve_refined(Ad, bd, x, handle=h)
    torch.cuda.synchronize()
agg = collections.defaultdict(lambda: [0, 0.0])
for ev in prof.events():
    if ev.device_type == torch.autograd.DeviceType.CUDA:
        agg[ev.name[:80]][0] += 1
        agg[ev.name[:80]][1] += ev.device_time_total
tot = sum(v[1] for v in agg.values())
print(f"kernel time sum {tot / 1e3:.3f} ms")
for k, (c, us) in sorted(agg.items(), key=lambda kv: -kv[1][1])[:16]:
    print(f"{us / 1e3:9.3f} ms {c:5d}x  {k}")
