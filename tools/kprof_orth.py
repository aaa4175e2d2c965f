"""CUPTI kernel breakdown of orthogonalize at BASELINE config 4 (2,097,152 x 256) (development tool)."""
import collections
import os
import sys
import time

import torch
from torch.profiler import ProfilerActivity, profile

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_hpdc_zhangbw20_b200 as rg  # noqa: E402

m, n = 2097152, 256
g = torch.Generator(device="cuda").manual_seed(5)
A0 = torch.randn(n, m, device="cuda", generator=g).t()
A = torch.empty_like(A0)
h = rg.Handle(0)
for _ in range(2):
    A.copy_(A0)
    rg.orthogonalize(A, None, orth_tol=1e-5, max_passes=3, handle=h)
torch.cuda.synchronize()
A.copy_(A0)
t0 = time.perf_counter()
_, _, p, est = rg.orthogonalize(A, None, orth_tol=1e-5, max_passes=3, handle=h)
torch.cuda.synchronize()
print(f"orth: {(time.perf_counter() - t0) * 1e3:.2f} ms wall, passes {p}, est {est:.3e}")
A.copy_(A0)
torch.cuda.synchronize()
with profile(activities=[ProfilerActivity.CUDA]) as prof:
    rg.orthogonalize(A, None, orth_tol=1e-5, max_passes=3, handle=h)
    torch.cuda.synchronize()
agg = collections.defaultdict(lambda: [0, 0.0])
for ev in prof.events():
    if ev.device_type == torch.autograd.DeviceType.CUDA and "Memcpy" not in ev.name:
        agg[ev.name[:80]][0] += 1
        agg[ev.name[:80]][1] += ev.device_time_total
tot = sum(v[1] for v in agg.values())
print(f"kernel time sum {tot / 1e3:.3f} ms")
for k, (c, us) in sorted(agg.items(), key=lambda kv: -kv[1][1])[:8]:
    print(f"  {us / 1e3:8.3f} ms {c:4d}x  {k}")
