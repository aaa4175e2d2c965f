import os, sys, time, collections
sys.path.insert(0, "/root/repo")
import torch
from torch.profiler import profile, ProfilerActivity
import paper_conf_hpdc_zhangbw20_b200 as rg
import synth
At, s = synth.svd_matrix_device(524288, 1024, "arithmetic", 1e6, seed=4)
A = At.t()
h = rg.Handle(0)
rg.lowrank_qrsvd(A, 512, handle=h); torch.cuda.synchronize()
t0 = time.perf_counter(); rg.lowrank_qrsvd(A, 512, handle=h); torch.cuda.synchronize(); print("wall ms", (time.perf_counter()-t0)*1e3)
with profile(activities=[ProfilerActivity.CUDA]) as prof:
    rg.lowrank_qrsvd(A, 512, handle=h); torch.cuda.synchronize()
agg = collections.defaultdict(lambda: [0, 0.0])
for ev in prof.events():
    if ev.device_type == torch.autograd.DeviceType.CUDA:
        agg[ev.name[:70]][0] += 1; agg[ev.name[:70]][1] += ev.device_time_total
tot = sum(v[1] for v in agg.values()); print("kernel sum ms", tot/1e3)
for k,(c,us) in sorted(agg.items(), key=lambda kv:-kv[1][1])[:6]: print(f"{us/1e3:8.3f} ms {c:5d}x {k}")
