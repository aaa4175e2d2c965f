import os, sys, time
sys.path.insert(0, "/root/repo")
import torch
import paper_conf_hpdc_zhangbw20_b200 as rg
P = int(sys.argv[1]) if len(sys.argv) > 1 else 2
m, n = 65536, 4096
group = rg.VGroup(P)
streams = [torch.cuda.Stream() for _ in range(P)]
hs = [rg.Handle(0, stream=s.cuda_stream) for s in streams]
for r, h in enumerate(hs):
    h.set_vcomm(group, r)
As = [torch.randn(n, m, device="cuda").t() for _ in range(P)]
Qs = [torch.empty(n, m, device="cuda").t() for _ in range(P)]
Rs = [torch.empty(n, n, device="cuda").t() for _ in range(P)]
def call():
    rg.run_ranks([lambda r=r: rg.rgsqr_factor(As[r], Q=Qs[r], R=Rs[r], handle=hs[r]) for r in range(P)])
    torch.cuda.synchronize()
call()
ts = []
for _ in range(3):
    t0 = time.perf_counter(); call(); ts.append(time.perf_counter() - t0)
print(f"P={P} virtual ranks x {m}x{n}: {min(ts)*1e3:.1f} ms wall (one GPU; per-rank dist-path estimate {min(ts)*1e3/P:.1f} ms), launches/rank {hs[0].last_launches()}")
for h in hs: h.close()
group.close()
