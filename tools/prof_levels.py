"""Per-op event profile of one call, summarised per (class, width).

RG_CALL=factor (default, BASELINE config 2: RG_M x RG_N) | orth (orthogonalize, config 4 with
RG_M=2097152 RG_N=256) | lowrank (config 5, RG_M x RG_M, rank 512)."""
import os, sys, subprocess, collections, re
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
if os.environ.get("_PROF_CHILD") is None:
    env = dict(os.environ, RGSQR_PROF_OPS="1", _PROF_CHILD="1")
    p = subprocess.run([sys.executable, __file__] + sys.argv[1:], env=env, capture_output=True, text=True)
    names = {0: "K2 update", 1: "K1 proj", 2: "panel", 3: "scale", 5: "other"}
    agg = collections.OrderedDict()
    for line in p.stderr.splitlines():
        mm = re.match(r"\[rgsqr op\] cls (\d+) w (\d+) us ([\d.]+) TF ([\d.a-z]+) GB/s ([\d.a-z]+)", line)
        if not mm:
            continue
        k = (names.get(int(mm.group(1)), mm.group(1)), int(mm.group(2)))
        a = agg.setdefault(k, [0, 0.0, []])
        a[0] += 1; a[1] += float(mm.group(3)); a[2].append((float(mm.group(4)), float(mm.group(5))))
    print(p.stdout)
    if p.returncode != 0:
        print("child failed, rc", p.returncode, "\n", "\n".join(p.stderr.splitlines()[-20:]))
    tot = sum(v[1] for v in agg.values())
    for (c, w), (n, us, tg) in sorted(agg.items(), key=lambda kv: (kv[0][0], -kv[0][1])):
        tf = sum(t for t, _ in tg) / len(tg); gb = sum(g for _, g in tg) / len(tg)
        print(f"{c:10s} w={w:5d} n={n:4d} total {us/1e3:7.3f} ms  avg {us/n:8.2f} us  {tf:7.1f} TF  {gb:7.0f} GB/s")
    print(f"sum {tot/1e3:.3f} ms (events per op, one call)")
    sys.exit(p.returncode)
import torch
import paper_conf_hpdc_zhangbw20_b200 as rg
m = int(os.environ.get("RG_M", 65536)); n = int(os.environ.get("RG_N", 4096))
call = os.environ.get("RG_CALL", "factor")
h = rg.Handle(0)
if call == "lowrank":
    n = m
A = torch.randn(n, m, device="cuda").t()
A0 = A.clone() if call == "orth" else None
Q = torch.empty(n, m, device="cuda").t() if call == "factor" else None
R = torch.empty(n, n, device="cuda").t() if call != "lowrank" else None
o = rg.make_opts(sync=False)


def run():
    if call == "factor":
        rg.rgsqr_factor(A, Q=Q, R=R, handle=h, opts=o, check=False)
    elif call == "orth":
        A.copy_(A0)
        print("passes", rg.orthogonalize(A, R, orth_tol=1e-5, max_passes=3, handle=h)[2:])
    else:
        rg.lowrank_approx(A, 512, oversample=16, power_iters=1, seed=7, handle=h)


for _ in range(3):
    run()
torch.cuda.synchronize()
h.profile(True); h.profile_reset()
ev = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
ev[0].record()
run()
ev[1].record()
torch.cuda.synchronize()
print("call ms (events, profiling on)", ev[0].elapsed_time(ev[1]))
print({c: h.profile_get(c) for c in ("update", "proj", "panel", "scale", "other")})
