"""Per-op event profile of one RGSQR call at BASELINE config 2, summarised per (class, width)."""
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
h = rg.Handle(0)
A = torch.randn(n, m, device="cuda").t()
Q = torch.empty(n, m, device="cuda").t(); R = torch.empty(n, n, device="cuda").t()
o = rg.make_opts(sync=False)
for _ in range(3):
    rg.rgsqr_factor(A, Q=Q, R=R, handle=h, opts=o, check=False)
torch.cuda.synchronize()
h.profile(True); h.profile_reset()
rg.rgsqr_factor(A, Q=Q, R=R, handle=h, opts=o, check=False)
torch.cuda.synchronize()
print({c: h.profile_get(c) for c in ("update", "proj", "panel", "scale", "other")})
