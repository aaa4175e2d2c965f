"""Top CUDA source lines by warp-stall samples from an ncu report (development tool).
python tools/ncu_lines.py report.ncu-rep [N]   (needs -lineinfo builds)"""
import csv, io, subprocess, sys
path = sys.argv[1]
N = int(sys.argv[2]) if len(sys.argv) > 2 else 30
out = subprocess.check_output(["ncu", "-i", path, "--page", "source", "--csv", "--print-source", "cuda,sass"], text=True)
rows = list(csv.reader(io.StringIO(out)))
hdr = None
fname = "?"
lines = []
cur = None
for r in rows:
    if r and r[0] == "File Path":
        fname = r[1].split("/")[-1]
        continue
    if r and r[0] == "Line No":
        hdr = r
        si = hdr.index("Warp Stall Sampling (All Samples)")
        continue
    if not hdr or len(r) < si:
        continue
    if r[0]:
        cur = [fname, r[0], r[1], 0.0]
        lines.append(cur)
        try:
            cur[3] += float(r[si] or 0)
        except ValueError:
            pass
tot = sum(l[3] for l in lines)
print("total samples", tot)
for l in sorted(lines, key=lambda l: -l[3])[:N]:
    print(f"{l[0]}:{l[1]:>5} {100 * l[3] / tot:5.1f}%  {l[2].strip()[:100]}")
