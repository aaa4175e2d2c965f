"""profiles/<round>_ncu_traffic.json from the leaf ncu report (bench.py's roofline `traffic`)."""
import csv, io, json, subprocess, sys
rep, out, tag = sys.argv[1], sys.argv[2], sys.argv[3]
rows = list(csv.reader(io.StringIO(subprocess.check_output(["ncu", "-i", rep, "--page", "raw", "--csv"], text=True))))
h = rows[0]
r = rows[2]   # first profiled launch: the plain leaf
val = lambda k: float(r[h.index(k)].replace(",", ""))
unit = lambda k: rows[1][h.index(k)]
def to_bytes(k):
    u = unit(k)
    return val(k) * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(u, 1)
d = {"panel": {"kernel": r[h.index("Kernel Name")].split("(")[0] + " (plain 64-column leaf)",
               "dram_read_bytes": to_bytes("dram__bytes_read.sum"), "dram_write_bytes": to_bytes("dram__bytes_write.sum"),
               "duration_ns_under_ncu": val("gpu__time_duration.sum") * {"usecond": 1e3, "us": 1e3, "msecond": 1e6, "ms": 1e6}.get(unit("gpu__time_duration.sum"), 1),
               "source": f"profiles/{tag}_ncu_leaf.md (ncu --set full, leaf_kernel, m=65536, 64 columns, tools/profile_round.sh {tag})",
               "note": "Q / shadow writes are still resident in the 126 MB L2 when the kernel ends, so most DRAM write bytes are attributed to later kernels"}}
json.dump(d, open(out, "w"), indent=1)
print(json.dumps(d, indent=1))
