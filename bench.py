#!/usr/bin/env python
"""bench.py -- RGSQR TFLOPS (2mn^2 - 2n^3/3) and refined LS solve time on B200.

Default (N=1): BASELINE.json config 2, RGSQR of a 65536 x 4096 fp32 N(0,1) matrix, fp16
tensor-core updates; K timed steps after W warm-ups, CUDA events on the launching stream.
Under torchrun (N>1) the path is row-sharded: every rank holds its own
65536 x 4096 block (weak scaling, m = 65536 N), NCCL allreduce/allgather of the small
n x n pieces inside the call; time = max over ranks.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference] [--no-ls]

One JSON line on rank 0.  --impl reference times the fp64 CPU oracle (Householder QR) on a
bounded sample of the same workload on the host cores (tier framing: the oracle is the
reference arm).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

M, N = 65536, 4096                 # BASELINE config 2
LS_M, LS_N, LS_KAPPA = 131072, 1024, 1e4  # BASELINE config 3
ORTH_M, ORTH_N = 2097152, 256     # BASELINE config 4
LR_M, LR_RANK = 32768, 512         # BASELINE config 5
SAMPLE_COLS_CPU = 640              # cpu_baseline: oracle Householder on 65536 x 640 (~10 s)
SAMPLE_COLS_REF = 256              # --impl reference: per-step sample 65536 x 256


def qr_flops(m, n):
    return 2.0 * m * n * n - 2.0 * n ** 3 / 3.0


def peaks():
    p = {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0, "src": "fallback"}
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(path):
        with open(path) as f:
            d = json.load(f)
        p.update({k: d[k] for k in ("hbm_gbs", "bf16_tflops", "bf16_tflops_sustained") if k in d})
        p["src"] = "measured"
    return p


class ClockSampler:
    """nvidia-smi sampling during the timed region (B200_PROFILING.md clocks line)."""

    FIELDS = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index=0):
        self.index = index
        self.rows = []
        self.proc = None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}",
                                          "--format=csv,noheader,nounits", "-lms", "25"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.thread = threading.Thread(target=self._read, daemon=True)
            self.thread.start()
        except Exception:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            parts = [x.strip() for x in line.split(",")]
            if len(parts) == 6:
                self.rows.append(parts)

    def __exit__(self, *a):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=2)
            except Exception:
                self.proc.kill()

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"], "samples": 0}
        sm = [float(r[0]) for r in self.rows if r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in self.rows for i in range(4) if r[2 + i] == "Active"})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(self.rows)}


def dist_env():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


# ------------------------------------------------------------------------ CPU oracle legs
def cpu_cores():
    try:
        return len(os.sched_getaffinity(0))
    except Exception:
        return os.cpu_count() or 1


def time_oracle_qr(m, n, seed):
    import numpy as np
    import oracle
    import synth
    os.environ.setdefault("OMP_NUM_THREADS", str(cpu_cores()))
    A = synth.gaussian(m, n, seed=seed)
    oracle.build()
    t0 = time.perf_counter()
    oracle.householder(A)
    dt = time.perf_counter() - t0
    return dt, qr_flops(m, n) / dt / 1e12


def run_reference(args, ws, rank):
    if rank != 0:
        return
    cores = cpu_cores()
    times = []
    for i in range(args.warmup + args.steps):
        dt, _ = time_oracle_qr(M, SAMPLE_COLS_REF, seed=1000 + i)
        if i >= args.warmup:
            times.append(dt)
    t = sum(times) / len(times)
    tf = qr_flops(M, SAMPLE_COLS_REF) / t / 1e12
    sample = f"fp64 Householder QR (oracle/oracle.c or_householder) of a {M} x {SAMPLE_COLS_REF} N(0,1) sample per step"
    print(json.dumps({
        "impl": "reference", "metric": "RGSQR TFLOPS (2mn^2-2n^3/3)", "value": tf, "unit": "TFLOP/s",
        "n_gpus": ws, "steps": args.steps, "warmup": args.warmup, "ms_per_step": t * 1e3,
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": f"RGSQR {M}x{N} fp32 N(0,1) (BASELINE config 2); reference timed on {M}x{SAMPLE_COLS_REF} samples",
                   "m": M, "n": N},
        "cpu_baseline": {"value": tf, "unit": "TFLOP/s", "cores": cores, "kind": "oracle", "sample": sample},
        "e2e": {"value": tf, "unit": "TFLOP/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }), flush=True)


# ------------------------------------------------------------------------ GPU arm
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-ls", action="store_true")
    ap.add_argument("--no-orth", action="store_true")
    ap.add_argument("--no-bf16", action="store_true")
    ap.add_argument("--no-lowrank", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--no-qrsvd", action="store_true")
    ap.add_argument("--e2e-steps", type=int, default=5)
    ap.add_argument("--comm", default="own", choices=["own", "torch"],
                    help="N > 1: the library's own NCCL communicator or torch's (rg_set_comm)")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3) if args.impl == "ours" else args.warmup
    ws, rank, local = dist_env()
    if args.impl == "reference":
        run_reference(args, ws, rank)
        return

    import numpy as np
    import torch
    import paper_conf_hpdc_zhangbw20_b200 as rg

    torch.cuda.set_device(local)
    dist = None
    if ws > 1:
        import torch.distributed as dist
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    h = rg.Handle(local)
    comm = None
    if ws > 1:
        if args.comm == "torch":
            h.attach_torch_comm()           # rg_set_comm on torch's ProcessGroupNCCL communicator
            comm = "torch ProcessGroupNCCL communicator (rg_set_comm)"
        else:
            h.init_comm(rank, ws)           # the library's own NCCL communicator (rg_comm_init)
            comm = "library NCCL communicator (rg_comm_init)"

    m_global = M * ws
    # synthetic input: N(0,1) fp32 drawn on the device (seeded per rank; > L2 so no flush needed)
    gen = torch.Generator(device="cuda").manual_seed(20200623 + 1 + rank)
    A = torch.randn(N, M, generator=gen, device="cuda", dtype=torch.float32).t()   # column-major M x N
    Q = torch.empty(N, M, device="cuda", dtype=torch.float32).t()
    R = torch.empty(N, N, device="cuda", dtype=torch.float32).t()
    opts = rg.make_opts(sync=False)

    def step():
        rg.rgsqr_factor(A, Q=Q, R=R, handle=h, opts=opts, check=False)

    def barrier():
        torch.cuda.synchronize()
        if dist is not None:
            dist.barrier()
            torch.cuda.synchronize()

    for _ in range(args.warmup):
        step()
    barrier()
    st = torch.cuda.current_stream()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with ClockSampler(local) as clk:
        barrier()
        e0.record(st)
        for _ in range(args.steps):
            step()
        e1.record(st)
        barrier()
    ms = e0.elapsed_time(e1) / args.steps
    if dist is not None:
        t = torch.tensor([ms], device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
    flops = qr_flops(m_global, N)
    tflops = flops / (ms * 1e-3) / 1e12
    launches = int(rg.lib().rg_last_launches(h.ptr)) if hasattr(rg.lib(), "rg_last_launches") else None

    # accuracy of the timed configuration (Hutchinson probes on the device copy; sampled)
    acc = accuracy_probe(rg, torch, A, Q, R)

    # ---- per-kernel profile pass (CUDA events around each kernel class, same stream)
    h.profile(True)
    h.profile_reset()
    for _ in range(2):
        step()
    torch.cuda.synchronize()
    prof = {c: h.profile_get(c) for c in ("update", "proj", "panel", "scale", "other")}
    h.profile(False)
    pk = peaks()
    dom = max(("update", "proj", "panel", "scale"), key=lambda c: prof[c]["ms"])
    d = prof[dom]
    step_ms_prof = sum(p["ms"] for p in prof.values()) / 2
    if dom in ("update", "proj"):
        achieved = d["flops"] / (d["ms"] * 1e-3) / 1e12
        roof = {"kernel": f"K{'2 update' if dom == 'update' else '1 projection'} GEMM (tcgen05)", "bound": "tensor",
                "achieved": achieved, "peak": pk["bf16_tflops_sustained"], "unit": "TFLOP/s",
                "frac": achieved / pk["bf16_tflops_sustained"],
                "peak_src": f"{pk['src']} bf16 sustained (fp16 same rate)"}
    else:
        achieved = d["bytes"] / (d["ms"] * 1e-3) / 1e9
        label = {"panel": "leaf (64-column CholQR2 panel + folded level above; latency-bound)",
                 "scale": "column scaling (colnorm + scale/cast)"}.get(dom, dom)
        roof = {"kernel": label, "bound": "hbm", "achieved": achieved, "peak": pk["hbm_gbs"], "unit": "GB/s",
                "frac": achieved / pk["hbm_gbs"], "peak_src": f"{pk['src']} copy bandwidth"}
    roof["traffic"] = None
    tpath = os.path.join(ROOT, "profiles", "r02_ncu_traffic.json")
    if os.path.exists(tpath):
        with open(tpath) as f:
            tr = json.load(f).get(dom)
        if tr:
            roof["traffic"] = tr["dram_read_bytes"] + tr["dram_write_bytes"]
            roof["traffic_src"] = f"{tr['source']}; algorithmic bytes per launch {d['bytes'] / max(d['launches'], 1):.0f}"
    roof["share_of_step"] = d["ms"] / 2 / step_ms_prof if step_ms_prof > 0 else None
    roof["launches_per_step"] = d["launches"] / 2
    breakdown = {c: {"ms_per_step": p["ms"] / 2, "launches_per_step": p["launches"] / 2,
                     "tflops": (p["flops"] / (p["ms"] * 1e-3) / 1e12) if p["ms"] > 0 and p["flops"] else None,
                     "gbs_alg": (p["bytes"] / (p["ms"] * 1e-3) / 1e9) if p["ms"] > 0 and p["bytes"] else None}
                 for c, p in prof.items()}

    # ---- e2e: same call through the C-ABI with HOST (pinned) buffers, copies inside the region
    e2e = None
    if ws == 1 and args.e2e_steps > 0:
        Ah = torch.empty(N, M, dtype=torch.float32, pin_memory=True)
        Ah.copy_(A.t())
        Ah = Ah.t()
        Qh = torch.empty(N, M, dtype=torch.float32, pin_memory=True).t()
        Rh = torch.empty(N, N, dtype=torch.float32, pin_memory=True).t()
        rg.rgsqr_factor(Ah, Q=Qh, R=Rh, handle=h)  # warm (staging buffers)
        t0 = time.perf_counter()
        for _ in range(args.e2e_steps):
            rg.rgsqr_factor(Ah, Q=Qh, R=Rh, handle=h)
        dt = (time.perf_counter() - t0) / args.e2e_steps
        e2e = {"value": flops / dt / 1e12, "unit": "TFLOP/s", "ms_per_step": dt * 1e3,
               "h2d_bytes_per_step": M * N * 4, "d2h_bytes_per_step": M * N * 4 + N * N * 4,
               "note": "rgsqr_factor on pinned host A/Q/R: column-chunked H2D of A overlapped with the factorization, Q/R columns D2H as their panels finish, status sync"}
        del Ah, Qh, Rh

    ls = None
    if not args.no_ls and ws == 1 and hasattr(rg.lib(), "ls_solve_refined") and not callable(getattr(rg.lib().ls_solve_refined, "__wrapped__", None)):
        try:
            ls = bench_ls(rg, torch, h, pk)
        except Exception as ex:  # keep the headline line even if the LS leg fails
            ls = {"error": str(ex)[:200]}

    # the same factorization with bf16 tensor-core operands (
    # reading #20): time and accuracy next to the fp16 headline
    bf16 = None
    if not args.no_bf16:
        try:
            ob = rg.make_opts(precision="bf16", sync=False)
            for _ in range(3):
                rg.rgsqr_factor(A, Q=Q, R=R, handle=h, opts=ob, check=False)
            torch.cuda.synchronize()
            b0, b1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            b0.record(st)
            for _ in range(5):
                rg.rgsqr_factor(A, Q=Q, R=R, handle=h, opts=ob, check=False)
            b1.record(st)
            torch.cuda.synchronize()
            bms = b0.elapsed_time(b1) / 5
            if dist is not None:
                t = torch.tensor([bms], device="cuda")
                dist.all_reduce(t, op=dist.ReduceOp.MAX)
                bms = float(t.item())
            bf16 = {"ms": bms, "tflops": flops / (bms * 1e-3) / 1e12,
                    "accuracy": accuracy_probe(rg, torch, A, Q, R) if ws == 1 else None,
                    "note": "rgsqr_factor(precision=bf16), same input and options otherwise"}
        except Exception as ex:
            bf16 = {"error": str(ex)[:200]}

    orth = None
    if not args.no_orth:
        try:
            orth = bench_orth(rg, torch, h, ws, rank, dist, pk)
        except Exception as ex:
            orth = {"error": str(ex)[:200]}
    lowrank = None
    if not args.no_lowrank and ws == 1:
        try:
            lowrank = bench_lowrank(rg, torch, h, pk)
        except Exception as ex:
            lowrank = {"error": str(ex)[:200]}

    qrsvd = None
    if not args.no_qrsvd and ws == 1:
        try:
            qrsvd = bench_qrsvd(rg, torch, h, pk)
        except Exception as ex:
            qrsvd = {"error": str(ex)[:200]}

    cpu = None
    if rank == 0 and not args.no_cpu:
        dt, tf = time_oracle_qr(M, SAMPLE_COLS_CPU, seed=7)
        cpu = {"value": tf, "unit": "TFLOP/s", "cores": cpu_cores(), "kind": "oracle",
               "sample": f"fp64 Householder QR (or_householder) of a {M} x {SAMPLE_COLS_CPU} N(0,1) sample "
                         f"({dt:.1f} s), same flop formula"}

    if rank == 0:
        out = {
            "metric": "RGSQR TFLOPS (2mn^2-2n^3/3)", "value": tflops, "unit": "TFLOP/s", "n_gpus": ws,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "fp16-in/fp32-acc (fp32 panel)", "data": "synthetic",
            "config": {"workload": f"RGSQR {m_global}x{N} fp32 N(0,1), fp16 tensor-core updates (BASELINE config 2"
                                   f"{'' if ws == 1 else ', row-sharded ' + str(M) + ' rows per GPU'})",
                       "m": m_global, "n": N, "nb": 32, "l2": "inputs (1 GiB per GPU) larger than L2, no flush",
                       "parallelism": f"row-sharded x{ws}" if ws > 1 else "single GPU", "comm": comm},
            "frac_of_spec_2250": tflops / 2250.0,
            "frac_of_measured_matmul": tflops / pk["bf16_tflops"],
            "accuracy": acc,
            "roofline": roof,
            "breakdown": breakdown,
            "cpu_baseline": cpu,
            "e2e": e2e,
            "ls": ls,
            "orthogonalize": orth,
            "bf16": bf16,
            "lowrank": lowrank,
            "qrsvd": qrsvd,
            "gpu_launches": (launches * args.steps) if launches else None,
            "clocks": clk.summary(),
        }
        print(json.dumps(out), flush=True)
    if dist is not None:
        dist.barrier()
        dist.destroy_process_group()


def accuracy_probe(rg, torch, A, Q, R, p=8):
    """Hutchinson estimates (fp64) of ||A-QR||_F/||A||_F and ||I-Q^T Q||_F on the device."""
    g = torch.Generator(device="cuda").manual_seed(99)
    n = A.shape[1]
    G = torch.randn(n, p, generator=g, device="cuda", dtype=torch.float64)
    A64, Q64, R64 = A.double(), Q.double(), R.double()
    be = (torch.linalg.norm(A64 @ G - Q64 @ (R64 @ G)) / torch.linalg.norm(A64 @ G)).item()
    orth = (torch.linalg.norm(G - Q64.t() @ (Q64 @ G)) / p ** 0.5).item()
    del A64, Q64, R64
    return {"backward_error": be, "orthogonality_F": orth, "method": "8 Hutchinson probes, fp64 (torch, check only)"}


def _time_calls(torch, call, restore, reps):
    """CUDA events around each call on the current stream; the untimed restore runs before it."""
    st = torch.cuda.current_stream()
    ts = []
    for _ in range(reps):
        restore()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(st)
        out = call()
        e1.record(st)
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    return ts, out


def bench_orth(rg, torch, h, ws, rank, dist, pk):
    """BASELINE config 4: orthogonalisation of 2,097,152 x 256 N(0,1), row-sharded over the ws ranks
    (strong scaling: 2,097,152 / ws rows per rank), reortho until orth <= 1e-5.  Time = max over
    ranks of the median of 5 calls.  HBM roofline: 8 m n bytes per pass (read A, write Q)."""
    m_all, n = ORTH_M, ORTH_N
    m = m_all // ws
    g = torch.Generator(device="cuda").manual_seed(20200623 + 4 + rank)
    A0 = torch.randn(n, m, generator=g, device="cuda", dtype=torch.float32).t()
    A = torch.empty_like(A0.t()).t()
    R = torch.zeros(n, n, device="cuda").t()
    res = {}

    def call():
        _, _, passes, est = rg.orthogonalize(A, R, orth_tol=1e-5, max_passes=3, handle=h)
        res["passes"], res["est"] = passes, est

    ts, _ = _time_calls(torch, call, lambda: A.copy_(A0), 2 + 5)
    ms = statistics.median(ts[2:])
    two = {}

    def call2():   # fixed CholQR2 / RGSQR + one reorthogonalisation pass (orth_tol = 0)
        _, _, passes, est = rg.orthogonalize(A, R, orth_tol=0.0, max_passes=2, handle=h)
        two["passes"], two["est"] = passes, est

    ts2, _ = _time_calls(torch, call2, lambda: A.copy_(A0), 2 + 5)
    ms2 = statistics.median(ts2[2:])
    if dist is not None:
        t = torch.tensor([ms, ms2], device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms, ms2 = float(t[0].item()), float(t[1].item())
    passes = res["passes"]
    alg_bytes = 8.0 * m_all * n * passes
    gbs = alg_bytes / (ms * 1e-3) / 1e9
    peak = pk["hbm_gbs"] * ws
    del A0, A
    return {"workload": f"orthogonalize {m_all}x{n} N(0,1), reortho to 1e-5 (BASELINE config 4), "
                        f"{'row-sharded x' + str(ws) if ws > 1 else '1 GPU'}",
            "ms": ms, "passes": passes, "orth_est": res["est"],
            "path": "tall CholQR passes on tcgen05 (split 16-bit Gram, fp64 norms; reading #33)" if m >= 131072
                    else "RGSQR passes",
            "two_pass": {"ms": ms2, "passes": two["passes"], "orth_est": two["est"],
                         "note": "orth_tol = 0, max_passes = 2: the factorization pass plus one reorthogonalisation pass"},
            "tflops": passes * qr_flops(m_all, n) / (ms * 1e-3) / 1e12,
            "roofline": {"bound": "hbm", "achieved": gbs, "peak": peak, "unit": "GB/s", "frac": gbs / peak,
                         "alg_bytes": alg_bytes, "note": "8 m n bytes per pass (read A fp32, write Q fp32)"}}


def bench_lowrank(rg, torch, h, pk):
    """BASELINE config 5: randomized rank-512 approximation of a 32768 x 32768 matrix (p = 16,
    q = 1).  Roofline: max(HBM, tensor) over the (2 + 2q) passes over A, each 2 m n l flops and
    4 m n bytes (fp32 A read)."""
    import numpy as np
    import synth
    m = n = LR_M
    rank, p, q = LR_RANK, 16, 1
    At, s = synth.lowrank_matrix(m, n, 2048, "geometric", 1e6, seed=synth.SEED_BASE + 5, device="cuda")
    A = At.t()
    U = torch.empty(rank, m, device="cuda").t()
    S = torch.empty(rank, device="cuda")
    V = torch.empty(rank, n, device="cuda").t()

    def call():
        rg.lowrank_approx(A, rank, oversample=p, power_iters=q, seed=7, U=U, S=S, V=V, handle=h)

    ts, _ = _time_calls(torch, call, lambda: None, 2 + 5)
    ms = statistics.median(ts[2:])
    l = rank + p
    passes = 2 + 2 * q
    t_tc = passes * 2.0 * m * n * l / (pk["bf16_tflops_sustained"] * 1e12)
    t_hbm = passes * 4.0 * m * n / (pk["hbm_gbs"] * 1e9)
    roof_ms = max(t_tc, t_hbm) * 1e3
    # accuracy: ||A - U S V^T||_F / ||A||_F against the closed-form optimum (check only)
    U64, V64, S64 = U.double(), V.double(), S.double()
    num = 0.0
    for j0 in range(0, n, 4096):
        num += torch.linalg.norm(A[:, j0:j0 + 4096].double() - (U64 * S64) @ V64[j0:j0 + 4096].t()).item() ** 2
    err = (num / float(np.sum(s ** 2))) ** 0.5
    opt = float(np.sqrt(np.sum(s[rank:] ** 2) / np.sum(s ** 2)))
    del A, At, U64, V64
    return {"workload": f"randomized low rank {m}x{n}, rank {rank}, p {p}, q {q} (BASELINE config 5)",
            "ms": ms, "lr_error": err, "lr_optimal": opt, "ratio_to_optimal": err / opt,
            "roofline": {"bound": "hbm" if t_hbm >= t_tc else "tensor", "roofline_ms": roof_ms,
                         "frac": roof_ms / ms,
                         "note": f"{passes} passes over fp32 A: max({passes} x 2mnl flops at the sustained bf16 peak, "
                                 f"{passes} x 4mn bytes at the copy bandwidth)"}}


def bench_qrsvd(rg, torch, h, pk):
    """deterministic QR-SVD low rank of the paper's Table 4 matrix (524288 x 1024,
    arithmetic singular values, cond 1e6), rank 512.  Time = median of 3 calls (CUDA events);
    the QR part is timed separately (rgsqr_factor on the same matrix); error vs the printed 3.53e-01."""
    import numpy as np
    import synth
    m, n, r = 524288, 1024, 512
    At, s = synth.svd_matrix_device(m, n, "arithmetic", 1e6, seed=4)
    A = At.t()
    U = torch.empty(r, m, device="cuda").t()
    S = torch.empty(r, device="cuda")
    V = torch.empty(r, n, device="cuda").t()
    ts, _ = _time_calls(torch, lambda: rg.lowrank_qrsvd(A, r, U=U, S=S, V=V, handle=h), lambda: None, 1 + 3)
    ms = statistics.median(ts[1:])
    Q = torch.empty(n, m, device="cuda").t()
    R = torch.empty(n, n, device="cuda").t()
    oq = rg.make_opts(sync=False)
    tq, _ = _time_calls(torch, lambda: rg.rgsqr_factor(A, Q=Q, R=R, handle=h, opts=oq, check=False), lambda: None,
                        2 + 3)
    qr_ms = statistics.median(tq[2:])
    del Q, R
    num = 0.0
    Us = U.double() * S.double()
    Vt = V.double().t()
    for i0 in range(0, m, 65536):
        num += torch.linalg.norm(A[i0:i0 + 65536].double() - Us[i0:i0 + 65536] @ Vt).item() ** 2
    err = float(np.sqrt(num) / torch.linalg.norm(At.double()).item())
    opt = float(np.sqrt(np.sum(s[r:] ** 2) / np.sum(s ** 2)))
    # roofline of the QR part (the paper's dominant step): 2mn^2 - 2n^3/3 at the sustained peak
    qr_roof_ms = qr_flops(m, n) / (pk["bf16_tflops_sustained"] * 1e12) * 1e3
    del A, At, U, Us, Vt
    return {"workload": f"QR-SVD rank {r} of {m}x{n}, arithmetic sigma, cond 1e6 (paper Table 4)", "ms": ms,
            "qr_ms": qr_ms, "svd_and_products_ms": ms - qr_ms, "error": err, "printed_error": 0.353,
            "optimal_error": opt, "paper_v100_ms": 274.95,
            "roofline": {"bound": "tensor (QR part)", "qr_roofline_ms": qr_roof_ms, "qr_frac": qr_roof_ms / qr_ms,
                         "note": "QR at the sustained bf16 peak; the 1024x1024 Jacobi SVD (block one-sided, fp64) "
                                 "is latency-bound and has no bandwidth roofline"}}


def bench_ls(rg, torch, h, pk):
    import numpy as np
    import synth
    A = synth.svd_matrix(LS_M, LS_N, "geometric", LS_KAPPA, seed=synth.SEED_BASE + 2)
    b = synth.rhs(A, seed=synth.SEED_BASE + 2, consistent=False)
    x_ref = np.linalg.lstsq(A, b, rcond=None)[0]   # check only (LAPACK), not timed
    Ad = torch.from_numpy(np.ascontiguousarray(A.T.astype(np.float32))).cuda().t()
    bd = torch.from_numpy(b.astype(np.float32)).cuda()
    x = torch.zeros(LS_N, dtype=torch.float64, device="cuda")
    for _ in range(2):
        rg.ls_solve_refined(Ad, bd, x, handle=h)
    torch.cuda.synchronize()
    st = torch.cuda.current_stream()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(st)
    reps = 5
    for _ in range(reps):
        _, it, rel, status = rg.ls_solve_refined(Ad, bd, x, handle=h)
    e1.record(st)
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / reps
    # fe against the fp32-rounded problem's LAPACK solution
    x_ref32 = np.linalg.lstsq(A.astype(np.float32).astype(np.float64), b.astype(np.float32).astype(np.float64),
                              rcond=None)[0]
    xv = x.cpu().numpy()
    # roofline: one read of A per CGLS iteration (the one-pass product, reading
    # #24) plus the initial A^T b, at the copy bandwidth, + the one split-precision RGSQR pass of
    # the default preconditioner (reading #8: three 16-bit products per K1 / K2) at the sustained
    # tensor peak
    roof_ms = ((it + 1) * 4.0 * LS_M * LS_N / (pk["hbm_gbs"] * 1e9)
               + 3 * qr_flops(LS_M, LS_N) / (pk["bf16_tflops_sustained"] * 1e12)) * 1e3
    # LSQR (NEXT-4) on the same problem and preconditioner
    ol = rg.make_opts(solver="lsqr")
    xl = torch.zeros(LS_N, dtype=torch.float64, device="cuda")
    rg.ls_solve_refined(Ad, bd, xl, handle=h, opts=ol)
    torch.cuda.synchronize()
    e0.record(st)
    for _ in range(reps):
        _, it_l, _, _ = rg.ls_solve_refined(Ad, bd, xl, handle=h, opts=ol)
    e1.record(st)
    torch.cuda.synchronize()
    lsqr = {"ms": e0.elapsed_time(e1) / reps, "iters": it_l,
            "fe_vs_fp32_problem": float(np.linalg.norm(xl.cpu().numpy() - x_ref32) / np.linalg.norm(x_ref32))}
    return {"workload": f"LS {LS_M}x{LS_N} cond 1e4 geometric, b ~ N(0,1) (BASELINE config 3)", "ms": ms,
            "lsqr": lsqr,
            "roofline": {"roofline_ms": roof_ms, "frac": roof_ms / ms,
                         "note": "(iters + 1) x 4mn bytes (A read once per CGLS iteration) at the copy bandwidth "
                                 "+ one split-precision RGSQR pass (3 x 16-bit products) at the sustained tensor peak"},
            "preconditioner": "one RGSQR pass with split-precision K1/K2, no reortho pass (reading #8)",
            "iters": it, "relres": rel, "status": status,
            "fe_vs_fp32_problem": float(np.linalg.norm(xv - x_ref32) / np.linalg.norm(x_ref32)),
            "fe_vs_fp64_problem": float(np.linalg.norm(xv - x_ref) / np.linalg.norm(x_ref))}


if __name__ == "__main__":
    main()
