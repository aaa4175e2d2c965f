"""PCIe floor of the e2e leg (development tool): 1 GiB pinned H2D alone, 1.06 GiB D2H alone, and
both at once on two streams (the pipelined rgsqr_factor cannot beat the concurrent figure)."""
import torch
n = 1 << 28   # floats = 1 GiB
h_in = torch.empty(n, dtype=torch.float32, pin_memory=True)
h_out = torch.empty(n + n // 16, dtype=torch.float32, pin_memory=True)
d_in = torch.empty(n, dtype=torch.float32, device="cuda")
d_out = torch.empty(n + n // 16, dtype=torch.float32, device="cuda")
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
def timed(f, reps=3):
    best = 1e9
    for _ in range(reps):
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        f()
        e1.record()
        torch.cuda.synchronize()
        best = min(best, e0.elapsed_time(e1))
    return best
def h2d():
    with torch.cuda.stream(s1):
        d_in.copy_(h_in, non_blocking=True)
    torch.cuda.current_stream().wait_stream(s1)
def d2h():
    with torch.cuda.stream(s2):
        h_out.copy_(d_out, non_blocking=True)
    torch.cuda.current_stream().wait_stream(s2)
def both():
    s1.wait_stream(torch.cuda.current_stream()); s2.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s1):
        d_in.copy_(h_in, non_blocking=True)
    with torch.cuda.stream(s2):
        h_out.copy_(d_out, non_blocking=True)
    torch.cuda.current_stream().wait_stream(s1); torch.cuda.current_stream().wait_stream(s2)
a, b, c = timed(h2d), timed(d2h), timed(both)
print(f"H2D 1 GiB {a:.2f} ms ({4 * n / a / 1e6:.1f} GB/s); D2H 1.06 GiB {b:.2f} ms ({4.25 * n / b / 1e6:.1f} GB/s); "
      f"both concurrently {c:.2f} ms")
