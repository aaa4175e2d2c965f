"""One orthogonalize call at BASELINE config 4 (2,097,152 x 256), for ncu captures."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_hpdc_zhangbw20_b200 as rg  # noqa: E402

m, n = (int(sys.argv[1]), int(sys.argv[2])) if len(sys.argv) > 2 else (2097152, 256)
A = torch.randn(n, m, device="cuda").t()
passes = int(os.environ.get("ORTH_PASSES", "3"))
tol = float(os.environ.get("ORTH_TOL", "1e-5"))
_, _, p, est = rg.orthogonalize(A, None, orth_tol=tol, max_passes=passes)
torch.cuda.synchronize()
print(f"orthogonalize {m}x{n}: passes {p} est {est:.3e}")
