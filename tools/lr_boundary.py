import sys; sys.path.insert(0, "/root/repo")
import numpy as np, torch, oracle, synth
import paper_conf_hpdc_zhangbw20_b200 as rg
def dev(A): return torch.from_numpy(np.ascontiguousarray(np.asarray(A, dtype=np.float32).T)).cuda().t()
A, s = synth.lowrank_matrix(2048, 1024, 600, "geometric", 1e6, seed=51)
A64 = A.astype(np.float64)
for rank in [int(r) for r in (sys.argv[1].split(",") if len(sys.argv) > 1 else ["230", "240", "241", "250", "300"])]:
    U, S, V = rg.lowrank_approx(dev(A), rank, oversample=16, power_iters=1, seed=1234)
    U, S, V = (x.cpu().numpy().astype(np.float64) for x in (U, S, V))
    err = oracle.lowrank_error(A64, U, S, V)
    sfull = np.zeros(1024); sfull[:600] = s
    opt = np.sqrt(np.sum(sfull[rank:] ** 2) / np.sum(sfull ** 2))
    print(f"rank {rank} l {rank+16}: err {err:.3e} opt {opt:.3e} ratio {err/opt:.2f}")
