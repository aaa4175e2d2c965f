import sys; sys.path.insert(0, "/root/repo")
import torch, synth
import paper_conf_hpdc_zhangbw20_b200 as rg
At, s = synth.lowrank_matrix(32768, 32768, 2048, "geometric", 1e6, seed=7, device="cuda")
rg.lowrank_approx(At.t(), 512, oversample=16, power_iters=1, seed=7)
torch.cuda.synchronize(); print("ok")
