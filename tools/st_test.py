import sys, torch
sys.path.insert(0, '.')
import paper_conf_sc_chenhplg0d021_b200 as etm
from et_synth import make_matrix
W = make_matrix(10, (256, 768), 0.05, "fp16"); X = make_matrix(12, (128, 768), 1.0, "fp16")
pk = etm.prune_pack(torch.tensor(W, dtype=torch.float16, device='cuda'), "tile", 0.0)
Y = etm.linear_fwd(pk, torch.tensor(X, dtype=torch.float16, device='cuda'), None, etm.EPI_BIAS)
torch.cuda.synchronize()
print("ok", Y.float().abs().sum().item())
