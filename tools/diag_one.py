import sys, numpy as np, torch
sys.path.insert(0, '.')
import paper_conf_sc_chenhplg0d021_b200 as etm
from et_synth import make_matrix
N, d, M, ratio = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3]), float(sys.argv[4])
W = make_matrix(10, (N, d), 0.05, "fp16"); X = make_matrix(12, (M, d), 1.0, "fp16")
pk = etm.prune_pack(torch.tensor(W, dtype=torch.float16, device='cuda'), "tile", ratio)
Y = etm.linear_fwd(pk, torch.tensor(X, dtype=torch.float16, device='cuda'), None, etm.EPI_BIAS)
torch.cuda.synchronize(); print("OK")
