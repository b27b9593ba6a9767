import sys, numpy as np, torch
sys.path.insert(0, '.')
import paper_conf_sc_chenhplg0d021_b200 as etm
from et_synth import make_matrix
from oracle import prune as op, encoder as oe
for (N, d, M, ratio) in [(2304, 768, 128, 0.0), (256, 768, 128, 0.0), (128, 256, 128, 0.0), (2304, 768, 128, 0.8)]:
    W = make_matrix(10, (N, d), 0.05, "fp16"); X = make_matrix(12, (M, d), 1.0, "fp16")
    pk = etm.prune_pack(torch.tensor(W, dtype=torch.float16, device='cuda'), "tile", ratio)
    Y = etm.linear_fwd(pk, torch.tensor(X, dtype=torch.float16, device='cuda'), None, etm.EPI_BIAS)
    torch.cuda.synchronize()
    ref = oe.linear(X, op.prune_tile(W, ratio)["W_pruned"], None)
    g = Y.float().cpu().numpy()
    err = np.abs(g - ref).reshape(M, N // 16, 16).max(axis=(0, 2))
    bad = np.nonzero(err > 0.02)[0]
    print(N, d, M, ratio, "bad tile rows:", bad.tolist()[:60], "n_bad", len(bad), "/", N // 16)
    errm = np.abs(g - ref).reshape(4, 32, N).max(axis=(1, 2))
    print("  err by lane quarter", errm)
