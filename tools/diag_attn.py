import sys, math, numpy as np, torch
sys.path.insert(0, '.')
import paper_conf_sc_chenhplg0d021_b200 as etm
S, dk, causal, mode = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3]), sys.argv[4]
B, H = 3, 2
d = H * dk
g = np.random.default_rng(0)
qkv = torch.tensor(g.standard_normal((B * S, 3 * d)), dtype=torch.float16, device='cuda')
L = torch.full((B,), S, dtype=torch.int32, device='cuda')
Z = etm.attn_core_fwd(qkv, B, S, H, d, 0, d, 2 * d, lengths=L, causal=bool(causal), mode=mode, scale=1 / math.sqrt(dk))
torch.cuda.synchronize()
print("OK", S, dk, causal, mode, float(Z.float().abs().max()))
