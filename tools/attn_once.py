"""One short-form attention launch on a random QKV buffer (for ncu): python tools/attn_once.py B S H d [causal]"""
import sys, os
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_chenhplg0d021_b200 as et  # noqa: E402
B, S, H, d = [int(a) for a in sys.argv[1:5]]
causal = len(sys.argv) > 5 and sys.argv[5] == "causal"
qkv = torch.randn(B * S, 3 * d, device="cuda").half()
for _ in range(3):
    et.attn_core_fwd(qkv, B, S, H, d, 0, d, 2 * d, scale=(d // H) ** -0.5, causal=causal, mode="short")
torch.cuda.synchronize()
