"""One partial OTF call (et_attn_partial_fwd) at a given shape, for ncu launch lists:
python tools/partial_prof.py S B [H]."""
import sys, os
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_chenhplg0d021_b200 as et  # noqa: E402

S, B = int(sys.argv[1]), int(sys.argv[2])
H = int(sys.argv[3]) if len(sys.argv) > 3 else 12
d = H * 64
qkv = (torch.randn(B * S, 3 * d, device="cuda") * 0.5).half()
Z = torch.empty(B * S, d, device="cuda").half()
sc = torch.empty(et.attn_partial_scores_bytes(B, S, H, d, "fp16") // 2, dtype=torch.float16, device="cuda")
for _ in range(3):
    et.attn_partial_fwd(qkv, B, S, H, d, 0, d, 2 * d, Z=Z, scores=sc)
    et.attn_core_fwd(qkv, B, S, H, d, 0, d, 2 * d, mode="long", scale=1.0, Z=Z)
torch.cuda.synchronize()
