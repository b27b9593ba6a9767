"""One eager encoder forward of a config (for ncu launch lists): python tools/one_forward.py C2 [scheme]"""
import sys, os
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_chenhplg0d021_b200 as et  # noqa: E402
from et_synth import CONFIGS, make_layer, make_lengths, make_x  # noqa: E402

cfg = CONFIGS[sys.argv[1] if len(sys.argv) > 1 else "C2"]
if len(sys.argv) > 2:   # scheme override, e.g. "tile" for an attention-aware config
    cfg = cfg.with_(scheme=sys.argv[2], layers=1)
layers = [et.pack_layer(make_layer(cfg, l), cfg.scheme, cfg.ratio, cfg.heads, cfg.dtype) for l in range(cfg.layers)]
L = torch.from_numpy(make_lengths(cfg, ragged=False)).cuda()
enc = et.Encoder(layers, cfg.batch, cfg.seq_len, cfg.heads, cfg.d_ff, act=cfg.act, ln_eps=cfg.ln_eps,
                 dtype=cfg.dtype, resid_dtype=cfg.dtype, causal=cfg.causal, mode=cfg.attn_mode, lengths=L)
X = torch.from_numpy(make_x(cfg).reshape(cfg.tokens, cfg.d_model)).cuda().half()
out = torch.empty_like(X)
torch.cuda.synchronize()
torch.cuda.nvtx.range_push("fwd")
for _ in range(2):
    enc(X, out)
torch.cuda.synchronize()
