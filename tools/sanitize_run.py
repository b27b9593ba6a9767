"""One small forward of each kind for compute-sanitizer (SURVEY §4 tier T6): C1 (FP32 validation build
and FP16), C2 (attention-aware, causal), a ragged short C3 slice and a long-form C4 slice."""
import sys
import numpy as np
import torch
sys.path.insert(0, '.')
import paper_conf_sc_chenhplg0d021_b200 as et
from et_synth import CONFIGS, make_layer, make_lengths, make_x

cases = [("C1", {}), ("C1", {"dtype": "fp16"}), ("C2", {}), ("C3", {"layers": 1, "batch": 2}),
         ("C4", {"layers": 1, "batch": 1, "seq_len": 384})]
if len(sys.argv) > 1:
    cases = [c for c in cases if c[0] in sys.argv[1:]]
for key, kw in cases:
    cfg = CONFIGS[key].with_(**kw)
    raws = [make_layer(cfg, l) for l in range(cfg.layers)]
    layers = [et.pack_layer(r, cfg.scheme, cfg.ratio, cfg.heads, cfg.dtype) for r in raws]
    L = torch.from_numpy(make_lengths(cfg)).cuda()
    enc = et.Encoder(layers, cfg.batch, cfg.seq_len, cfg.heads, cfg.d_ff, act=cfg.act, ln_eps=cfg.ln_eps,
                     dtype=cfg.dtype, causal=cfg.causal, mode=cfg.attn_mode, lengths=L)
    X = torch.from_numpy(make_x(cfg).reshape(cfg.tokens, cfg.d_model)).cuda().to(et.torch_dtype(cfg.dtype))
    Y = enc(X)
    torch.cuda.synchronize()
    print(key, kw, "ok", float(Y.float().abs().max()))
