"""C5 full depth (12 layers, S = 2048) parity margin vs residual-stream dtype (reading C-22), and the
throughput cost of each choice (sequences 0 and 1 compared with the oracle; batch 4)."""
import sys
import time
import numpy as np
import torch
sys.path.insert(0, '.')
import paper_conf_sc_chenhplg0d021_b200 as et
from et_synth import CONFIGS, make_layer, make_lengths, make_x
from oracle import encoder as oe
cfg = CONFIGS["C5"].with_(batch=4)
raws = [make_layer(cfg, l) for l in range(cfg.layers)]
X = make_x(cfg)
lens = make_lengths(cfg)
ref = oe.encoder(X[:2].astype(np.float64), [oe.prune_layer(r, cfg.scheme, cfg.ratio)[0] for r in raws], cfg.heads,
                 lens[:2], False, cfg.act, cfg.ln_eps).reshape(-1, cfg.d_model)
layers = [et.pack_layer(r, cfg.scheme, cfg.ratio, cfg.heads, "fp16") for r in raws]
L = torch.from_numpy(lens).cuda()
for rd in ("fp16", "fp32"):
    enc = et.Encoder(layers, cfg.batch, cfg.seq_len, cfg.heads, cfg.d_ff, ln_eps=cfg.ln_eps, dtype="fp16",
                     resid_dtype=rd, lengths=L, mode="long")
    Xd = torch.from_numpy(X.reshape(cfg.tokens, cfg.d_model)).cuda().to(torch.float16 if rd == "fp16" else torch.float32)
    Y = enc(Xd)
    torch.cuda.synchronize()
    g = Y[: 2 * cfg.seq_len].double().cpu().numpy()
    d = g - ref
    for _ in range(2):
        enc(Xd, Y)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(3):
        enc(Xd, Y)
    torch.cuda.synchronize()
    ms = (time.perf_counter() - t0) / 3 * 1e3
    print(f"resid {rd}: max-abs {np.abs(d).max():.4g} rel-fro {np.linalg.norm(d) / np.linalg.norm(ref):.3g}  "
          f"forward of 4 x 2048 tokens: {ms:.2f} ms")
