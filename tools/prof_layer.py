"""Run the C3 encoder (bench launch configuration, all lengths = S) `--calls` times; used as the
target of ncu captures (tools/profile_round.sh).  Launch order per call: 12 x [qkv GEMM, attention,
O GEMM, LN1, FFN1 GEMM, FFN2 GEMM, LN2]."""
import argparse, sys
import torch
sys.path.insert(0, '.')
import paper_conf_sc_chenhplg0d021_b200 as et
from et_synth import CONFIGS, make_layer, make_x

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C3")
ap.add_argument("--calls", type=int, default=2)
a = ap.parse_args()
cfg = CONFIGS[a.config]
raws = [make_layer(cfg, l) for l in range(cfg.layers)]
layers = [et.pack_layer(r, cfg.scheme, cfg.ratio, cfg.heads, cfg.dtype) for r in raws]
L = torch.full((cfg.batch,), cfg.seq_len, dtype=torch.int32, device="cuda")
enc = et.Encoder(layers, cfg.batch, cfg.seq_len, cfg.heads, cfg.d_ff, act=cfg.act, ln_eps=cfg.ln_eps,
                 dtype=cfg.dtype, resid_dtype=cfg.dtype, causal=cfg.causal, mode=cfg.attn_mode, lengths=L)
X = torch.from_numpy(make_x(cfg).reshape(cfg.tokens, cfg.d_model)).cuda().to(
    torch.float16 if cfg.dtype == "fp16" else torch.bfloat16)
out = torch.empty_like(X)
for _ in range(a.calls):
    enc(X, out)
torch.cuda.synchronize()
print("prof_layer done", a.config, a.calls)
