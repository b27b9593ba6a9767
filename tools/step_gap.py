"""Where does a small config's step time go?  Times one CUDA-graph replay of the encoder (C2 by default)
(a) back to back without an L2 flush, (b) after a 256 MiB flush write (bench.py's discipline), and
(c) the empty-stream event pair, to separate graph launch latency, cold-L2 effects and kernel time.
Usage: python tools/step_gap.py [C2|C3|...]"""
import json, sys, os
import numpy as np
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_chenhplg0d021_b200 as et  # noqa: E402
from et_synth import CONFIGS, make_layer, make_lengths, make_x  # noqa: E402

cfg = CONFIGS[sys.argv[1] if len(sys.argv) > 1 else "C2"]
raws = [make_layer(cfg, l) for l in range(cfg.layers)]
layers = [et.pack_layer(r, cfg.scheme, cfg.ratio, cfg.heads, cfg.dtype) for r in raws]
L = torch.from_numpy(make_lengths(cfg, ragged=False)).cuda()
enc = et.Encoder(layers, cfg.batch, cfg.seq_len, cfg.heads, cfg.d_ff, act=cfg.act, ln_eps=cfg.ln_eps,
                 dtype=cfg.dtype, resid_dtype=cfg.dtype, causal=cfg.causal, mode=cfg.attn_mode, lengths=L)
X = torch.from_numpy(make_x(cfg).reshape(cfg.tokens, cfg.d_model)).cuda().half()
out = torch.empty_like(X)
for _ in range(3):
    enc(X, out)
g = enc.capture(X, out)
flush = torch.empty(64 * 1024 * 1024, dtype=torch.float32, device="cuda")
s = torch.cuda.current_stream()


def run(n, pre=None, body=True):
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(n)]
    for i in range(n):
        if pre:
            pre(i)
        ev[i][0].record(s)
        if body:
            g.launch()
        ev[i][1].record(s)
    torch.cuda.synchronize()
    return float(np.median([a.elapsed_time(b) * 1e3 for a, b in ev]))


for _ in range(5):
    g.launch()
torch.cuda.synchronize()
res = {"config": cfg.name if hasattr(cfg, "name") else sys.argv[1:],
       "empty_events_us": run(50, body=False),
       "warm_back_to_back_us": run(50),
       "after_flush_us": run(50, pre=lambda i: flush.fill_(float(i))),
       "after_flush_then_sleep_us": run(20, pre=lambda i: (flush.fill_(float(i)), torch.cuda._sleep(200000)))}
# eager (no graph) for comparison
ev0, ev1 = torch.cuda.Event(True), torch.cuda.Event(True)
ev0.record(s)
for _ in range(20):
    enc(X, out)
ev1.record(s)
torch.cuda.synchronize()
res["eager_us"] = ev0.elapsed_time(ev1) * 1e3 / 20
print(json.dumps(res))
