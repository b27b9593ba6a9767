import sys, time, numpy as np, torch
sys.path.insert(0, '.')
import paper_conf_sc_chenhplg0d021_b200 as et
from et_synth import CONFIGS, make_layer, make_lengths, make_x
cfg = CONFIGS["C3"]
raws = [make_layer(cfg, l) for l in range(cfg.layers)]
layers = [et.pack_layer(r, cfg.scheme, cfg.ratio, cfg.heads, "fp16") for r in raws]
enc = et.Encoder(layers, cfg.batch, cfg.seq_len, cfg.heads, cfg.d_ff, lengths=torch.full((32,), 128, dtype=torch.int32, device='cuda'))
Xd = torch.from_numpy(make_x(cfg).reshape(cfg.tokens, cfg.d_model)).cuda().half(); out = torch.empty_like(Xd)
for _ in range(5): enc(Xd, out)
torch.cuda.synchronize()
t0 = time.perf_counter()
for _ in range(20): enc(Xd, out)
t1 = time.perf_counter(); torch.cuda.synchronize(); t2 = time.perf_counter()
print(f"host per call {1e3*(t1-t0)/20:.3f} ms, total per call {1e3*(t2-t0)/20:.3f} ms")
# CUDA graph
g = torch.cuda.CUDAGraph()
s = torch.cuda.Stream()
s.wait_stream(torch.cuda.current_stream())
with torch.cuda.stream(s):
    enc(Xd, out)
torch.cuda.synchronize()
with torch.cuda.graph(g):
    enc(Xd, out)
for _ in range(3): g.replay()
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(20): g.replay()
e1.record(); torch.cuda.synchronize()
print(f"graph replay per step {e0.elapsed_time(e1)/20:.3f} ms")
