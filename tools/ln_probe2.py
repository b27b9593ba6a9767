"""LN1-form timing vs rows (warm L2, graph replays): is the LayerNorm kernel bound by a fixed
per-launch latency or by throughput?  usage: python tools/ln_probe2.py"""
import json, sys
import torch
sys.path.insert(0, '.')
import paper_conf_sc_chenhplg0d021_b200 as et
from tools.sweeps import timed

N = 768
h = torch.float16
g = torch.ones(N, device='cuda')
b = torch.zeros(N, device='cuda')
bias = torch.zeros(N, device='cuda').to(h)
out = {}
for M in (128, 512, 1024, 2048, 4096, 8192, 16384):
    p1 = torch.randn(1, M, N, device='cuda').to(h)
    p4 = torch.randn(4, M, N, device='cuda').to(h)
    res = torch.randn(M, N, device='cuda').to(h)
    o = torch.empty(M, N, device='cuda', dtype=h)
    out[f"ln1_M{M}"] = round(timed(lambda: et.layernorm_fwd(p1, bias, res, g, b, 1e-12, "fp16", "fp16", out_act=o)), 2)
    out[f"ln2_M{M}"] = round(timed(lambda: et.layernorm_fwd(p4, bias, res, g, b, 1e-12, "fp16", "fp16", out_act=o)), 2)
# an empty-ish kernel for reference: a cast of 16 elements
x = torch.zeros(16, device='cuda')
print(json.dumps(out))
