"""LayerNorm timing probe (C3 shapes, M = 4096, N = 768): the LN1 form (1 FP16 partial + bias +
residual) and the LN2 form (4 FP16 partials), timed (a) alone back to back in a CUDA graph (warm
L2), (b) after the producing GEMM (FFN2 -> LN2, O-proj -> LN1) minus the GEMM alone, i.e. the
increment the LN adds inside the pipeline.  usage: python tools/ln_probe.py"""
import json, sys
import torch
sys.path.insert(0, '.')
import paper_conf_sc_chenhplg0d021_b200 as et
from et_synth import CONFIGS, make_layer
from tools.sweeps import timed

cfg = CONFIGS["C3"]
lay = et.pack_layer(make_layer(cfg, 0), "tile", 0.8, 12, "fp16")
M, N = 4096, 768
h = torch.float16
Z = torch.randn(M, N, device='cuda').to(h)
U = torch.randn(M, 3072, device='cuda').to(h) * 0.1
res = torch.randn(M, N, device='cuda').to(h)
g = torch.ones(N, device='cuda')
b = torch.zeros(N, device='cuda')
bias = torch.zeros(N, device='cuda').to(h)
p1 = torch.empty(1, M, N, device='cuda', dtype=h)
p4 = torch.empty(4, M, N, device='cuda', dtype=h)
out = torch.empty(M, N, device='cuda', dtype=h)
ln1 = lambda: et.layernorm_fwd(p1, bias, res, g, b, 1e-12, "fp16", "fp16", out_act=out)
ln2 = lambda: et.layernorm_fwd(p4, bias, res, g, b, 1e-12, "fp16", "fp16", out_act=out)
oproj = lambda: et.linear_fwd(lay.packed["wo"], Z, None, et.EPI_PART16, out=p1.view(M, N))
ffn2 = lambda: et.linear_fwd(lay.packed["w2"], U, None, et.EPI_PART16, out=p4)
r = {}
r["ln1_alone"] = timed(ln1)
r["ln2_alone"] = timed(ln2)
r["oproj"] = timed(oproj)
r["oproj_ln1"] = timed(lambda: (oproj(), ln1()))
r["ffn2"] = timed(ffn2)
r["ffn2_ln2"] = timed(lambda: (ffn2(), ln2()))
r["ln1_in_pipe"] = r["oproj_ln1"] - r["oproj"]
r["ln2_in_pipe"] = r["ffn2_ln2"] - r["ffn2"]
print(json.dumps({k: round(v, 2) for k, v in r.items()}))
