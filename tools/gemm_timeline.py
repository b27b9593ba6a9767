"""Timeline of CTA (0,0,0) of each GEMM of one C3 layer (debug build with -DET_TIMELINE)."""
import ctypes, sys, numpy as np, torch
sys.path.insert(0, '.')
import os
os.environ.setdefault("ET_LIB_PATH", "build/et_dbg/libet_dbg.so")
import paper_conf_sc_chenhplg0d021_b200 as et
from et_synth import CONFIGS, make_layer, make_x
cfg = CONFIGS["C3"]
raw = make_layer(cfg, 0)
lay = et.pack_layer(raw, "tile", 0.8, 12, "fp16")
M = 4096
X = torch.randn(M, 768, device='cuda').half()
U = torch.randn(M, 3072, device='cuda').half()
buf = (ctypes.c_ulonglong * 512)()
for name, w, x, epi in [("ffn1", "w1", X, et.EPI_BIAS_GELU), ("oproj", "wo", X, et.EPI_F32), ("ffn2", "w2", U, et.EPI_F32)]:
    for rep in range(2):
        et.linear_fwd(lay.packed[w], x, lay.dense["b1"] if w == "w1" else None, epi)
    torch.cuda.synchronize()
    et._lib.et_diag_gemm_timeline(buf)
    t = np.array(buf, dtype=np.float64)
    t0 = t[0]
    rel = lambda i: (t[i] - t0) / 1e3 if t[i] >= t0 else float('nan')
    print(f"== {name}: end {rel(255):.2f} us, staged {rel(1):.2f}, A chunks " + " ".join(f"{rel(2+j):.1f}" for j in range(12)) + f" | tiles issued {rel(14):.2f}")
    for w in range(8):
        print(f"  mma w{w}: " + " ".join(f"[{rel(16+8*w+2*k):.1f},{rel(16+8*w+2*k+1):.1f}]" for k in range(4)))
    print("  w0 round1 MMA issues: " + " ".join(f"{rel(300+i):.2f}" for i in range(24)) + f" | acc_full seen {rel(330):.2f}")
    print("  epi quads: " + " ".join(f"{r}:{rel(96+2*r):.1f}/{rel(97+2*r):.1f}" for r in range(0, 48, 4)))
