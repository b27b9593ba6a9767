"""Cycle timeline (clock64, SM cycles) of CTA (0,0,0) of single GEMM launches on C3 layer-0 shapes
(debug build with -DET_TIMELINE).  Slots: see the ET_TIMELINE comment in csrc/kernels/tsgemm.cu."""
import os, sys, numpy as np, torch
sys.path.insert(0, '.')
os.environ.setdefault("ET_LIB_PATH", "build/et_dbg/libet_dbg.so")
import ctypes
import paper_conf_sc_chenhplg0d021_b200 as et
from et_synth import CONFIGS, make_layer
cfg = CONFIGS["C3"]
raw = make_layer(cfg, 0)
lay = et.pack_layer(raw, "tile", 0.8, 12, "fp16")
M = int(sys.argv[1]) if len(sys.argv) > 1 else 4096
X = torch.randn(M, 768, device='cuda').half()
U = torch.randn(M, 3072, device='cuda').half()
buf = (ctypes.c_ulonglong * 512)()
for name, w, x, epi, b in [("wq", "wq", X, et.EPI_BIAS_SCALE, "bq"), ("ffn1", "w1", X, et.EPI_BIAS_GELU, "b1"),
                           ("oproj", "wo", X, et.EPI_F32, None), ("ffn2", "w2", U, et.EPI_F32, None)]:
    for rep in range(3):
        et.linear_fwd(lay.packed[w], x, lay.dense[b] if b else None, epi)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    e0.record()
    et.linear_fwd(lay.packed[w], x, lay.dense[b] if b else None, epi)
    e1.record()
    torch.cuda.synchronize()
    print(f"   one launch (events): {e0.elapsed_time(e1) * 1e3:.2f} us")
    et._lib.et_diag_gemm_timeline(buf)
    t = np.array(buf, dtype=np.int64)
    t0 = t[0]
    rel = lambda i: int(t[i] - t0) if t[i] >= t0 and t[i] - t0 < 10**7 else -1
    t[t == np.iinfo(np.int64).min] = -1
    spans = (ctypes.c_ulonglong * (2048 * 3))()
    et._lib.et_diag_gemm_cta_spans(spans)
    sp = np.array(spans, dtype=np.int64).reshape(2048, 3)
    ncta = {"wq": 0, "ffn1": 0, "oproj": 0, "ffn2": 0}
    sp = sp[(sp[:, 1] > sp[:, 0]) & (sp[:, 0] > 0)]
    sp = sp[sp[:, 0] >= sp[:, 0].max() - 10**6] if len(sp) else sp   # this launch only
    if len(sp):
        s0 = sp[:, 0].min()
        st, en, dur = (sp[:, 0] - s0) / 1e3, (sp[:, 1] - s0) / 1e3, (sp[:, 1] - sp[:, 0]) / 1e3
        print(f"   CTAs {len(sp)} on {len(set(sp[:, 2]))} SMs: start us min/med/max {st.min():.2f}/{np.median(st):.2f}/{st.max():.2f};"
              f" end {en.min():.2f}/{np.median(en):.2f}/{en.max():.2f}; duration {dur.min():.2f}/{np.median(dur):.2f}/{dur.max():.2f}")
    print(f"== {name}: end {rel(500)} cyc, staged {rel(1)}, A chunks " + " ".join(str(rel(2 + j)) for j in range(12))
          + f" | tiles issued {rel(14)}")
    print("  tile chunk first seen: " + " ".join(str(rel(400 + c)) for c in range(12)) +
          " | A chunk seen by w0: " + " ".join(str(rel(450 + j)) for j in range(12)))
    for w in range(8):
        print(f"  mma w{w}: " + " ".join(f"[{rel(16+24*w+3*k)},{rel(17+24*w+3*k)},{rel(18+24*w+3*k)}]" for k in range(6)))
    for g in range(4):
        print(f"  epi g{g}: " + " ".join("[" + ",".join(str(rel(208 + 40 * g + 5 * k + i)) for i in range(4)) + "]"
                                       for k in range(6)))
    print("  w0/w1 next row prepared (rounds 0-7): " + " ".join(str(rel(370 + i)) for i in range(16)))
    print("  g0 quarters 1-3 drained (rounds 0-3): " + " ".join(str(rel(386 + i)) for i in range(12)))
