import ctypes, os, sys, numpy as np, torch
sys.path.insert(0, '.')
os.environ.setdefault("ET_LIB_PATH", "build/et_dbg/libet_dbg.so")
import paper_conf_sc_chenhplg0d021_b200 as et
et._sig("et_diag_attn_timeline", ctypes.c_int, [et._vp])
B, S, H, d = [int(a) for a in sys.argv[1:5]] if len(sys.argv) >= 5 else (32, 128, 12, 768)
causal = len(sys.argv) >= 6 and sys.argv[5] == 'causal'
qkv = torch.randn(B * S, 3 * d, device='cuda').half()
buf = (ctypes.c_ulonglong * 64)()
for _ in range(3):
    et.attn_core_fwd(qkv, B, S, H, d, 0, d, 2 * d, scale=(d // H) ** -0.5, causal=causal, mode='short')
torch.cuda.synchronize()
et._lib.et_diag_attn_timeline(buf)
t = np.array(buf, dtype=np.float64); t0 = t[0]
names = ["start", "tmem+sync", "Q loaded (mma warp)", "QK issued", "P ready (mma)", "S ready (softmax)", "P written", "O ready", "epilogue done", "end"]
for i, n in enumerate(names): print(f"{n:22s} {(t[i]-t0)/1e3:8.2f} us")
