"""Per-kernel average device time (library trace events) of the C3 encoder, L2 flushed before each
step, for one or more library builds: python tools/kernel_times.py [lib.so ...] (default: in-tree)."""
import ctypes, json, os, subprocess, sys
libs = sys.argv[1:] or [""]
if len(libs) > 1 or os.environ.get("ET_KT_CHILD") is None and libs != [""]:
    # one child process per library (the binding loads its library once)
    for lib in libs:
        env = dict(os.environ, ET_KT_CHILD="1")
        if lib:
            env["ET_LIB_PATH"] = lib
        subprocess.run([sys.executable, __file__], env=env, check=False)
    sys.exit(0)
import numpy as np, torch
sys.path.insert(0, ".")
import paper_conf_sc_chenhplg0d021_b200 as et
from et_synth import CONFIGS, make_layer, make_x
cfg = CONFIGS[os.environ.get("ET_KT_CONFIG", "C3")]
raws = [make_layer(cfg, l) for l in range(cfg.layers)]
layers = [et.pack_layer(r, cfg.scheme, cfg.ratio, cfg.heads, cfg.dtype) for r in raws]
L = torch.full((cfg.batch,), cfg.seq_len, dtype=torch.int32, device="cuda")
enc = et.Encoder(layers, cfg.batch, cfg.seq_len, cfg.heads, cfg.d_ff, act=cfg.act, ln_eps=cfg.ln_eps,
                 dtype=cfg.dtype, resid_dtype=cfg.dtype, causal=cfg.causal, mode=cfg.attn_mode, lengths=L)
X = torch.from_numpy(make_x(cfg).reshape(cfg.tokens, cfg.d_model)).cuda().to(et.torch_dtype(cfg.dtype))
out = torch.empty_like(X)
flush = torch.empty(64 << 20, dtype=torch.float32, device="cuda")
for _ in range(5):
    enc(X, out)
K = 20
ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(K)]
torch.cuda.synchronize()
et._check(et._lib.et_trace_begin(K * (cfg.layers * 8 + 4) + 8))
for s in range(K):
    flush.fill_(float(s))
    ev[s][0].record()
    enc(X, out)
    ev[s][1].record()
n = ctypes.c_int32()
et._check(et._lib.et_trace_end(ctypes.byref(n)))
torch.cuda.synchronize()
names = ["qkv", "attn", "oproj", "ln1", "ffn1", "ffn2", "ln2", "other"]
kind, ms = ctypes.c_int32(), ctypes.c_float()
per = {}
for i in range(n.value):
    et._check(et._lib.et_trace_get(i, ctypes.byref(kind), ctypes.byref(ms)))
    per.setdefault(names[min(kind.value, 7)], []).append(ms.value * 1e3)
step = sorted(a.elapsed_time(b) for a, b in ev)[K // 2]
print(os.environ.get("ET_LIB_PATH", "in-tree"), f"step {step:.3f} ms ({cfg.batch / step * 1e3:.0f} seq/s)",
      " ".join(f"{k} {np.mean(v):.1f}" for k, v in per.items()))
