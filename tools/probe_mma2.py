"""M1b microbenchmark driver (round 2): single-warp issue rate of N=16 TS MMAs over many
independent accumulators, tcgen05.cp vs register-path TMEM fill, and the K-outer streaming
pattern (diag/mma_probe2.cu).  Exactness is checked on CTA 0's TMEM contents.
Writes gpurun_out/probe_mma2.json."""
import ctypes
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
lib = ctypes.CDLL(os.path.join(ROOT, "paper_conf_sc_chenhplg0d021_b200", "libet_diag.so"))
lib.et_diag_mma_probe2.argtypes = [ctypes.c_void_p] * 3 + [ctypes.c_int] * 6 + [ctypes.c_void_p, ctypes.c_int,
                                                                             ctypes.c_void_p]
dev = torch.device("cuda")
g = np.random.default_rng(0)
A = g.integers(-2, 3, size=(128, 64)).astype(np.float64)
B = g.integers(-2, 3, size=(16, 16)).astype(np.float64)
tA = torch.tensor(A, dtype=torch.float16, device=dev)
tB = torch.tensor(B, dtype=torch.float16, device=dev)
P = [A[:, 16 * s:16 * s + 16] @ B.T for s in range(4)]   # one MMA with A sub-tile s
res = []


def run(mode, nw=1, n_acc=16, n_mma=0, n_chunks=0, mpc=0, grid=148):
    D = torch.zeros(128, 512, dtype=torch.float32, device=dev)
    cyc = torch.zeros(grid, dtype=torch.int64, device=dev)
    rc = lib.et_diag_mma_probe2(tA.data_ptr(), tB.data_ptr(), D.data_ptr(), mode, nw, n_acc, n_mma, n_chunks, mpc,
                                cyc.data_ptr(), grid, torch.cuda.current_stream().cuda_stream)
    torch.cuda.synchronize()
    Dh = D.cpu().numpy().astype(np.float64)
    exp = np.zeros((128, 512))
    if mode in (4, 5):
        exp = None
        err = 0.0
        nm = nw * n_mma
    elif mode == 0:
        for w in range(nw):
            accs = list(range(w, n_acc, nw))
            ai = 0
            for u in range(0, n_mma - n_mma % 4, 4):
                for i in range(4):
                    a = accs[ai]
                    exp[:, 16 * a:16 * a + 16] += P[i]
                    ai = (ai + 1) % len(accs)
        exp[:, 384:416] = Dh[:, 384:416]   # A slot (not checked)
        err = float(np.abs(Dh[:, :384] - exp[:, :384]).max())
        nm = nw * n_mma
    elif mode == 2:
        ai = 0
        for c in range(n_chunks):
            for u in range(0, mpc, 4):
                for i in range(4):
                    exp[:, 16 * ai:16 * ai + 16] += P[i]
                    ai = (ai + 1) % n_acc
        err = float(np.abs(Dh[:, :384] - exp[:, :384]).max())
        nm = n_chunks * mpc
    else:   # A ring holds the chunk (packed 16-bit pairs) in every slot that was written
        a16 = torch.tensor(A, dtype=torch.float16).numpy().view(np.uint16).astype(np.uint32)
        packed = (a16[:, 0::2] | (a16[:, 1::2] << 16)).view(np.float32).astype(np.float64)
        err = max(float(np.abs(Dh[:, 384 + 32 * s:416 + 32 * s] - packed).max()) for s in range(min(4, n_chunks)))
        nm = 0
    c = float(cyc.float().median())
    row = dict(mode=mode, nw=nw, n_acc=n_acc, n_mma=nm, n_chunks=n_chunks, mpc=mpc, rc=rc, max_err=err,
               cycles=c, cycles_per_mma=round(c / nm, 2) if nm else None,
               bytes_per_cycle=round(n_chunks * 16384 / c, 1) if mode in (1, 3) else None)
    res.append(row)
    print(json.dumps(row), flush=True)


for mode in (4, 5):
    for nw in (1, 2, 4, 8):
        run(mode, nw=nw, n_acc=24, n_mma=256)
if "--only45" in sys.argv:
    sys.exit(0)
for nw in (1, 2, 4):
    for n_acc in (8, 16, 24):
        if n_acc % nw == 0:
            run(0, nw=nw, n_acc=n_acc, n_mma=256 // nw * 4)
for nch in (4, 12, 48):
    run(1, n_chunks=nch)
    run(3, n_chunks=nch)
for mpc in (8, 12, 16, 24, 32):
    run(2, n_acc=24, n_chunks=12, mpc=mpc)
    run(2, n_acc=24, n_chunks=48, mpc=mpc)
os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
with open(os.path.join(ROOT, "gpurun_out", "probe_mma2.json"), "w") as f:
    json.dump(res, f, indent=1)
bad = [r for r in res if r["max_err"] != 0 or r["rc"] != 0]
print("BAD", len(bad))
sys.exit(1 if bad else 0)
