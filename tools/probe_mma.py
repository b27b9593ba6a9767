"""M1 microbenchmark driver: tcgen05.mma at M=128, N in {16..256}, A from SMEM vs TMEM.

Checks each (a_mode, b_mode, N) for exactness against an integer-valued float64 product and
prints cycles per MMA (K=16) at one CTA per SM on all SMs.  Writes gpurun_out/probe_mma.json.
"""
import ctypes
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
lib = ctypes.CDLL(os.path.join(ROOT, "paper_conf_sc_chenhplg0d021_b200", "libet_diag.so"))
lib.et_diag_mma_probe.argtypes = [ctypes.c_void_p] * 3 + [ctypes.c_int] * 6 + [ctypes.c_void_p, ctypes.c_int,
                                                                            ctypes.c_void_p]

dev = torch.device("cuda")
g = np.random.default_rng(0)
A = g.integers(-2, 3, size=(128, 64)).astype(np.float64)
res = []
cases = []
for (N, n_acc, issue_mode) in ((16, 8, 8), (16, 8, 108), (16, 8, 116), (16, 16, 16), (16, 4, 116)):
    cases.append((1, N, 1, n_acc, issue_mode))
for (b_mode, N, a_mode, n_acc, issue_mode) in cases:
    B = g.integers(-2, 3, size=(N, 64)).astype(np.float64)       # logical [N, K]
    for iters in (1, 256):
        grid = 1 if iters == 1 else 148
        Bdev = B.T.copy() if b_mode == 2 else B                # MN-major input is [K, N]
        tA = torch.tensor(A, dtype=torch.float16, device=dev)
        tB = torch.tensor(Bdev, dtype=torch.float16, device=dev).contiguous()
        D = torch.zeros(128, N * n_acc, dtype=torch.float32, device=dev)
        cyc = torch.zeros(grid + 1, dtype=torch.int64, device=dev)
        rc = lib.et_diag_mma_probe(tA.data_ptr(), tB.data_ptr(), D.data_ptr(), N, a_mode, b_mode, iters, n_acc, issue_mode,
                                   cyc.data_ptr(), grid, torch.cuda.current_stream().cuda_stream)
        torch.cuda.synchronize()
        mult = ((issue_mode - 100) // n_acc) if issue_mode >= 100 else 1
        ref = np.tile(mult * iters * (A @ B.T), (1, n_acc))
        err = float(np.abs(D.cpu().numpy().astype(np.float64) - ref).max())
        cpm = float(cyc[:grid].float().median()) / (iters * 4 * n_acc)
        row = dict(cp_cycles=int(cyc[grid]), issue=issue_mode, a_mode=("ss", "ts", "ts_cp")[a_mode], b_mode=("k_sw128", "k_tile_none", "mn_sw128")[b_mode],
                   N=N, n_acc=n_acc, iters=iters, rc=rc, max_err=err, cycles_per_mma=round(cpm, 2),
                   floor=128 * N / 256, frac_of_peak=round(128 * N / 256 / cpm, 3))
        res.append(row)
        if True:
            print(json.dumps(row), flush=True)
os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
with open(os.path.join(ROOT, "gpurun_out", "probe_mma.json"), "w") as f:
    json.dump(res, f, indent=1)
bad = [r for r in res if r["max_err"] != 0 or r["rc"] != 0]
print("BAD", len(bad))
sys.exit(1 if bad else 0)
