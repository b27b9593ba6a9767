"""L2 -> SM pull rate of the GEMM's activation block: unicast vs 4-CTA TMA multicast vs no sharing
(csrc/kernels/tma_probe.cu).  Device time per launch from events; per-CTA cycles to full arrival."""
import ctypes, sys
import numpy as np, torch
sys.path.insert(0, '.')
import paper_conf_sc_chenhplg0d021_b200 as et
import os
f = ctypes.CDLL(os.path.join(os.path.dirname(et.__file__), "libet_diag.so")).et_diag_tma_probe
f.restype = ctypes.c_int
f.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p]
for grid in (128, 148):
    rows = 128 * grid
    X = torch.randn(rows, 768, device='cuda').half()
    cyc = torch.zeros(grid, dtype=torch.int64, device='cuda')
    for mode in (0, 1, 2):
        if mode == 1 and grid % 4:
            continue
        s = torch.cuda.current_stream().cuda_stream
        for _ in range(5):
            assert f(X.data_ptr(), rows, 768, mode, grid, 12, cyc.data_ptr(), s) == 0
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
        e0.record()
        n = 50
        for _ in range(n):
            f(X.data_ptr(), rows, 768, mode, grid, 12, cyc.data_ptr(), s)
        e1.record()
        torch.cuda.synchronize()
        us = e0.elapsed_time(e1) / n * 1e3
        c = cyc.cpu().numpy()
        delivered = grid * 12 * 16384
        print(f"grid {grid} mode {mode}: {us:7.2f} us/launch, delivered {delivered/1e6:.1f} MB -> {delivered/us/1e3:.2f} TB/s; "
              f"cycles to full median {int(np.median(c))} max {int(c.max())}")
