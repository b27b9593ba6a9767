import sys, subprocess
attn = r'''
import sys, math, numpy as np, torch
sys.path.insert(0, '.')
import paper_conf_sc_chenhplg0d021_b200 as etm
B, S, dk = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3])
H = 2; d = H * dk
g = np.random.default_rng(0)
qkv = torch.tensor(g.standard_normal((B * S, 3 * d)), dtype=torch.float16, device='cuda')
Z = etm.attn_core_fwd(qkv, B, S, H, d, 0, d, 2 * d, mode="short", scale=0.125)
torch.cuda.synchronize(); print("OK")
'''
gemm = r'''
import sys, numpy as np, torch
sys.path.insert(0, '.')
import paper_conf_sc_chenhplg0d021_b200 as etm
M = int(sys.argv[1])
W = torch.randn(256, 256, device='cuda').half(); X = torch.randn(M, 256, device='cuda').half()
pk = etm.prune_pack(W, "tile", 0.5)
Y = etm.linear_fwd(pk, X); torch.cuda.synchronize(); print("OK")
'''
for name, code, args in [("gemm", gemm, ["16"]), ("gemm", gemm, ["100"]), ("attn", attn, ["8", "16", "64"]),
                         ("attn", attn, ["3", "16", "64"]), ("attn", attn, ["1", "128", "64"]), ("attn", attn, ["2", "64", "64"])]:
    try:
        r = subprocess.run([sys.executable, "-c", code] + args, capture_output=True, text=True, timeout=25)
        out = (r.stdout + r.stderr).strip().splitlines()
        print(name, args, "OK" if "OK" in r.stdout else "FAIL " + " | ".join(out[-2:]), flush=True)
    except subprocess.TimeoutExpired:
        print(name, args, "TIMEOUT", flush=True)
