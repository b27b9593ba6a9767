"""A few launches of one C3 tile GEMM (default: the QKV projection) for ncu captures."""
import sys

import torch

sys.path.insert(0, '.')
import paper_conf_sc_chenhplg0d021_b200 as et   # noqa: E402
from et_synth import CONFIGS, make_layer   # noqa: E402

cfg = CONFIGS["C3"]
raw = make_layer(cfg, 0)
lay = et.pack_layer(raw, "tile", 0.8, 12, "fp16")
which = sys.argv[1] if len(sys.argv) > 1 else "w1"
X = torch.randn(4096, 768 if which != "w2" else 3072, device="cuda").half()
epi = {"wq": et.EPI_BIAS_SCALE, "w1": et.EPI_BIAS_GELU, "wo": et.EPI_BIAS, "w2": et.EPI_BIAS}[which]
b = {"wq": "bq", "w1": "b1", "wo": "bo", "w2": "b2"}[which]
for _ in range(5):
    et.linear_fwd(lay.packed[which], X, lay.dense[b], epi)
torch.cuda.synchronize()
print("ok")
