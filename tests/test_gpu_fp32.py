"""FP32 validation build (BASELINE.json configs[0]: C1 in FP32; north_star: "1e-5 for an FP32
validation build") vs the float64 oracle: packing (bit-exact), the tile-sparse linear layer with
every epilogue and split-K, the attention core (masks, causal, long rows), the attention-aware
block and the C1 encoder.  Error measure: relative Frobenius error AND
max-abs / max(1, max|ref|), both <= 1e-5."""
import math

import numpy as np
import pytest
import torch

from et_synth import CONFIGS, make_layer, make_lengths, make_matrix, make_x
from oracle import encoder as oe
from oracle import prune as op
from tests.gpu_util import dev_tensor, errors, to64

pytestmark = pytest.mark.gpu
TOL32 = 1e-5


@pytest.fixture(scope="module")
def etm():
    import paper_conf_sc_chenhplg0d021_b200 as m
    assert torch.cuda.is_available()
    return m


def assert_close32(gpu, ref, what=""):
    assert np.all(np.isfinite(gpu)), f"{what}: non-finite values"
    ma, rf = errors(gpu, ref)
    scale = max(1.0, float(np.abs(ref).max()))
    assert ma / scale <= TOL32 and rf <= TOL32, f"{what}: max-abs {ma:.3e} (scaled {ma / scale:.3e}), rel-fro {rf:.3e}"


@pytest.mark.parametrize("pattern", ["tile", "row"])
def test_fp32_pack_bit_exact(etm, pattern):
    W = make_matrix(40, (256, 192), 0.02, "fp32")
    pk = etm.prune_pack(dev_tensor(W, "fp32"), pattern, 0.7, group_rows=64 if pattern == "row" else 0)
    torch.cuda.synchronize()
    rec = op.prune(W, pattern, 0.7)
    nw = rec["mask"].size                                              # (the buffer is padded to 16 B)
    assert np.array_equal(pk.mask().cpu().numpy().view(np.uint32)[:nw], rec["mask"])
    assert np.array_equal(to64(etm.unpack(pk)), rec["W_pruned"])       # FP32 values moved, not rounded


@pytest.mark.parametrize("M", [16, 100, 300])
@pytest.mark.parametrize("epi", ["bias", "scale", "gelu", "relu"])
def test_fp32_linear(etm, M, epi):
    d, N = 192, 320
    W = make_matrix(41, (N, d), 0.05, "fp32")
    b = make_matrix(42, (N,), 0.02, "fp32")
    X = make_matrix(43, (M, d), 1.0, "fp32")
    pk = etm.prune_pack(dev_tensor(W, "fp32"), "tile", 0.5)
    code = {"bias": etm.EPI_BIAS, "scale": etm.EPI_BIAS_SCALE, "gelu": etm.EPI_BIAS_GELU,
            "relu": etm.EPI_BIAS_RELU}[epi]
    s = 1.0 / math.sqrt(64)
    Y = etm.linear_fwd(pk, dev_tensor(X, "fp32"), dev_tensor(b, "fp32"), code, scale=s, scale_cols=64)
    torch.cuda.synchronize()
    ref = oe.linear(X, op.prune_tile(W, 0.5)["W_pruned"], b)
    if epi == "scale":
        ref[:, :64] *= s
    elif epi == "gelu":
        ref = oe.gelu(ref)
    elif epi == "relu":
        ref = oe.relu(ref)
    assert_close32(to64(Y), ref, what=f"fp32 linear {epi} M={M}")


def test_fp32_linear_split_k(etm):
    M, d, N = 200, 1536, 256             # K = 1536: two K parts -> two FP32 partial planes
    W = make_matrix(44, (N, d), 0.02, "fp32")
    X = make_matrix(45, (M, d), 1.0, "fp32")
    pk = etm.prune_pack(dev_tensor(W, "fp32"), "tile", 0.8)
    P = etm.linear_fwd(pk, dev_tensor(X, "fp32"), None, etm.EPI_F32)
    torch.cuda.synchronize()
    assert P.shape[0] == 2
    ref = oe.linear(X, op.prune_tile(W, 0.8)["W_pruned"], None)
    assert_close32(to64(P).sum(0), ref, what="fp32 split-K")


@pytest.mark.parametrize("S,causal,dk", [(16, False, 64), (16, True, 64), (130, False, 128), (600, True, 64)])
def test_fp32_attention_core(etm, S, causal, dk):
    B, H = 3, 2
    d = H * dk
    g = np.random.Generator(np.random.PCG64(S + dk))
    Q, K, V = (g.standard_normal((B, S, d), dtype=np.float32) * s for s in (1.5, 1.5, 1.0))
    lens = g.integers(max(1, S // 4), S + 1, size=B).astype(np.int32)
    lens[0], lens[1] = S, 1
    qkv = dev_tensor(np.concatenate([Q, K, V], axis=2).reshape(B * S, 3 * d), "fp32")
    Z = etm.attn_core_fwd(qkv, B, S, H, d, 0, d, 2 * d, lengths=torch.from_numpy(lens).cuda(), causal=causal,
                          scale=1.0 / math.sqrt(dk))
    torch.cuda.synchronize()
    ref = oe.attention_core(Q, K, V, H, lens, causal).reshape(B * S, d)
    assert_close32(to64(Z), ref, what=f"fp32 attention S={S} causal={causal} dk={dk}")


@pytest.mark.parametrize("key,kw", [
    ("C1", {}),                                          # configs[0]: the FP32 validation config
    ("C1", {"batch": 3, "seq_len": 40}),
    ("C2", {"dtype": "fp32", "d_model": 256, "heads": 2, "d_ff": 1024, "seq_len": 64}),   # attention-aware, causal
])
def test_fp32_encoder_matches_oracle(etm, key, kw):
    cfg = CONFIGS[key].with_(**kw)
    assert cfg.dtype == "fp32"
    raws = [make_layer(cfg, l) for l in range(cfg.layers)]
    X = make_x(cfg)
    lens = make_lengths(cfg)
    layers = [etm.pack_layer(r, cfg.scheme, cfg.ratio, cfg.heads, "fp32") for r in raws]
    enc = etm.Encoder(layers, cfg.batch, cfg.seq_len, cfg.heads, cfg.d_ff, act=cfg.act, ln_eps=cfg.ln_eps,
                      dtype="fp32", resid_dtype="fp32", causal=cfg.causal, lengths=torch.from_numpy(lens).cuda())
    Y = enc(dev_tensor(X.reshape(cfg.tokens, cfg.d_model), "fp32"))
    torch.cuda.synchronize()
    ref = oe.encoder(X.astype(np.float64), [oe.prune_layer(r, cfg.scheme, cfg.ratio)[0] for r in raws], cfg.heads,
                     lens, cfg.causal, cfg.act, cfg.ln_eps).reshape(cfg.tokens, cfg.d_model)
    assert_close32(to64(Y), ref, what=f"fp32 encoder {key} {kw}")
