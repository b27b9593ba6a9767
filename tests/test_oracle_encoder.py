"""Pins for oracle/encoder.py (CPU): closed forms, torch float64 library routines at ratio 0,
the paper's own identities (Eq. 4, Eq. 5, scale reordering), scalar brute force and
invariances."""
import math

import numpy as np
import pytest
import torch

from et_synth import CONFIGS, make_layer, make_lengths, make_x
from oracle import encoder as oe
from oracle import variants as ov
from oracle.prune import prune_tile, prune_row


def _small_cfg(**kw):
    base = CONFIGS["C2"].with_(d_model=64, heads=4, d_ff=256, seq_len=16, batch=3, causal=False,
                              act="gelu", ln_eps=1e-12)
    return base.with_(**kw)


def _dense_layer(cfg, layer=0):
    return {k: np.asarray(v, np.float64) for k, v in make_layer(cfg, layer).items()}


# ---------------------------------------------------------------- P3 library cross-check
@pytest.mark.parametrize("causal", [False, True])
def test_ratio0_matches_torch_mha_float64(causal):
    cfg = _small_cfg(causal=causal)
    w = _dense_layer(cfg)
    X = make_x(cfg).astype(np.float64)
    lens = make_lengths(cfg)
    attn = oe.attention_block(X, w, cfg.heads, lens, causal)
    xt = torch.from_numpy(X).transpose(0, 1).contiguous()        # [S, B, d]
    kpm = torch.from_numpy(np.arange(cfg.seq_len)[None, :] >= lens[:, None])
    am = torch.triu(torch.ones(cfg.seq_len, cfg.seq_len, dtype=torch.bool), 1) if causal else None
    out, _ = torch.nn.functional.multi_head_attention_forward(
        xt, xt, xt, cfg.d_model, cfg.heads,
        torch.from_numpy(np.concatenate([w["wq"], w["wk"], w["wv"]])),
        torch.from_numpy(np.concatenate([w["bq"], w["bk"], w["bv"]])),
        None, None, False, 0.0, torch.from_numpy(w["wo"]), torch.from_numpy(w["bo"]),
        training=False, key_padding_mask=kpm, need_weights=False, attn_mask=am)
    ref = out.transpose(0, 1).numpy()
    assert np.abs(attn - ref).max() <= 1e-12


@pytest.mark.parametrize("act", ["gelu", "relu"])
def test_ratio0_matches_torch_encoder_layer_float64(act):
    cfg = _small_cfg(act=act, ln_eps=1e-12 if act == "gelu" else 1e-5)
    w = _dense_layer(cfg)
    X = make_x(cfg).astype(np.float64)
    lens = make_lengths(cfg)
    Y = oe.encoder_layer(X, w, cfg.heads, lens, False, act, cfg.ln_eps)
    layer = torch.nn.TransformerEncoderLayer(cfg.d_model, cfg.heads, cfg.d_ff, dropout=0.0,
                                             activation=act, layer_norm_eps=cfg.ln_eps,
                                             batch_first=True, norm_first=False).double()
    with torch.no_grad():
        layer.self_attn.in_proj_weight.copy_(torch.from_numpy(np.concatenate([w["wq"], w["wk"], w["wv"]])))
        layer.self_attn.in_proj_bias.copy_(torch.from_numpy(np.concatenate([w["bq"], w["bk"], w["bv"]])))
        layer.self_attn.out_proj.weight.copy_(torch.from_numpy(w["wo"]))
        layer.self_attn.out_proj.bias.copy_(torch.from_numpy(w["bo"]))
        layer.linear1.weight.copy_(torch.from_numpy(w["w1"]))
        layer.linear1.bias.copy_(torch.from_numpy(w["b1"]))
        layer.linear2.weight.copy_(torch.from_numpy(w["w2"]))
        layer.linear2.bias.copy_(torch.from_numpy(w["b2"]))
        layer.norm1.weight.copy_(torch.from_numpy(w["ln1_g"]))
        layer.norm1.bias.copy_(torch.from_numpy(w["ln1_b"]))
        layer.norm2.weight.copy_(torch.from_numpy(w["ln2_g"]))
        layer.norm2.bias.copy_(torch.from_numpy(w["ln2_b"]))
    layer.eval()
    kpm = torch.from_numpy(np.arange(cfg.seq_len)[None, :] >= lens[:, None])
    # grad enabled + params requiring grad => torch takes the reference (non fast) path
    ref = layer(torch.from_numpy(X), src_key_padding_mask=kpm).detach().numpy()
    assert np.abs(Y - ref).max() <= 1e-11


# ---------------------------------------------------------------- P1, P2 closed forms
def test_softmax_rows_sum_to_one_and_masked_are_exact_zero():
    cfg = _small_cfg(causal=True)
    w = _dense_layer(cfg)
    X = make_x(cfg).astype(np.float64)
    lens = make_lengths(cfg)
    _, inter = oe.attention_block(X, w, cfg.heads, lens, True, return_all=True)
    P = inter["P"]
    assert np.all(P >= 0)
    assert np.abs(P.sum(-1) - 1).max() <= 1e-14
    for b in range(cfg.batch):
        allowed = oe.key_mask(cfg.seq_len, int(lens[b]), True)
        assert np.all(P[b][:, ~allowed] == 0.0)


@pytest.mark.parametrize("causal", [False, True])
def test_uniform_scores_give_mean_of_v(causal):
    cfg = _small_cfg()
    w = _dense_layer(cfg)
    w["wq"][:] = 0.0
    w["bq"][:] = 0.0                   # Q = 0 => every score 0 => uniform over allowed keys
    X = make_x(cfg).astype(np.float64)
    lens = make_lengths(cfg)
    _, inter = oe.attention_block(X, w, cfg.heads, lens, causal, return_all=True)
    V = inter["V"]
    for b in range(cfg.batch):
        for i in range(cfg.seq_len):
            hi = min(int(lens[b]), i + 1) if causal else int(lens[b])
            np.testing.assert_allclose(inter["Z"][b, i], V[b, :hi].mean(0), rtol=0, atol=1e-15)


def test_fully_pruned_closed_form():
    """P4: ratio 1 => W' = 0 => attn == b_O exactly; Y1 = LN(X + b_O); Y2 = LN(Y1 + b_2)."""
    cfg = _small_cfg()
    raw = make_layer(cfg, 0)
    w, _ = oe.prune_layer(raw, "tile", 1.0)
    X = make_x(cfg).astype(np.float64)
    lens = make_lengths(cfg)
    Y2, inter = oe.encoder_layer(X, w, cfg.heads, lens, False, "gelu", 1e-12, return_all=True)
    np.testing.assert_array_equal(inter["attn"], np.broadcast_to(w["bo"], inter["attn"].shape))
    Y1 = oe.layer_norm(X + w["bo"], w["ln1_g"], w["ln1_b"], 1e-12)
    np.testing.assert_array_equal(inter["Y1"], Y1)
    np.testing.assert_allclose(Y2, oe.layer_norm(Y1 + w["b2"], w["ln2_g"], w["ln2_b"], 1e-12), atol=1e-14)


def test_layer_norm_and_activation_closed_forms():
    v = np.array([[1.0, 2.0, 3.0, 4.0]])
    y = oe.layer_norm(v, np.ones(4), np.zeros(4), 0.0)
    np.testing.assert_allclose(y, (v - 2.5) / math.sqrt(1.25), rtol=1e-15)   # biased variance 1.25
    assert oe.gelu(np.array([0.0]))[0] == 0.0
    np.testing.assert_allclose(oe.gelu(np.array([1.0])), [0.8413447460685429], rtol=1e-15)  # x*Phi(x)
    np.testing.assert_array_equal(oe.relu(np.array([-1.0, 2.0])), [0.0, 2.0])


# ---------------------------------------------------------------- P6 fully pruned tile row
def test_fully_pruned_tile_row_equals_bias_exactly():
    W = make_layer(_small_cfg(), 0)["wq"].astype(np.float64)
    tm = np.ones((4, 4), bool)
    tm[2, :] = False
    rec = prune_tile(W, 0.0, 16, 16, mask_in=tm)
    X = make_x(_small_cfg()).astype(np.float64)
    b = np.arange(64, dtype=float) / 7
    Y = oe.linear(X, rec["W_pruned"], b)
    np.testing.assert_array_equal(Y[..., 32:48], np.broadcast_to(b[32:48], Y[..., 32:48].shape))


# ---------------------------------------------------------------- P8 reorder, P12 per-row OTF
@pytest.mark.parametrize("dk,exact", [(16, True), (64, True), (32, False)])
def test_scale_reorder_identity(dk, exact):
    g = np.random.Generator(np.random.PCG64(dk))
    Q = g.standard_normal((8, dk))
    K = g.standard_normal((8, dk))
    s = 1.0 / math.sqrt(dk)
    a = (s * Q) @ K.T
    b = s * (Q @ K.T)
    if exact:          # 1/sqrt(dk) is a power of two for dk a power of 4
        np.testing.assert_array_equal(a, b)
    else:
        np.testing.assert_allclose(a, b, rtol=1e-15, atol=1e-15)


@pytest.mark.parametrize("causal", [False, True])
def test_otf_rowwise_scale_first_equals_matrix_form(causal):
    cfg = _small_cfg(causal=causal, batch=2)
    w = _dense_layer(cfg)
    X = make_x(cfg).astype(np.float64)
    lens = make_lengths(cfg)
    _, inter = oe.attention_block(X, w, cfg.heads, lens, causal, return_all=True)
    Z2 = ov.otf_rowwise(inter["Q"], inter["K"], inter["V"], cfg.heads, lens, causal)
    np.testing.assert_allclose(inter["Z"], Z2, rtol=0, atol=1e-14)


def test_bruteforce_scalar_layer_c1():
    """P12: configs[0] (C1: 1 head, d=64, S=16, 50% tile pruning) with scalar loops == oracle."""
    cfg = CONFIGS["C1"]
    raw = make_layer(cfg, 0)
    w, _ = oe.prune_layer(raw, cfg.scheme, cfg.ratio)
    X = make_x(cfg).astype(np.float64)
    lens = make_lengths(cfg, ragged=False)
    Y = oe.encoder_layer(X, w, cfg.heads, lens, cfg.causal, cfg.act, cfg.ln_eps)
    Yb = ov.brute_force_layer(X, w, cfg.heads, lens, cfg.causal, cfg.act, cfg.ln_eps)
    assert np.abs(Y - Yb).max() <= 1e-12


def test_bruteforce_scalar_layer_causal_ragged_multihead():
    cfg = _small_cfg(d_model=32, heads=2, d_ff=64, seq_len=8, batch=3, causal=True, act="relu",
                     ln_eps=1e-5)
    raw = make_layer(cfg, 1)
    w, _ = oe.prune_layer(raw, "attention-aware", 0.5)
    X = make_x(cfg).astype(np.float64)
    lens = make_lengths(cfg)
    Y = oe.encoder_layer(X, w, cfg.heads, lens, True, "relu", 1e-5)
    Yb = ov.brute_force_layer(X, w, cfg.heads, lens, True, "relu", 1e-5)
    assert np.abs(Y - Yb).max() <= 1e-12


# ---------------------------------------------------------------- P9, P10, P11 paper identities
def test_eq4_concat_equals_sum_over_heads():
    cfg = _small_cfg()
    w = _dense_layer(cfg)
    X = make_x(cfg).astype(np.float64)
    lens = make_lengths(cfg)
    _, inter = oe.attention_block(X, w, cfg.heads, lens, False, return_all=True)
    Z = inter["Z"]
    dk = cfg.d_k
    s = sum(Z[..., h * dk:(h + 1) * dk] @ w["wo"][:, h * dk:(h + 1) * dk].T for h in range(cfg.heads))
    np.testing.assert_allclose(Z @ w["wo"].T, s, rtol=0, atol=1e-12)


@pytest.mark.parametrize("causal", [False, True])
def test_eq5_precomputed_operator_equals_standard(causal):
    cfg = _small_cfg(causal=causal)
    raw = make_layer(cfg, 0)
    w, _ = oe.prune_layer(raw, "attention-aware", 0.5)
    X = make_x(cfg).astype(np.float64)
    lens = make_lengths(cfg)
    a = oe.attention_block(X, w, cfg.heads, lens, causal)
    b = ov.precomputed_attn(X, w, cfg.heads, lens, causal)
    assert np.abs(a - b).max() <= 1e-12 * max(1.0, np.abs(a).max())


def test_v_bias_fold_under_row_pruning():
    """P11 / reading C-6: a pruned V feature f has V[:, f] = b_V[f], so Z[:, f] = b_V[f]; folding
    W_O[:, f] b_V[f] into b_O is exact in real arithmetic."""
    cfg = _small_cfg()
    raw = make_layer(cfg, 0)
    w = {k: np.asarray(v, np.float64) for k, v in raw.items()}
    rr = prune_row(w["wv"], 0.8)
    w["wv"] = rr["W_pruned"]
    X = make_x(cfg).astype(np.float64)
    lens = make_lengths(cfg)
    a, inter = oe.attention_block(X, w, cfg.heads, lens, False, return_all=True)
    pruned = ~rr["keep"]
    np.testing.assert_allclose(inter["Z"][..., pruned],
                               np.broadcast_to(w["bv"][pruned], inter["Z"][..., pruned].shape),
                               rtol=0, atol=1e-15)
    w2 = dict(w)
    w2["bv"] = np.where(pruned, 0.0, w["bv"])
    w2["bo"] = w["bo"] + w["wo"][:, pruned] @ w["bv"][pruned]
    b = oe.attention_block(X, w2, cfg.heads, lens, False)
    assert np.abs(a - b).max() <= 1e-12


# ---------------------------------------------------------------- P13, P14 invariances
def test_head_permutation_invariance():
    cfg = _small_cfg()
    w = _dense_layer(cfg)
    X = make_x(cfg).astype(np.float64)
    lens = make_lengths(cfg)
    a = oe.attention_block(X, w, cfg.heads, lens, False)
    perm = [2, 0, 3, 1]
    dk = cfg.d_k
    idx = np.concatenate([np.arange(h * dk, (h + 1) * dk) for h in perm])
    w2 = dict(w)
    for k in ("wq", "wk", "wv"):
        w2[k] = w[k][idx]
    for k in ("bq", "bk", "bv"):
        w2[k] = w[k][idx]
    w2["wo"] = w["wo"][:, idx]
    b = oe.attention_block(X, w2, cfg.heads, lens, False)
    assert np.abs(a - b).max() <= 1e-13


def test_token_permutation_equivariance_full_length_noncausal():
    cfg = _small_cfg(batch=1)
    w = _dense_layer(cfg)
    X = make_x(cfg).astype(np.float64)
    lens = np.array([cfg.seq_len])
    Y = oe.encoder_layer(X, w, cfg.heads, lens, False, "gelu", 1e-12)
    perm = np.random.Generator(np.random.PCG64(5)).permutation(cfg.seq_len)
    Yp = oe.encoder_layer(X[:, perm], w, cfg.heads, lens, False, "gelu", 1e-12)
    assert np.abs(Y[:, perm] - Yp).max() <= 1e-12


def test_padding_invariance_bit_exact():
    """P14: valid rows of sequence b do not depend on X[b, j >= len_b]."""
    cfg = _small_cfg()
    w = _dense_layer(cfg)
    X = make_x(cfg).astype(np.float64)
    lens = make_lengths(cfg)
    Y = oe.encoder_layer(X, w, cfg.heads, lens, False, "gelu", 1e-12)
    X2 = X.copy()
    for b in range(cfg.batch):
        X2[b, lens[b]:] *= 100.0
    Y2 = oe.encoder_layer(X2, w, cfg.heads, lens, False, "gelu", 1e-12)
    for b in range(cfg.batch):
        np.testing.assert_array_equal(Y[b, :lens[b]], Y2[b, :lens[b]])


def test_encoder_stack_is_layer_composition():
    cfg = _small_cfg(layers=2)
    layers = [_dense_layer(cfg, l) for l in range(2)]
    X = make_x(cfg).astype(np.float64)
    lens = make_lengths(cfg)
    Y = oe.encoder(X, layers, cfg.heads, lens, False, "gelu", 1e-12)
    Y1 = oe.encoder_layer(X, layers[0], cfg.heads, lens, False, "gelu", 1e-12)
    np.testing.assert_array_equal(Y, oe.encoder_layer(Y1, layers[1], cfg.heads, lens, False, "gelu", 1e-12))
