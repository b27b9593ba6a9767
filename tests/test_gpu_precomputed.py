"""Pre-computed linear transformation operator (et_precompute_vo + et_attention_pre_fwd; PAPER.md
line 115-131, §3.1 Eq. 5, Fig. 3(b)) vs the float64 oracle's Eq. 5 form
(oracle/variants.py precomputed_attn, pinned to the standard form by P10) on the pattern the paper
pairs with it (line 107, 317: W_Q / W_K tile, W_O row, W_V dense): the kept W_O rows bit-exact,
W_VO within one 16-bit rounding, and the block output at the north star's bar (max-abs 2e-2,
rel-Frobenius 5e-3) — d_k 64 / 128, ragged and causal masks, one and two 256-column VO chunks, a
tail batch smaller than one TMA box, FP16 and BF16."""
import numpy as np
import pytest
import torch

from et_synth import CONFIGS, make_layer, make_lengths, make_x, to_storage
from oracle import encoder as oe
from oracle import variants as ov
from oracle.prune import prune
from tests.gpu_util import assert_close, dev_tensor, to64

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def etm():
    import paper_conf_sc_chenhplg0d021_b200 as m
    assert torch.cuda.is_available()
    return m


def _case(d, heads, S, B, ratio, dtype, causal=False, seed=0):
    cfg = CONFIGS["C2"].with_(d_model=d, heads=heads, seq_len=S, batch=B, ratio=ratio, dtype=dtype, causal=causal,
                              d_ff=4 * d, layers=1)
    raw = make_layer(cfg, seed)
    X = make_x(cfg, seed=1000 + seed)
    lens = make_lengths(cfg, seed=3000 + seed)
    return cfg, raw, X, lens


def _oracle_weights(raw, ratio):
    """Fig. 3(b) pattern (line 107, 317): W_Q / W_K tile, W_O row, W_V dense."""
    w = {k: np.asarray(v, np.float64) for k, v in raw.items()}
    w["wq"] = prune(raw["wq"], "tile", ratio)["W_pruned"]
    w["wk"] = prune(raw["wk"], "tile", ratio)["W_pruned"]
    rec_o = prune(raw["wo"], "row", ratio)
    w["wo"] = rec_o["W_pruned"]
    return w, rec_o


CASES = [
    # d, H, S, B, ratio, dtype, causal
    (768, 12, 128, 4, 0.8, "fp16", False),     # BERT-base shape (DistilBERT of Fig. 9)
    (512, 8, 100, 3, 0.8, "fp16", True),       # Transformer shape, ragged tail, causal
    (768, 6, 128, 2, 0.8, "fp16", False),      # d_k = 128
    (768, 12, 64, 3, 0.5, "bf16", False),      # 50 %: Dv = 384 -> two VO chunks
    (1024, 8, 128, 2, 0.8, "fp16", False),     # d_k = 128, Dv = 208
    (512, 8, 8, 1, 0.8, "fp16", False),        # 8 tokens: smaller than one TMA box
]


@pytest.mark.parametrize("d,H,S,B,ratio,dtype,causal", CASES)
def test_precomputed_block_matches_oracle(etm, d, H, S, B, ratio, dtype, causal):
    cfg, raw, X, lens = _case(d, H, S, B, ratio, dtype, causal)
    layer = etm.PreLayer(raw, ratio, H, dtype)
    w, rec_o = _oracle_weights(raw, ratio)
    # kept W_O rows (ROW mask, bit-exact) and the offline product W_VO (one 16-bit rounding of an
    # FP32 sum of d_k exact products)
    kept = layer.kept.cpu().numpy()
    np.testing.assert_array_equal(kept, np.nonzero(rec_o["keep"])[0])
    dk = d // H
    got_vo = to64(layer.wvo_dense).reshape(H, layer.Dv, d)
    ulp = 2.0 ** -10 if dtype == "fp16" else 2.0 ** -7
    for h in range(H):
        sl = slice(h * dk, (h + 1) * dk)
        exact = (w["wv"][sl, :].T @ w["wo"][:, sl].T).T[kept]          # [n_kept, d]
        g = got_vo[h, :len(kept)]
        assert np.all(np.abs(g - exact) <= ulp * np.abs(exact) + 1e-6), f"W_VO head {h}"
        assert np.all(got_vo[h, len(kept):] == 0.0)
    L = torch.from_numpy(lens).cuda()
    Xd = dev_tensor(X.reshape(cfg.tokens, d), dtype)
    attn = layer(Xd, B, S, lengths=L, causal=causal, ln=False)
    out = layer(Xd, B, S, lengths=L, causal=causal, ln=True, ln_eps=cfg.ln_eps)
    torch.cuda.synchronize()
    X64 = X.astype(np.float64)
    ref_attn = ov.precomputed_attn(X64, w, H, lens, causal)
    ref = oe.layer_norm(X64 + ref_attn, w["ln1_g"], w["ln1_b"], cfg.ln_eps)
    assert_close(to64(attn), ref_attn.reshape(-1, d), max_abs=2e-2, rel_fro=5e-3, what="pre attn")
    assert_close(to64(out), ref.reshape(-1, d), max_abs=2e-2, rel_fro=5e-3, what="pre block")


def test_precomputed_equals_standard_block(etm):
    """Line 131: the pre-computed operator "yields the same results as the original design" —
    the GPU Eq. 5 form against the oracle's standard form (Eq. 3-4) on the same pruned weights."""
    d, H, S, B, ratio = 768, 12, 128, 3, 0.8
    cfg, raw, X, lens = _case(d, H, S, B, ratio, "fp16", seed=5)
    layer = etm.PreLayer(raw, ratio, H, "fp16")
    w, _ = _oracle_weights(raw, ratio)
    X64 = X.astype(np.float64)
    std = oe.attention_block(X64, w, H, lens, False)
    out = layer(dev_tensor(X.reshape(cfg.tokens, d), "fp16"), B, S, lengths=torch.from_numpy(lens).cuda(), ln=False)
    torch.cuda.synchronize()
    assert_close(to64(out), std.reshape(-1, d), max_abs=2e-2, rel_fro=5e-3, what="Eq. 5 vs Eq. 3-4")


def test_precomputed_graph_capture_deterministic(etm):
    """Same inputs, same bits: eager call vs CUDA-graph replay (head groups reduce in a fixed order)."""
    d, H, S, B, ratio = 512, 8, 128, 6, 0.8
    cfg, raw, X, lens = _case(d, H, S, B, ratio, "fp16", seed=9)
    layer = etm.PreLayer(raw, ratio, H, "fp16")
    L = torch.from_numpy(lens).cuda()
    Xd = dev_tensor(X.reshape(cfg.tokens, d), "fp16")
    ws = torch.empty(layer.workspace_size(B, S), dtype=torch.uint8, device="cuda")
    out1 = layer(Xd, B, S, lengths=L, workspace=ws)
    out2 = torch.empty_like(out1)
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    g = torch.cuda.CUDAGraph()
    with torch.cuda.stream(s):
        layer(Xd, B, S, lengths=L, workspace=ws, out=out2, stream=s)   # warm-up on the capture stream
        with torch.cuda.graph(g, stream=s):
            layer(Xd, B, S, lengths=L, workspace=ws, out=out2, stream=s)
    torch.cuda.current_stream().wait_stream(s)
    out2.zero_()
    g.replay()
    torch.cuda.synchronize()
    assert torch.equal(out1, out2)


def test_precomputed_rejects_long_sequences(etm):
    d, H, S, B = 512, 8, 256, 1
    cfg, raw, X, lens = _case(d, H, S, B, 0.8, "fp16")
    layer = etm.PreLayer(raw, 0.8, H, "fp16")
    with pytest.raises(RuntimeError, match="seq_len <= 128"):
        layer(dev_tensor(X.reshape(cfg.tokens, d), "fp16"), B, S)


@pytest.mark.parametrize("d,H,scheme", [(1024, 8, "attention-aware"), (2048, 16, "tile"), (1024, 16, "tile")])
def test_wide_d_model_attention_block(etm, d, H, scheme):
    """d_model > 768 (Fig. 9's 1024 / 2048): the QKV projection's K exceeds one 768-column TMEM part,
    so it runs as FP32 split-K planes + the reduce epilogue (bias, Q-scale); the O-projection's planes
    go to LayerNorm.  Standard form (Eq. 3-4) against the oracle."""
    S, B, ratio = 128, 2, 0.8
    cfg, raw, X, lens = _case(d, H, S, B, ratio, "fp16", seed=11)
    cfg = cfg.with_(scheme=scheme)
    layer = etm.pack_layer(raw, scheme, ratio, H, "fp16")
    out = etm.attention_fwd(dev_tensor(X.reshape(cfg.tokens, d), "fp16"), layer, B, S, H,
                            lengths=torch.from_numpy(lens).cuda(), ln_eps=cfg.ln_eps)
    torch.cuda.synchronize()
    w, _ = oe.prune_layer(raw, scheme, ratio)
    X64 = X.astype(np.float64)
    ref = oe.layer_norm(X64 + oe.attention_block(X64, w, H, lens, False), w["ln1_g"], w["ln1_b"], cfg.ln_eps)
    assert_close(to64(out), ref.reshape(-1, d), max_abs=2e-2, rel_fro=5e-3, what=f"d={d}")


def test_wide_d_model_encoder_layer(etm):
    """One encoder layer at d_model = 1024 (FFN1's K = 1024 through the split-K reduce with GELU)."""
    d, H, S, B, ratio = 1024, 16, 128, 2, 0.8
    cfg, raw, X, lens = _case(d, H, S, B, ratio, "fp16", seed=13)
    cfg = cfg.with_(scheme="tile", act="gelu")
    layer = etm.pack_layer(raw, "tile", ratio, H, "fp16")
    L = torch.from_numpy(lens).cuda()
    enc = etm.Encoder([layer], B, S, H, cfg.d_ff, act="gelu", ln_eps=cfg.ln_eps, dtype="fp16", lengths=L)
    Y = enc(dev_tensor(X.reshape(cfg.tokens, d), "fp16"))
    torch.cuda.synchronize()
    w, _ = oe.prune_layer(raw, "tile", ratio)
    ref = oe.encoder(X.astype(np.float64), [w], H, lens, False, "gelu", cfg.ln_eps)
    assert_close(to64(Y), ref.reshape(-1, d), max_abs=2e-2, rel_fro=5e-3, what="encoder d=1024")
