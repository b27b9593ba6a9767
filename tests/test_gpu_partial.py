"""Paper-literal partial OTF attention (et_attn_partial_fwd; §3.2, Fig. 8)
vs the oracle (Eq. 3 with masks, line 70-73): kernel A's materialised 16-bit scores against Q.K^T,
kernel B's Z against oracle.attention_core, ragged lengths, causal, d_k 64 / 128, several 128-row
query blocks plus a ragged tail, the fused forms agreeing with it, and the argument checks.

Tolerance (reading C-23): the scores are stored in 16 bit (the paper's pure FP16,
line 157-159) — one extra rounding of every logit (relative 2^-11 FP16, 2^-8 BF16) on top of the
fused forms' P rounding: |logit| up to ~10 here, so a logit moves by up to 5e-3 (FP16) and P by up
to 0.5 %, i.e. Z by up to ~2e-2 against |V| <= 4 in the worst case.  FP16 is held to max-abs 1e-2
(inside the north star's 2e-2) and the fused forms' rel-Frobenius 2e-3; BF16 (2^-8 logits) to
max-abs 3e-2, rel-Frobenius 1.5e-2."""
import math

import numpy as np
import pytest
import torch

from et_synth import to_storage
from oracle import encoder as oe
from tests.gpu_util import assert_close, dev_tensor, to64

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def etm():
    import paper_conf_sc_chenhplg0d021_b200 as m
    assert torch.cuda.is_available()
    return m


def _inputs(B, S, H, dk, dtype, seed):
    g = np.random.Generator(np.random.PCG64(seed))
    d = H * dk
    # Q pre-scaled by 1/sqrt(d_k) (the reordering of line 159): scores of O(1-10)
    Q = to_storage(g.standard_normal((B, S, d), dtype=np.float32) * (1.5 / math.sqrt(dk)), dtype)
    K = to_storage(g.standard_normal((B, S, d), dtype=np.float32) * 1.5, dtype)
    V = to_storage(g.standard_normal((B, S, d), dtype=np.float32), dtype)
    lens = g.integers(max(1, S // 4), S + 1, size=B).astype(np.int32)
    lens[0] = S
    if B > 1:
        lens[1] = 1
    return Q, K, V, lens


def _tol(dtype):
    return dict(max_abs=1e-2, rel_fro=2e-3) if dtype == "fp16" else dict(max_abs=3e-2, rel_fro=1.5e-2)


@pytest.mark.parametrize("S", [8, 64, 200, 256, 392, 512, 776])
@pytest.mark.parametrize("causal", [False, True])
@pytest.mark.parametrize("dk", [64, 128])
def test_partial_matches_oracle(etm, S, causal, dk):
    B, H, dtype = 3, 2, "fp16"
    d = H * dk
    Q, K, V, lens = _inputs(B, S, H, dk, dtype, seed=S * 3 + dk + causal)
    qkv = dev_tensor(np.concatenate([Q, K, V], axis=2).reshape(B * S, 3 * d), dtype)
    Z, _ = etm.attn_partial_fwd(qkv, B, S, H, d, 0, d, 2 * d, lengths=torch.from_numpy(lens).cuda(), causal=causal)
    torch.cuda.synchronize()
    ref = oe.attention_core(Q, K, V, H, lens, causal, dk=1).reshape(B * S, d)
    assert_close(to64(Z), ref, **_tol(dtype), what=f"partial S={S} causal={causal} dk={dk}")


@pytest.mark.parametrize("dtype", ["fp16", "bf16"])
def test_partial_scores_are_rounded_qkt(etm, dtype):
    """Kernel A alone: every stored score of a block kernel B reads is Q_h K_h^T rounded once to the
    16-bit dtype (FP32 tensor-core accumulation of 16-bit products: within one 16-bit ulp of the
    exact product)."""
    B, S, H, dk = 2, 264, 3, 64
    d = H * dk
    Q, K, V, lens = _inputs(B, S, H, dk, dtype, seed=5)
    qkv = dev_tensor(np.concatenate([Q, K, V], axis=2).reshape(B * S, 3 * d), dtype)
    nb = etm.attn_partial_scores_bytes(B, S, H, d, dtype)
    ld = (S + 7) // 8 * 8
    assert nb == B * H * S * ld * 2
    scores = torch.full((nb // 2,), float("nan"), dtype=qkv.dtype, device="cuda")
    etm.attn_partial_fwd(qkv, B, S, H, d, 0, d, 2 * d, lengths=torch.from_numpy(lens).cuda(), scores=scores)
    torch.cuda.synchronize()
    got = scores.view(B, H, S, ld)[..., :S].float().cpu().numpy().astype(np.float64)
    ulp = 2.0 ** -10 if dtype == "fp16" else 2.0 ** -7
    for b in range(B):
        kend = (int(lens[b]) + 127) // 128 * 128          # key blocks kernel A writes
        kend = min(kend, S)
        for h in range(H):
            sl = slice(h * dk, (h + 1) * dk)
            exact = Q[b][:, sl].astype(np.float64) @ K[b][:, sl].astype(np.float64).T
            g = got[b, h][:, :kend]
            e = exact[:, :kend]
            assert np.all(np.isfinite(g))
            assert np.all(np.abs(g - e) <= ulp * np.maximum(np.abs(e), 2.0 ** -14) + 1e-6), f"b={b} h={h}"


@pytest.mark.parametrize("dtype", ["fp16", "bf16"])
def test_partial_agrees_with_fused_forms(etm, dtype):
    """Same attention through the partial OTF and the fused long form (line 145 vs 147)."""
    B, S, H, dk = 2, 392, 3, 64
    d = H * dk
    Q, K, V, lens = _inputs(B, S, H, dk, dtype, seed=17)
    qkv = dev_tensor(np.concatenate([Q, K, V], axis=2).reshape(B * S, 3 * d), dtype)
    L = torch.from_numpy(lens).cuda()
    Zp, _ = etm.attn_partial_fwd(qkv, B, S, H, d, 0, d, 2 * d, lengths=L)
    Zl = etm.attn_core_fwd(qkv, B, S, H, d, 0, d, 2 * d, lengths=L, mode="long", scale=1.0)
    torch.cuda.synchronize()
    ref = oe.attention_core(Q, K, V, H, lens, False, dk=1).reshape(B * S, d)
    assert_close(to64(Zp), ref, **_tol(dtype), what="partial")
    # both are within _tol of the oracle: they agree within twice that
    assert_close(to64(Zp), to64(Zl), **{k: 2 * v for k, v in _tol(dtype).items()}, what="partial vs long")


def test_partial_head_range_and_bf16_causal(etm):
    """Head range [1, 3) of 4 heads (Z columns of the range only) and BF16 causal at a ragged tail."""
    B, S, H, dk = 2, 136, 4, 64
    d = H * dk
    Q, K, V, lens = _inputs(B, S, H, dk, "bf16", seed=23)
    qkv = dev_tensor(np.concatenate([Q, K, V], axis=2).reshape(B * S, 3 * d), "bf16")
    L = torch.from_numpy(lens).cuda()
    import ctypes
    desc = etm.attn_desc(B, S, H, d, "bf16", L, True, head_begin=1, head_end=3)
    Z = torch.zeros(B * S, 2 * dk, dtype=torch.bfloat16, device="cuda")
    nb = etm.attn_partial_scores_bytes(B, S, H, d, "bf16", head_begin=1, head_end=3)
    scores = torch.empty(nb // 2, dtype=torch.bfloat16, device="cuda")
    etm._check(etm._partial(ctypes.byref(desc), qkv.data_ptr(), qkv.stride(0), 0, d, 2 * d, 1.0, Z.data_ptr(),
                            Z.stride(0), scores.data_ptr(), nb, None))
    torch.cuda.synchronize()
    ref = oe.attention_core(Q, K, V, H, lens, True, dk=1).reshape(B * S, d)
    assert_close(to64(Z), ref[:, dk:3 * dk], **_tol("bf16"), what="head range")


def test_partial_padding_invariance_bitexact(etm):
    """P14 for the partial form: rows below len_b ignore Q/K/V rows >= len_b (bit-exact)."""
    B, S, H, dk = 3, 200, 2, 64
    d = H * dk
    Q, K, V, lens = _inputs(B, S, H, dk, "fp16", seed=29)
    L = torch.from_numpy(lens).cuda()
    x1 = np.concatenate([Q, K, V], axis=2)
    x2 = x1.copy()
    for b in range(B):
        x2[b, lens[b]:] = to_storage(x2[b, lens[b]:] * 3.0 + 1.0, "fp16")
    Z1, _ = etm.attn_partial_fwd(dev_tensor(x1.reshape(B * S, 3 * d), "fp16"), B, S, H, d, 0, d, 2 * d, lengths=L)
    Z2, _ = etm.attn_partial_fwd(dev_tensor(x2.reshape(B * S, 3 * d), "fp16"), B, S, H, d, 0, d, 2 * d, lengths=L)
    torch.cuda.synchronize()
    for b in range(B):
        r = slice(b * S, b * S + int(lens[b]))
        assert torch.equal(Z1[r], Z2[r])


def test_partial_argument_errors(etm):
    B, S, H, dk = 1, 100, 2, 64       # S % 8 != 0
    d = H * dk
    qkv = torch.zeros(B * S, 3 * d, dtype=torch.float16, device="cuda")
    with pytest.raises(RuntimeError, match="multiple of 8"):
        etm.attn_partial_fwd(qkv, B, S, H, d, 0, d, 2 * d)
    S = 128
    qkv = torch.zeros(B * S, 3 * d, dtype=torch.float16, device="cuda")
    small = torch.empty(16, dtype=torch.float16, device="cuda")
    with pytest.raises(RuntimeError, match="score buffer"):
        etm.attn_partial_fwd(qkv, B, S, H, d, 0, d, 2 * d, scores=small)
