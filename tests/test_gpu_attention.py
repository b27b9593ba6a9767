"""On-the-fly attention core (et_attn_core_fwd) vs the oracle (Eq. 3 with masks):
short and long forms, causal and padding masks, d_k 64 / 128, ragged per-head V widths (row-pruned
W_V), padding invariance (P14, bit-exact) and the FP16 overflow case of §3.3 (P15)."""
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


def _qkv(B, S, H, dk, dtype, seed, qstd=1.5):
    g = np.random.Generator(np.random.PCG64(seed))
    d = H * dk
    Q = to_storage(g.standard_normal((B, S, d), dtype=np.float32) * qstd, dtype)
    K = to_storage(g.standard_normal((B, S, d), dtype=np.float32) * qstd, dtype)
    V = to_storage(g.standard_normal((B, S, d), dtype=np.float32), dtype)
    return Q, K, V


def _lengths(B, S, seed):
    g = np.random.Generator(np.random.PCG64(seed))
    lens = g.integers(max(1, S // 4), S + 1, size=B).astype(np.int32)
    lens[0] = S
    if B > 1:
        lens[1] = 1
    return lens


@pytest.mark.parametrize("S", [16, 100, 128, 200, 256, 384, 512, 777])
@pytest.mark.parametrize("causal", [False, True])
@pytest.mark.parametrize("dk", [64, 128])
def test_attn_core_matches_oracle(etm, S, causal, dk):
    B, H, dtype = 3, 2, "fp16"
    d = H * dk
    Q, K, V = _qkv(B, S, H, dk, dtype, seed=S + dk)
    lens = _lengths(B, S, seed=S)
    qkv = dev_tensor(np.concatenate([Q, K, V], axis=2).reshape(B * S, 3 * d), dtype)
    Z = etm.attn_core_fwd(qkv, B, S, H, d, 0, d, 2 * d, lengths=torch.from_numpy(lens).cuda(), causal=causal,
                          scale=1.0 / math.sqrt(dk))
    torch.cuda.synchronize()
    ref = oe.attention_core(Q, K, V, H, lens, causal).reshape(B * S, d)
    assert_close(to64(Z), ref, max_abs=5e-3, rel_fro=2e-3, what=f"attn S={S} causal={causal} dk={dk}")


@pytest.mark.parametrize("dtype", ["fp16", "bf16"])
def test_short_and_long_forms_agree(etm, dtype):
    B, S, H, dk = 2, 200, 3, 64
    d = H * dk
    Q, K, V = _qkv(B, S, H, dk, dtype, seed=7)
    lens = _lengths(B, S, seed=8)
    qkv = dev_tensor(np.concatenate([Q, K, V], axis=2).reshape(B * S, 3 * d), dtype)
    L = torch.from_numpy(lens).cuda()
    Zs = etm.attn_core_fwd(qkv, B, S, H, d, 0, d, 2 * d, lengths=L, mode="short", scale=0.125)
    Zl = etm.attn_core_fwd(qkv, B, S, H, d, 0, d, 2 * d, lengths=L, mode="long", scale=0.125)
    torch.cuda.synchronize()
    ref = oe.attention_core(Q, K, V, H, lens, False).reshape(B * S, d)
    tol = 5e-3 if dtype == "fp16" else 2e-2
    assert_close(to64(Zs), ref, max_abs=tol, what="short")
    assert_close(to64(Zl), ref, max_abs=tol, what="long")


def test_prescaled_q_reordering(etm):
    """§3.3 (line 159): scaling Q before Q.K^T gives the same attention as scaling the scores."""
    B, S, H, dk = 2, 128, 2, 64
    d = H * dk
    Q0, K, V = _qkv(B, S, H, dk, "fp16", seed=11)
    Qs = to_storage(Q0 / 8.0, "fp16")
    Q = Qs * 8.0                               # exact: 1/sqrt(64) is a power of two
    np.testing.assert_array_equal(to_storage(Q, "fp16"), Q)
    lens = np.full(B, S, np.int32)
    qkv = dev_tensor(np.concatenate([Qs, K, V], axis=2).reshape(B * S, 3 * d), "fp16")
    Z = etm.attn_core_fwd(qkv, B, S, H, d, 0, d, 2 * d, scale=1.0)
    torch.cuda.synchronize()
    ref = oe.attention_core(Q, K, V, H, lens, False).reshape(B * S, d)
    assert_close(to64(Z), ref, max_abs=5e-3, what="prescaled")


def test_fp16_overflow_case_p15(etm):
    """P15: |q.k| up to 65536 > FP16 max; with the scale moved before Q.K^T the FP16 path stays finite."""
    B, S, H, dk = 2, 128, 2, 64
    d = H * dk
    g = np.random.Generator(np.random.PCG64(15))
    Q = (np.where(g.random((B, S, d)) < 0.5, -32.0, 32.0)).astype(np.float32)
    K = (np.where(g.random((B, S, d)) < 0.5, -32.0, 32.0)).astype(np.float32)
    K[:, 0, :] = Q[:, 0, :]                       # some products reach 64 * 32 * 32 = 65536
    V = g.standard_normal((B, S, d), dtype=np.float32).astype(np.float16).astype(np.float32)
    Qs = Q / 8.0                                  # reordered: scale first (exact)
    qkv = dev_tensor(np.concatenate([Qs, K, V], axis=2).reshape(B * S, 3 * d), "fp16")
    Z = etm.attn_core_fwd(qkv, B, S, H, d, 0, d, 2 * d, scale=1.0)
    torch.cuda.synchronize()
    ref = oe.attention_core(Q, K, V, H, np.full(B, S), False).reshape(B * S, d)
    g64 = to64(Z)
    assert np.all(np.isfinite(g64))
    assert_close(g64, ref, what="overflow")


def test_padding_invariance_bitexact(etm):
    """P14: rows of sequence b below len_b do not depend on Q/K/V rows >= len_b (bit-exact)."""
    B, S, H, dk = 3, 160, 2, 64
    d = H * dk
    Q, K, V = _qkv(B, S, H, dk, "fp16", seed=21)
    lens = _lengths(B, S, seed=22)
    L = torch.from_numpy(lens).cuda()
    qkv1 = np.concatenate([Q, K, V], axis=2)
    qkv2 = qkv1.copy()
    for b in range(B):
        qkv2[b, lens[b]:] = to_storage(qkv2[b, lens[b]:] * 3.0 + 1.0, "fp16")
    Z1 = etm.attn_core_fwd(dev_tensor(qkv1.reshape(B * S, 3 * d), "fp16"), B, S, H, d, 0, d, 2 * d, lengths=L,
                           scale=0.125)
    Z2 = etm.attn_core_fwd(dev_tensor(qkv2.reshape(B * S, 3 * d), "fp16"), B, S, H, d, 0, d, 2 * d, lengths=L,
                           scale=0.125)
    torch.cuda.synchronize()
    for b in range(B):
        r = slice(b * S, b * S + int(lens[b]))
        assert torch.equal(Z1[r], Z2[r])


def test_ragged_v_widths_and_scatter(etm):
    """Row-pruned W_V (reading C-5): per-head packed V of widths padded to 16,
    scattered to the original feature columns through z_map."""
    B, S, H, dk = 2, 128, 4, 64
    d = H * dk
    g = np.random.Generator(np.random.PCG64(31))
    kept = [np.sort(g.choice(dk, size=k, replace=False)) + h * dk for h, k in enumerate([10, 32, 0, 49])]
    widths = [(len(k) + 15) // 16 * 16 for k in kept]
    vcol = np.cumsum([0] + widths[:-1]).astype(np.int32)
    vtot = int(sum(widths))
    zmap = -np.ones(vtot, np.int32)
    for h in range(H):
        zmap[vcol[h]:vcol[h] + len(kept[h])] = kept[h]
    Q, K, _ = _qkv(B, S, H, dk, "fp16", seed=32)
    Vp = to_storage(g.standard_normal((B, S, vtot), dtype=np.float32), "fp16")
    for h in range(H):
        Vp[:, :, vcol[h] + len(kept[h]):vcol[h] + widths[h]] = 0.0   # padding rows of W_V give zeros
    lens = _lengths(B, S, seed=33)
    vpad = (vtot + 7) // 8 * 8
    qkv = np.zeros((B, S, 2 * d + vpad), np.float32)
    qkv[:, :, :d], qkv[:, :, d:2 * d], qkv[:, :, 2 * d:2 * d + vtot] = Q, K, Vp
    Z = etm.attn_core_fwd(dev_tensor(qkv.reshape(B * S, -1), "fp16"), B, S, H, d, 0, d, 2 * d,
                          lengths=torch.from_numpy(lens).cuda(), scale=0.125,
                          v_col=torch.from_numpy(vcol).cuda(), v_width=torch.tensor(widths, dtype=torch.int32).cuda(),
                          v_width_max=64, z_map=torch.from_numpy(zmap).cuda())
    torch.cuda.synchronize()
    Vfull = np.zeros((B, S, d), np.float32)
    for h in range(H):
        Vfull[:, :, kept[h]] = Vp[:, :, vcol[h]:vcol[h] + len(kept[h])]
    ref = oe.attention_core(Q, K, Vfull, H, lens, False).reshape(B * S, d)
    g64 = to64(Z)
    keptall = np.concatenate(kept)
    assert_close(g64[:, keptall], ref[:, keptall], max_abs=5e-3, what="ragged V")
    pruned = np.setdiff1d(np.arange(d), keptall)
    assert np.all(g64[:, pruned] == 0.0)       # untouched (pre-zeroed) columns


@pytest.mark.parametrize("generic", [False, True])
@pytest.mark.parametrize("S,causal,dtype", [(128, False, "fp16"), (128, True, "bf16"), (96, False, "fp16"),
                                            (16, True, "fp16"), (1, False, "fp16")])
def test_s128_kernel_and_generic_short_form(etm, generic, S, causal, dtype):
    """seq_len <= 128, d_k = 64 routes to the one-thread-per-row kernel (attention128.cu);
    mode ET_ATTN_SHORT_GENERIC forces the generic short form.  Both match the oracle, ragged lengths
    included, at the north star's bounds for both dtypes (max-abs 2e-2, rel-Frobenius 5e-3) and the
    FP16 kernel also at 5e-3 max-abs."""
    B, H, dk = 5, 3, 64
    d = H * dk
    Q, K, V = _qkv(B, S, H, dk, dtype, seed=90 + S)
    lens = np.minimum(_lengths(B, S, seed=91), S).astype(np.int32)
    qkv = dev_tensor(np.concatenate([Q, K, V], axis=2).reshape(B * S, 3 * d), dtype)
    Z = etm.attn_core_fwd(qkv, B, S, H, d, 0, d, 2 * d, lengths=torch.from_numpy(lens).cuda(), causal=causal,
                          scale=0.125, mode="short_generic" if generic else "short")
    torch.cuda.synchronize()
    ref = oe.attention_core(Q, K, V, H, lens, causal).reshape(B * S, d)
    tol = 5e-3 if dtype == "fp16" else 2e-2
    assert_close(to64(Z), ref, max_abs=tol, rel_fro=2e-3 if dtype == "fp16" else 5e-3, what=f"S={S} generic={generic}")
