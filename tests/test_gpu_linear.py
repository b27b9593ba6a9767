"""Tile-sparse linear layer (et_linear_fwd) vs the oracle: X . W'^T + b with every epilogue,
ragged M, split-K, pruned-tile independence (P5) and fully-pruned tile rows (P6)."""
import math

import numpy as np
import pytest
import torch

from et_synth import CONFIGS, make_layer, make_matrix
from oracle import prune as op
from oracle import encoder as oe
from tests.gpu_util import assert_close, dev_tensor, to64

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def etm():
    import paper_conf_sc_chenhplg0d021_b200 as m
    assert torch.cuda.is_available()
    return m


def _rounding_bound(ref, dtype):
    # fp32 accumulation + one rounding to the 16-bit output: |err| <= ulp/2 of |y| (+ tiny slack)
    eps = 2.0 ** -11 if dtype == "fp16" else 2.0 ** -8
    return eps * np.abs(ref) * 1.01 + 1e-4


@pytest.mark.parametrize("dtype", ["fp16", "bf16"])
@pytest.mark.parametrize("M", [128, 300, 4096])
@pytest.mark.parametrize("ratio", [0.0, 0.8, 0.95])
def test_linear_bias_matches_oracle(etm, dtype, M, ratio):
    d = 768
    Wnp = make_matrix(10, (3 * d, d), 0.05, dtype)
    b = make_matrix(11, (3 * d,), 0.02, dtype)
    X = make_matrix(12, (M, d), 1.0, dtype)
    pk = etm.prune_pack(dev_tensor(Wnp, dtype), "tile", ratio)
    Y = etm.linear_fwd(pk, dev_tensor(X, dtype), dev_tensor(b, dtype), etm.EPI_BIAS)
    torch.cuda.synchronize()
    ref = oe.linear(X, op.prune_tile(Wnp, ratio)["W_pruned"], b)
    g = to64(Y)
    assert_close(g, ref, what=f"linear {dtype} M={M} r={ratio}")
    assert np.all(np.abs(g - ref) <= _rounding_bound(ref, dtype))


@pytest.mark.parametrize("epi", ["scale", "gelu", "relu"])
def test_linear_epilogues(etm, epi):
    dtype, M, d = "fp16", 512, 768
    N = 3072 if epi != "scale" else 3 * d
    Wnp = make_matrix(20, (N, d), 0.05, dtype)
    b = make_matrix(21, (N,), 0.02, dtype)
    X = make_matrix(22, (M, d), 1.0, dtype)
    pk = etm.prune_pack(dev_tensor(Wnp, dtype), "tile", 0.8)
    code = {"scale": etm.EPI_BIAS_SCALE, "gelu": etm.EPI_BIAS_GELU, "relu": etm.EPI_BIAS_RELU}[epi]
    s = 1.0 / math.sqrt(64)
    Y = etm.linear_fwd(pk, dev_tensor(X, dtype), dev_tensor(b, dtype), code, scale=s, scale_cols=d)
    torch.cuda.synchronize()
    ref = oe.linear(X, op.prune_tile(Wnp, 0.8)["W_pruned"], b)
    if epi == "scale":
        ref[:, :d] *= s                     # the Q columns, scaled before Q.K^T
    elif epi == "gelu":
        ref = oe.gelu(ref)
    else:
        ref = oe.relu(ref)
    g = to64(Y)
    assert_close(g, ref, what=epi)
    assert np.all(np.abs(g - ref) <= _rounding_bound(ref, dtype) + 1e-5)


@pytest.mark.parametrize("K", [768, 3072])
def test_linear_fp32_partials_split_k(etm, K):
    dtype, M = "fp16", 384
    N = 768
    Wnp = make_matrix(30, (N, K), 0.02, dtype)
    X = make_matrix(31, (M, K), 1.0, dtype)
    pk = etm.prune_pack(dev_tensor(Wnp, dtype), "tile", 0.8)
    P = etm.linear_fwd(pk, dev_tensor(X, dtype), None, etm.EPI_F32)
    torch.cuda.synchronize()
    assert P.shape[0] == K // 768
    ref = oe.linear(X, op.prune_tile(Wnp, 0.8)["W_pruned"], None)
    g = P.double().sum(0).cpu().numpy()
    assert np.abs(g - ref).max() <= 1e-5 * max(1.0, np.abs(ref).max())


@pytest.mark.parametrize("K,M", [(768, 384), (3072, 300)])
def test_linear_fp16_partials_split_k(etm, K, M):
    """ET_EPI_PART16: each split-K plane is the FP32 accumulator rounded once to FP16; the planes sum
    to X . W'^T within the per-plane rounding bound (the FP16 path's O-proj / FFN2 partial sums)."""
    dtype, N = "fp16", 768
    Wnp = make_matrix(32, (N, K), 0.02, dtype)
    X = make_matrix(33, (M, K), 1.0, dtype)
    pk = etm.prune_pack(dev_tensor(Wnp, dtype), "tile", 0.8)
    P = etm.linear_fwd(pk, dev_tensor(X, dtype), None, etm.EPI_PART16)
    torch.cuda.synchronize()
    assert P.dtype == torch.float16 and P.shape == (K // 768, M, N)
    Wp = op.prune_tile(Wnp, 0.8)["W_pruned"]
    g = P.double().cpu().numpy()
    for z in range(K // 768):   # each plane: its K part's exact product, rounded to fp16 once
        ref = oe.linear(X[:, z * 768:(z + 1) * 768], Wp[:, z * 768:(z + 1) * 768], None)
        assert np.all(np.abs(g[z] - ref) <= _rounding_bound(ref, dtype) + 1e-5)


def test_pruned_tile_values_do_not_matter_bitexact(etm):
    """P5: same mask, different values inside pruned tiles => bit-identical output."""
    dtype, M, d = "fp16", 256, 768
    Wnp = make_matrix(40, (d, d), 0.05, dtype)
    ref = op.prune_tile(Wnp, 0.8)
    mask_in = torch.from_numpy(ref["mask"].view(np.int32)).cuda()
    W2 = Wnp.copy()
    for i in range(48):
        for j in range(48):
            if not ref["tile_mask"][i, j]:
                W2[i * 16:(i + 1) * 16, j * 16:(j + 1) * 16] = 1.5
    X = dev_tensor(make_matrix(41, (M, d), 1.0, dtype), dtype)
    b = dev_tensor(make_matrix(42, (d,), 0.02, dtype), dtype)
    Y1 = etm.linear_fwd(etm.prune_pack(dev_tensor(Wnp, dtype), "tile", 0.8, mask_in=mask_in), X, b)
    Y2 = etm.linear_fwd(etm.prune_pack(dev_tensor(W2, dtype), "tile", 0.8, mask_in=mask_in), X, b)
    torch.cuda.synchronize()
    assert torch.equal(Y1, Y2)


def test_fully_pruned_tile_row_is_bias_exactly(etm):
    """P6: an output tile row with no kept tile equals the bias bit-exactly."""
    dtype, M, d = "fp16", 256, 256
    Wnp = make_matrix(50, (d, d), 0.05, dtype)
    tm = np.ones((16, 16), bool)
    tm[3, :] = False
    tm[7, :] = False
    mask_in = torch.from_numpy(op.bitmap(tm).view(np.int32)).cuda()
    pk = etm.prune_pack(dev_tensor(Wnp, dtype), "tile", 0.0, mask_in=mask_in)
    b = make_matrix(51, (d,), 0.5, dtype)
    Y = etm.linear_fwd(pk, dev_tensor(make_matrix(52, (M, d), 1.0, dtype), dtype), dev_tensor(b, dtype))
    torch.cuda.synchronize()
    g = Y.float().cpu().numpy()
    for r in (3, 7):
        np.testing.assert_array_equal(g[:, r * 16:(r + 1) * 16], np.broadcast_to(b[r * 16:(r + 1) * 16], (M, 16)))


def test_row_pruned_condensed_linear(etm):
    """Row pruning (Fig. 5(a)): X . W_condensed^T through the packed, per-head
    padded layout; padded rows produce the bias of nothing (zero weights)."""
    cfg = CONFIGS["C2"]
    dtype = "fp16"
    Wnp = make_layer(cfg, 0)["wv"]
    X = make_matrix(60, (256, cfg.d_model), 1.0, dtype)
    pk = etm.prune_pack(dev_tensor(Wnp, dtype), "row", cfg.ratio, group_rows=cfg.d_k)
    Y = etm.linear_fwd(pk, dev_tensor(X, dtype), None, etm.EPI_BIAS)
    torch.cuda.synchronize()
    rmap = pk.bufs["row_map"][:pk.rows_padded].cpu().numpy()
    ref_full = oe.linear(X, op.prune_row(Wnp, cfg.ratio)["W_pruned"], None)
    g = to64(Y)
    for pr, orow in enumerate(rmap):
        if orow >= 0:
            np.testing.assert_allclose(g[:, pr], ref_full[:, orow], rtol=2 ** -10, atol=1e-4)
        else:
            assert np.all(g[:, pr] == 0.0)
