"""Column pruning with X_adjusted (§4.1, Fig. 5(b)) on the GPU:
et_gather_cols is a bit-exact gather; the column-pruned linear layer (kept-column selection by
et_prune_pack(ET_PRUNE_COL), condensed weight, X_adjusted gather, tcgen05 tile GEMM) matches the
oracle's X . W'^T + b with W' = W with the pruned columns zeroed."""
import numpy as np
import pytest
import torch

from et_synth import make_matrix
from oracle import encoder as oe
from oracle import prune as op
from tests.gpu_util import assert_close, dev_tensor, to64

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def etm():
    import paper_conf_sc_chenhplg0d021_b200 as m
    assert torch.cuda.is_available()
    return m


@pytest.mark.parametrize("dtype", ["fp16", "bf16", "fp32"])
@pytest.mark.parametrize("nk,nk_pad", [(0, 8), (1, 8), (154, 192), (768, 768)])
def test_gather_cols_bit_exact(etm, dtype, nk, nk_pad):
    rows, cols = 300, 768
    A = dev_tensor(make_matrix(40, (rows, cols), 1.0, dtype), dtype)
    rng = np.random.default_rng(41)
    idx = np.sort(rng.choice(cols, nk, replace=False)).astype(np.int32)
    out = etm.gather_cols(A, torch.from_numpy(idx).cuda(), nk_pad)
    torch.cuda.synchronize()
    ref = np.zeros((rows, nk_pad), np.float32)
    ref[:, :nk] = A.float().cpu().numpy()[:, idx]
    np.testing.assert_array_equal(out.float().cpu().numpy(), ref)


def test_gather_cols_rejects_bad_pad(etm):
    A = torch.zeros(4, 64, dtype=torch.float16, device="cuda")
    idx = torch.arange(10, dtype=torch.int32, device="cuda")
    with pytest.raises(etm.EtError):
        etm.gather_cols(A, idx, 12)    # nk_pad not a multiple of 8


@pytest.mark.parametrize("dtype", ["fp16", "bf16"])
@pytest.mark.parametrize("M", [128, 300, 4096])
@pytest.mark.parametrize("ratio", [0.0, 0.5, 0.8, 0.95])
def test_col_linear_matches_oracle(etm, dtype, M, ratio):
    d = 768
    Wnp = make_matrix(42, (d, d), 0.05, dtype)
    b = make_matrix(43, (d,), 0.02, dtype)
    X = make_matrix(44, (M, d), 1.0, dtype)
    cl = etm.ColLinear(dev_tensor(Wnp, dtype), ratio)
    ref_sel = op.prune_col(Wnp, ratio)
    np.testing.assert_array_equal(cl.keep.cpu().numpy(), ref_sel["idx"])     # selection bit-exact
    assert cl.nk == ref_sel["nnz"] and cl.nk_pad % 64 == 0
    Y = cl(dev_tensor(X, dtype), dev_tensor(b, dtype))
    torch.cuda.synchronize()
    ref = oe.linear(X, ref_sel["W_pruned"], b)
    g = to64(Y)
    assert_close(g, ref, what=f"col linear {dtype} M={M} r={ratio}")
    eps = 2.0 ** -11 if dtype == "fp16" else 2.0 ** -8   # fp32 accumulation + one output rounding
    assert np.all(np.abs(g - ref) <= eps * np.abs(ref) * 1.01 + 1e-4)


def test_col_linear_ffn_shape_gelu(etm):
    # FFN1 shape (3072 x 768) with the GELU epilogue, K condensed to 154 -> 192
    dtype, M = "fp16", 512
    Wnp = make_matrix(45, (3072, 768), 0.05, dtype)
    b = make_matrix(46, (3072,), 0.02, dtype)
    X = make_matrix(47, (M, 768), 1.0, dtype)
    cl = etm.ColLinear(dev_tensor(Wnp, dtype), 0.8)
    assert cl.nk == 154 and cl.nk_pad == 192
    Y = cl(dev_tensor(X, dtype), dev_tensor(b, dtype), etm.EPI_BIAS_GELU)
    torch.cuda.synchronize()
    ref = oe.gelu(oe.linear(X, op.prune_col(Wnp, 0.8)["W_pruned"], b))
    assert_close(to64(Y), ref, what="col linear gelu")


def test_col_linear_fully_pruned_is_bias(etm):
    # degenerate case: every column pruned -> X_adjusted is all padding, Y = b exactly
    dtype, M, d = "fp16", 256, 768
    Wnp = make_matrix(48, (d, d), 0.05, dtype)
    b = make_matrix(49, (d,), 0.02, dtype)
    X = make_matrix(50, (M, d), 1.0, dtype)
    cl = etm.ColLinear(dev_tensor(Wnp, dtype), 1.0)
    assert cl.nk == 0 and cl.nk_pad == 64
    Y = cl(dev_tensor(X, dtype), dev_tensor(b, dtype))
    torch.cuda.synchronize()
    np.testing.assert_array_equal(to64(Y), np.broadcast_to(b.astype(np.float64), (M, d)))
