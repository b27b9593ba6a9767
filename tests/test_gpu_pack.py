"""et_prune_pack on the GPU vs the oracle: masks, CSR indices and kept-row indices BIT-EXACT;
unpacked values == W' bit-exactly (SURVEY §4 tier T1)."""
import json
import os

import numpy as np
import pytest
import torch

from et_synth import CONFIGS, make_layer, make_matrix
from oracle import prune as op
from tests.gpu_util import dev_tensor

pytestmark = pytest.mark.gpu



@pytest.fixture(scope="module")
def etm():
    import paper_conf_sc_chenhplg0d021_b200 as m
    assert torch.cuda.is_available(), "gpu tests need a CUDA device"
    return m


def _check_tile(etm, Wnp, dtype, ratio, tile=16):
    W = dev_tensor(Wnp, dtype)
    pk = etm.prune_pack(W, "tile", ratio, (tile, tile))
    ref = op.prune_tile(Wnp.astype(np.float64), ratio, tile, tile)
    T = (Wnp.shape[0] // tile) * (Wnp.shape[1] // tile)
    words = (T + 31) // 32
    np.testing.assert_array_equal(pk.mask()[:words].cpu().numpy().view(np.uint32), ref["mask"])
    rp, ci = pk.csr()
    np.testing.assert_array_equal(rp.cpu().numpy(), ref["row_ptr"])
    np.testing.assert_array_equal(ci.cpu().numpy(), ref["col_idx"])
    assert pk.nnz == ref["nnz"]
    if tile == 16 and dtype != "fp32":
        dense = etm.unpack(pk).float().cpu().numpy().astype(np.float64)
        np.testing.assert_array_equal(dense, ref["W_pruned"])
    return pk


@pytest.mark.parametrize("ratio", [0.0, 0.5, 0.8, 0.95, 1.0])
@pytest.mark.parametrize("dtype", ["fp16", "bf16"])
def test_tile_pack_bitexact_bert_matrices(etm, ratio, dtype):
    cfg = CONFIGS["C3"]
    w = make_layer(cfg, 0, dtype)
    for name in ("wq", "w1", "w2"):
        _check_tile(etm, w[name], dtype, ratio)


def test_tile_pack_all_configs(etm):
    for key in ("C1", "C2", "C4"):
        cfg = CONFIGS[key]
        w = make_layer(cfg, 0)
        for name in ("wq", "wo", "w1", "w2"):
            _check_tile(etm, w[name], cfg.dtype, cfg.ratio)


def test_fig6_fixture_on_gpu(etm, golden_dir):
    with open(os.path.join(golden_dir, "fig6_tile_prune_handworked.json")) as f:
        g = json.load(f)
    W = np.array(g["W"], dtype=np.float32)
    for case in g["cases"]:
        pk = etm.prune_pack(dev_tensor(W, "fp32"), "tile", case["ratio"], tuple(g["tile"]))
        assert pk.mask()[:1].cpu().numpy().view(np.uint32)[0] == case["bitmap"][0]
        rp, ci = pk.csr()
        assert rp.cpu().tolist() == case["row_ptr"]
        assert ci.cpu().tolist() == case["col_idx"]


def test_ties_all_zero_and_duplicates(etm):
    W = np.zeros((64, 64), np.float32)
    pk = _check_tile(etm, W, "fp16", 0.5)
    assert pk.mask()[:1].cpu().numpy().view(np.uint32)[0] == 0xFF00
    W = np.zeros((32, 32), np.float32)
    blk = (np.arange(256, dtype=np.float32).reshape(16, 16) / 100).astype(np.float16).astype(np.float32)
    for i in range(2):
        for j in range(2):
            W[i * 16:(i + 1) * 16, j * 16:(j + 1) * 16] = blk
    for r in (0.25, 0.5, 0.75):
        _check_tile(etm, W, "fp16", r)


@pytest.mark.parametrize("dtype", ["fp16", "bf16"])
def test_row_pack_bitexact_attention_aware(etm, dtype):
    for key in ("C2", "C4"):
        cfg = CONFIGS[key]
        Wnp = make_layer(cfg, 0, dtype)["wv"]
        pk = etm.prune_pack(dev_tensor(Wnp, dtype), "row", cfg.ratio, (16, 16), group_rows=cfg.d_k)
        ref = op.prune_row(Wnp.astype(np.float64), cfg.ratio)
        words = (Wnp.shape[0] + 31) // 32
        np.testing.assert_array_equal(pk.mask()[:words].cpu().numpy().view(np.uint32), ref["mask"])
        np.testing.assert_array_equal(pk.kept_index().cpu().numpy(), ref["idx"])
        # per-head padding of the packed rows (layout only): each head padded to a multiple of 16
        kept = ref["keep"].reshape(cfg.heads, cfg.d_k).sum(1)
        assert pk.rows_padded == int(sum((k + 15) // 16 * 16 for k in kept))
        dense = etm.unpack(pk).float().cpu().numpy().astype(np.float64)
        np.testing.assert_array_equal(dense, ref["W_pruned"])


def test_col_pattern_mask_and_index(etm):
    Wnp = make_matrix(77, (64, 96), 0.02, "fp16")
    pk = etm.prune_pack(dev_tensor(Wnp, "fp16"), "col", 0.5, (16, 16))
    ref = op.prune_col(Wnp.astype(np.float64), 0.5)
    np.testing.assert_array_equal(pk.kept_index().cpu().numpy(), ref["idx"])


def test_mask_in_fixes_the_kept_set(etm):
    Wnp = make_matrix(3, (128, 128), 0.02, "fp16")
    ref = op.prune_tile(Wnp.astype(np.float64), 0.7, 16, 16)
    mask_in = torch.from_numpy(ref["mask"].view(np.int32)).cuda()
    W2 = Wnp.copy()
    for i in range(8):
        for j in range(8):
            if not ref["tile_mask"][i, j]:
                W2[i * 16:(i + 1) * 16, j * 16:(j + 1) * 16] = 5.0   # would be kept by score
    pk = etm.prune_pack(dev_tensor(W2, "fp16"), "tile", 0.7, (16, 16), mask_in=mask_in)
    np.testing.assert_array_equal(pk.mask()[:2].cpu().numpy().view(np.uint32), ref["mask"])
    dense = etm.unpack(pk).float().cpu().numpy().astype(np.float64)
    np.testing.assert_array_equal(dense, ref["W_pruned"])
