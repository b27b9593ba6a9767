"""Pins for oracle/prune.py (CPU).  Each test fixes the oracle to something other than itself:
hand-computed fixtures (tests/golden/), a brute-force rank definition, scalar-loop
accumulation order, closed-form counts and invariants."""
import json
import math
import os

import numpy as np
import pytest

from oracle import prune as op
from et_synth import make_matrix


def _load(golden_dir, name):
    with open(os.path.join(golden_dir, name)) as f:
        return json.load(f)


def test_fig6_handworked_fixture(golden_dir):
    g = _load(golden_dir, "fig6_tile_prune_handworked.json")
    W = np.array(g["W"], dtype=np.float64)
    r, c = g["tile"]
    np.testing.assert_array_equal(op.tile_scores(W, r, c), np.array(g["tile_scores_sq"], float))
    for case in g["cases"]:
        rec = op.prune_tile(W, case["ratio"], r, c)
        assert op.n_pruned(case["ratio"], 8) == case["n_prune"]
        np.testing.assert_array_equal(rec["tile_mask"].astype(int), np.array(case["tile_mask"]))
        np.testing.assert_array_equal(rec["mask"], np.array(case["bitmap"], dtype=np.uint32))
        np.testing.assert_array_equal(rec["row_ptr"], np.array(case["row_ptr"]))
        np.testing.assert_array_equal(rec["col_idx"], np.array(case["col_idx"], dtype=np.int32))
        if "W_pruned" in case:
            np.testing.assert_array_equal(rec["W_pruned"], np.array(case["W_pruned"], float))


def test_fig5a_row_prune_fixture(golden_dir):
    g = _load(golden_dir, "fig5a_row_prune_handworked.json")
    W = np.array(g["W"], float)
    rec = op.prune_row(W, g["ratio"])
    np.testing.assert_array_equal(rec["scores"], np.array(g["row_scores_sq"], float))
    np.testing.assert_array_equal(rec["idx"], np.array(g["kept_rows"]))
    np.testing.assert_array_equal(rec["mask"], np.array(g["bitmap"], dtype=np.uint32))
    np.testing.assert_array_equal(rec["W_condensed"], np.array(g["W_condensed"], float))
    X = np.array(g["X"], float)
    np.testing.assert_array_equal(X @ rec["W_condensed"].T, np.array(g["XWcT"], float))
    # condensed product == the pruned full-shape product restricted to kept columns
    np.testing.assert_array_equal((X @ rec["W_pruned"].T)[:, rec["idx"]], X @ rec["W_condensed"].T)


def test_fig3_toy_shapes(golden_dir):
    g = _load(golden_dir, "fig3_toy_shapes.json")
    assert g["d_model"] // g["heads"] == g["d_k"]


def test_n_pruned_rounding_closed_form():
    # floor(p*T + 0.5): SURVEY §8(a) a1 counts
    assert op.n_pruned(0.8, 2304) == 1843            # keep 461 of a 768x768 matrix
    assert op.n_pruned(0.8, 9216) == 7373            # keep 1843 of a 3072x768 matrix
    assert op.n_pruned(0.8, 1024) == 819             # C2 d=512: keep 205
    assert op.n_pruned(0.8, 4096) == 3277            # C2 FFN: keep 819
    assert op.n_pruned(0.5, 16) == 8 and op.n_pruned(0.5, 64) == 32   # C1
    assert op.n_pruned(0.8, 768) == 614              # C4 W_V rows: keep 154
    assert op.n_pruned(0.0, 100) == 0 and op.n_pruned(1.0, 100) == 100
    with pytest.raises(ValueError):
        op.n_pruned(1.5, 10)


def test_score_accumulation_order_is_the_scalar_loop():
    """Reading C-2 fixes the FP64 order a-outer, b-inner; pin it against a scalar loop."""
    W = make_matrix(11, (48, 32), 0.02, "fp16").astype(np.float64)
    s = op.tile_scores(W, 16, 16)
    for i in range(3):
        for j in range(2):
            acc = 0.0
            for a in range(16):
                for b in range(16):
                    w = float(W[i * 16 + a, j * 16 + b])
                    acc = acc + w * w
            assert s[i, j] == acc                      # bit-exact
    rs = op.row_scores(W)
    for i in (0, 17, 47):
        acc = 0.0
        for j in range(32):
            acc = acc + float(W[i, j]) ** 2
        assert rs[i] == acc


def _brute_rank_keep(scores_flat, ratio):
    """Definition by counting (no sort): rank(t) = #{u : (s_u, u) < (s_t, t)}; pruned iff rank < n_prune."""
    T = len(scores_flat)
    k = int(math.floor(ratio * T + 0.5))
    keep = []
    for t in range(T):
        rank = sum(1 for u in range(T) if scores_flat[u] < scores_flat[t]
                   or (scores_flat[u] == scores_flat[t] and u < t))
        keep.append(rank >= k)
    return np.array(keep)


@pytest.mark.parametrize("shape,tile,ratio,dtype", [
    ((64, 96), 16, 0.8, "fp16"), ((64, 96), 16, 0.5, "bf16"), ((32, 32), 4, 0.3, "fp32"),
    ((48, 16), 16, 0.95, "fp16"), ((16, 64), 8, 0.0, "fp16"), ((16, 64), 8, 1.0, "fp16")])
def test_tile_selection_matches_bruteforce_l2_ranking(shape, tile, ratio, dtype):
    W = make_matrix(100 + shape[0] + tile, shape, 0.05, dtype).astype(np.float64)
    rec = op.prune_tile(W, ratio, tile, tile)
    p, q = shape[0] // tile, shape[1] // tile
    # independent score: exactly rounded sum of squares (math.fsum) of each tile
    sc = [math.fsum(float(v) ** 2 for v in W[i * tile:(i + 1) * tile, j * tile:(j + 1) * tile].ravel())
          for i in range(p) for j in range(q)]
    np.testing.assert_array_equal(rec["tile_mask"].reshape(-1), _brute_rank_keep(sc, ratio))
    # invariants (P7)
    T = p * q
    assert rec["nnz"] == T - op.n_pruned(ratio, T)
    nrm = np.array([np.linalg.norm(W[i * tile:(i + 1) * tile, j * tile:(j + 1) * tile])
                    for i in range(p) for j in range(q)])
    km = rec["tile_mask"].reshape(-1)
    if km.any() and (~km).any():
        assert nrm[km].min() >= nrm[~km].max()
    # CSR consistency
    assert rec["row_ptr"][0] == 0 and rec["row_ptr"][-1] == rec["nnz"]
    for i in range(p):
        cols = rec["col_idx"][rec["row_ptr"][i]:rec["row_ptr"][i + 1]]
        assert list(cols) == sorted(cols)
        np.testing.assert_array_equal(cols, np.nonzero(rec["tile_mask"][i])[0])
    # bitmap round trip and bit order
    np.testing.assert_array_equal(op.unbitmap(rec["mask"], T), km)
    # W' = mask (.) W
    for i in range(p):
        for j in range(q):
            blk = rec["W_pruned"][i * tile:(i + 1) * tile, j * tile:(j + 1) * tile]
            ref = W[i * tile:(i + 1) * tile, j * tile:(j + 1) * tile]
            np.testing.assert_array_equal(blk, ref if rec["tile_mask"][i, j] else 0 * ref)


def test_ties_lower_index_pruned_first():
    # all-zero W: every score ties, so the first n_prune tiles by linear index go (P7)
    W = np.zeros((64, 64))
    rec = op.prune_tile(W, 0.5, 16, 16)
    np.testing.assert_array_equal(rec["tile_mask"].reshape(-1), np.arange(16) >= 8)
    # duplicated tiles: identical content => identical score; lower index pruned first
    W = np.zeros((32, 32))
    blk = np.arange(256, dtype=float).reshape(16, 16) / 100
    for i in range(2):
        for j in range(2):
            W[i * 16:(i + 1) * 16, j * 16:(j + 1) * 16] = blk
    rec = op.prune_tile(W, 0.25, 16, 16)
    np.testing.assert_array_equal(rec["tile_mask"].reshape(-1), [False, True, True, True])
    rec = op.prune_tile(W, 0.75, 16, 16)
    np.testing.assert_array_equal(rec["tile_mask"].reshape(-1), [False, False, False, True])


def test_row_and_col_selection_bruteforce():
    W = make_matrix(7, (64, 48), 0.02, "fp16").astype(np.float64)
    rr = op.prune_row(W, 0.8)
    sc = [math.fsum(float(v) ** 2 for v in W[i]) for i in range(64)]
    np.testing.assert_array_equal(rr["keep"], _brute_rank_keep(sc, 0.8))
    assert rr["nnz"] == 64 - op.n_pruned(0.8, 64)
    np.testing.assert_array_equal(rr["W_condensed"], W[rr["idx"]])
    cc = op.prune_col(W, 0.5)
    sc = [math.fsum(float(v) ** 2 for v in W[:, j]) for j in range(48)]
    np.testing.assert_array_equal(cc["keep"], _brute_rank_keep(sc, 0.5))
    X = make_matrix(8, (5, 64), 1.0, "fp16").astype(np.float64)
    # Fig. 5(b): X_adjusted (kept columns of X) times condensed W^T == X times pruned W^T
    Wt = make_matrix(9, (32, 64), 0.02, "fp16").astype(np.float64)
    c2 = op.prune_col(Wt, 0.5)
    np.testing.assert_allclose(X[:, c2["idx"]] @ c2["W_condensed"].T, X @ c2["W_pruned"].T,
                               rtol=1e-13, atol=1e-15)


def test_mask_in_overrides_and_pruned_values_do_not_matter():
    """P5 (oracle side): with a fixed mask, changing values inside pruned tiles leaves W' unchanged."""
    W = make_matrix(5, (64, 64), 0.02, "fp16").astype(np.float64)
    rec = op.prune_tile(W, 0.6, 16, 16)
    W2 = W.copy()
    for i in range(4):
        for j in range(4):
            if not rec["tile_mask"][i, j]:
                W2[i * 16:(i + 1) * 16, j * 16:(j + 1) * 16] += 7.0
    rec2 = op.prune_tile(W2, 0.6, 16, 16, mask_in=rec["tile_mask"])
    np.testing.assert_array_equal(rec["W_pruned"], rec2["W_pruned"])


def test_bad_shapes_rejected():
    with pytest.raises(ValueError):
        op.tile_scores(np.zeros((20, 16)), 16, 16)


def _zero_structure(Wp, t=16):
    """(all-zero rows, all-zero t x t blocks, blocks that are partly zero) of a pruned matrix."""
    zr = int(np.sum(np.all(Wp == 0, axis=1)))
    r, c = Wp.shape[0] // t, Wp.shape[1] // t
    blocks = Wp.reshape(r, t, c, t).transpose(0, 2, 1, 3).reshape(r, c, t * t)
    zb = int(np.sum(np.all(blocks == 0, axis=2)))
    partial = int(np.sum(np.any(blocks == 0, axis=2) & ~np.all(blocks == 0, axis=2)))
    return zr, zb, partial


@pytest.mark.parametrize("scheme", ["attention-aware", "tile"])
def test_pattern_assignment_per_matrix(scheme):
    """The per-matrix pattern of oracle.prune_layer, read off the pruned weights themselves
    (§5.3 (i): attention-aware = "row pruned for W_V on all encoder layers and
    tensor tile pruned for other weights"; (iv): tile pruning for all weights).  Under
    attention-aware pruning W_V (and only W_V) has exactly floor(p d + 0.5) all-zero ROWS whose
    zeros cut across 16x16 tiles; W_Q, W_K, W_O, W_1, W_2 have exactly floor(p T + 0.5) all-zero
    16x16 TILES and no other zeros.  Swapping any two table entries fails this test."""
    from et_synth import CONFIGS, make_layer
    from oracle.encoder import prune_layer
    cfg = CONFIGS["C2"]            # d = 512, d_ff = 2048, p = 0.8
    raw = make_layer(cfg, 0)
    w, _ = prune_layer(raw, scheme, cfg.ratio)
    d, f, p = cfg.d_model, cfg.d_ff, cfg.ratio
    for name, (rows, cols) in {"wq": (d, d), "wk": (d, d), "wv": (d, d), "wo": (d, d), "w1": (f, d),
                               "w2": (d, f)}.items():
        zr, zb, partial = _zero_structure(w[name])
        if scheme == "attention-aware" and name == "wv":
            assert zr == math.floor(p * rows + 0.5), name          # row pattern: whole rows gone
            assert partial > 0, name                                # ... that do not align with tiles
        else:
            T = (rows // 16) * (cols // 16)
            assert zb == math.floor(p * T + 0.5), name               # tile pattern: whole tiles gone
            assert partial == 0 and zr == 0, name                   # ... and nothing else
