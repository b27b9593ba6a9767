"""Oracle: tensor-tile / row / column pruning and packing (CPU, float64).

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

Follows PAPER.md line 196 (§4.2, Fig. 6 step (v) 1-4) step by step:
  1. divide W (m x n) into p x q tiles of r x c            (line 179: p = m/r, q = n/c)
  2. compute the l2 norm of every tile -> p x q norm matrix
     ("select ... the largest group l2 norm"; tiles below the pre-set
      percentile are set to 0)
  3. generate the p x q pruning mask (0 / 1)
  4. multiply the mask with W element-wise -> tile-pruned W'
Row / column pruning and condensing: line 169-171 (§4.1, Fig. 5).

Readings of the garbled / silent passages:
  C-1  tile r = c = 16 by default; r, c must divide m, n.
  C-2  rank tiles by the squared l2 norm sum(w^2) (same order as the l2 norm,
       without sqrt ties), accumulated in float64 in a FIXED order: a (tile row)
       outer, b (tile column) inner, sequential; prune exactly
       n_prune = floor(ratio * T + 0.5) tiles; ties broken by the linear tile
       index i*q + j, the lower index pruned first.  This makes the mask unique.
  C-3  the ratio is per matrix.
  C-5  row pruning ranks all m rows globally (no per-head quota).
Parity: pinned by tests/test_oracle_prune.py (hand-computed Fig. 6 fixture,
brute-force l2-norm ranking, invariants P7, P16).
"""
from __future__ import annotations

import math

import numpy as np


def n_pruned(ratio: float, units: int) -> int:
    """Number of pruned units: floor(ratio * T + 0.5) computed in double (reading C-2)."""
    if not (0.0 <= ratio <= 1.0):
        raise ValueError("ratio must be in [0, 1]")
    return int(math.floor(ratio * units + 0.5))


def tile_scores(W: np.ndarray, r: int = 16, c: int = 16) -> np.ndarray:
    """Step 2: squared l2 norm of every r x c tile, float64, fixed accumulation order.

    score[i, j] = sum_{a<r} sum_{b<c} W[i*r + a, j*c + b]^2, with the sum taken
    sequentially, a outer, b inner (vectorised across tiles only).
    """
    W = np.asarray(W, dtype=np.float64)
    m, n = W.shape
    if m % r or n % c:
        raise ValueError("tile size must divide the matrix shape (reading C-1)")
    p, q = m // r, n // c
    t = W.reshape(p, r, q, c)
    s = np.zeros((p, q), dtype=np.float64)
    for a in range(r):
        for b in range(c):
            w = t[:, a, :, b]
            s = s + w * w
    return s


def row_scores(W: np.ndarray) -> np.ndarray:
    """Squared l2 norm of every row, float64, sequential over the columns."""
    W = np.asarray(W, dtype=np.float64)
    s = np.zeros(W.shape[0], dtype=np.float64)
    for j in range(W.shape[1]):
        s = s + W[:, j] * W[:, j]
    return s


def col_scores(W: np.ndarray) -> np.ndarray:
    """Squared l2 norm of every column, float64, sequential over the rows."""
    W = np.asarray(W, dtype=np.float64)
    s = np.zeros(W.shape[1], dtype=np.float64)
    for i in range(W.shape[0]):
        s = s + W[i, :] * W[i, :]
    return s


def select_kept(scores: np.ndarray, ratio: float) -> np.ndarray:
    """Step 2-3: boolean keep-mask over the flattened units.

    Units are sorted by (score ascending, linear index ascending); the first
    n_prune of that order are pruned (reading C-2).
    """
    flat = np.asarray(scores, dtype=np.float64).reshape(-1)
    T = flat.size
    k = n_pruned(ratio, T)
    order = np.lexsort((np.arange(T), flat))   # primary key: score, secondary: index
    keep = np.ones(T, dtype=bool)
    keep[order[:k]] = False
    return keep


def bitmap(keep: np.ndarray) -> np.ndarray:
    """Pack a flat boolean keep-vector into uint32 words: unit t -> bit t%32 of word t//32."""
    keep = np.asarray(keep, dtype=bool).reshape(-1)
    words = np.zeros((keep.size + 31) // 32, dtype=np.uint32)
    for t in np.nonzero(keep)[0]:
        words[t // 32] |= np.uint32(1) << np.uint32(t % 32)
    return words


def unbitmap(words: np.ndarray, units: int) -> np.ndarray:
    words = np.asarray(words, dtype=np.uint32)
    t = np.arange(units)
    return ((words[t // 32] >> (t % 32).astype(np.uint32)) & 1).astype(bool)


def prune_tile(W: np.ndarray, ratio: float, r: int = 16, c: int = 16, mask_in=None) -> dict:
    """Tensor-tile pruning (steps 1-4 of PAPER.md line 196).

    Returns the p x q tile mask (bool), its bitmap, the CSR tile index
    (row_ptr[p+1], col_idx[nnz] ascending within each tile row) and
    W' = mask (.) W (float64).  `mask_in` (bool [p, q]) overrides selection.
    """
    W64 = np.asarray(W, dtype=np.float64)
    m, n = W64.shape
    p, q = m // r, n // c
    scores = tile_scores(W64, r, c)
    if mask_in is None:
        tmask = select_kept(scores, ratio).reshape(p, q)
    else:
        tmask = np.asarray(mask_in, dtype=bool).reshape(p, q)
    row_ptr = np.zeros(p + 1, dtype=np.int32)
    cols = []
    for i in range(p):
        js = np.nonzero(tmask[i])[0]
        cols.extend(js.tolist())
        row_ptr[i + 1] = row_ptr[i] + len(js)
    col_idx = np.asarray(cols, dtype=np.int32)
    full = np.kron(tmask.astype(np.float64), np.ones((r, c)))      # step 3: expand the p x q mask
    return {
        "pattern": "tile", "scores": scores, "tile_mask": tmask, "mask": bitmap(tmask),
        "row_ptr": row_ptr, "col_idx": col_idx, "nnz": int(tmask.sum()),
        "W_pruned": W64 * full,                                      # step 4
    }


def prune_row(W: np.ndarray, ratio: float, mask_in=None) -> dict:
    """Row pruning + condensing (Fig. 5(a)).

    The kept rows form W_pruned_condensed (dense, fewer rows); X . W_condensed^T
    gives the non-zero output columns.  W_pruned keeps the full shape with
    pruned rows zeroed (what the encoder computes with).
    """
    W64 = np.asarray(W, dtype=np.float64)
    scores = row_scores(W64)
    keep = select_kept(scores, ratio) if mask_in is None else np.asarray(mask_in, dtype=bool)
    idx = np.nonzero(keep)[0].astype(np.int32)
    Wp = W64 * keep[:, None]
    return {
        "pattern": "row", "scores": scores, "keep": keep, "mask": bitmap(keep),
        "idx": idx, "nnz": int(keep.sum()), "W_pruned": Wp, "W_condensed": W64[idx],
    }


def prune_col(W: np.ndarray, ratio: float, mask_in=None) -> dict:
    """Column pruning + condensing (Fig. 5(b)); X_adjusted gathers X's columns."""
    W64 = np.asarray(W, dtype=np.float64)
    scores = col_scores(W64)
    keep = select_kept(scores, ratio) if mask_in is None else np.asarray(mask_in, dtype=bool)
    idx = np.nonzero(keep)[0].astype(np.int32)
    return {
        "pattern": "col", "scores": scores, "keep": keep, "mask": bitmap(keep),
        "idx": idx, "nnz": int(keep.sum()), "W_pruned": W64 * keep[None, :],
        "W_condensed": W64[:, idx],
    }


def prune(W: np.ndarray, pattern: str, ratio: float, r: int = 16, c: int = 16, mask_in=None) -> dict:
    if pattern == "tile":
        return prune_tile(W, ratio, r, c, mask_in)
    if pattern == "row":
        return prune_row(W, ratio, mask_in)
    if pattern == "col":
        return prune_col(W, ratio, mask_in)
    if pattern == "none":
        W64 = np.asarray(W, dtype=np.float64)
        return {"pattern": "none", "W_pruned": W64.copy(), "nnz": W64.size}
    raise ValueError(pattern)
