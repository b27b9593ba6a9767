"""Oracle: the pruned Transformer-encoder forward pass, literally (CPU, float64).

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

E.T.'s on-the-fly operator, pre-computed operator and scale reordering all
reach exactly (up to rounding order) the plain definition of the encoder
(§3.1: OTF computes Eq. 3; line 159 §3.3: the reorder
"yields the same results"; line 131: the pre-computed operator "yields the
same results").  So this module IS that definition, written out:

  * linear projections Q = X W_Q'^T + b_Q, K = ..., V = ...   (line 68, §2.1)
    with W' the pruned weights from oracle.prune (zeros where pruned);
  * per (batch b, head h): A = Q_h K_h^T / sqrt(d_k)          (Eq. 3, line 70)
    (the scale AFTER the product, as in the plain Eq. 3);
  * mask: A[i, j] = -inf for keys j >= len_b (padding) and, if causal, j > i
    (line 73: masked entries set to negative infinity before softmax);
  * P = softmax_row(A) (max-subtracted, two passes);  Z_h = P V_h;
    Z = ||_h Z_h;   attn = Z W_O'^T + b_O                     (Eq. 3-4, lines 70-73, 119)
  * encoder layer (line 75, §2.1): Y1 = LN(X + attn);
    U = act(Y1 W_1'^T + b_1); Y2 = LN(Y1 + U W_2'^T + b_2)
    LayerNorm with biased variance (reading C-11); GELU(erf) / ReLU (C-12).

Readings: biases are never pruned (C-6); padded query rows are
computed and compared like any other row (C-19); lengths 1 <= len_b <= S (C-7).
Parity: pinned by tests/test_oracle_encoder.py (torch float64 MHA /
TransformerEncoderLayer at ratio 0, closed forms P1/P2/P4, Eq. 4/5 identities,
brute force scalar loops, invariances).
"""
from __future__ import annotations

import math

import numpy as np
from scipy.special import erf


def linear(X: np.ndarray, W: np.ndarray, b: np.ndarray | None) -> np.ndarray:
    """Y = X . W^T (+ b); W is [out, in]."""
    Y = np.asarray(X, np.float64) @ np.asarray(W, np.float64).T
    if b is not None:
        Y = Y + np.asarray(b, np.float64)
    return Y


def gelu(x: np.ndarray) -> np.ndarray:
    """GELU(x) = 0.5 x (1 + erf(x / sqrt(2))) (reading C-12)."""
    return 0.5 * x * (1.0 + erf(x / math.sqrt(2.0)))


def relu(x: np.ndarray) -> np.ndarray:
    return np.maximum(x, 0.0)


def activation(name: str):
    return {"gelu": gelu, "relu": relu}[name]


def layer_norm(v: np.ndarray, gamma, beta, eps: float) -> np.ndarray:
    """LN over the last axis: gamma (.) (v - mu) / sqrt(var + eps) + beta, biased var (C-11)."""
    v = np.asarray(v, np.float64)
    mu = v.mean(axis=-1, keepdims=True)
    var = ((v - mu) ** 2).mean(axis=-1, keepdims=True)
    return np.asarray(gamma, np.float64) * (v - mu) / np.sqrt(var + eps) + np.asarray(beta, np.float64)


def key_mask(S: int, length: int, causal: bool) -> np.ndarray:
    """Boolean [S, S] matrix: True where query i may attend key j (line 73; reading C-7)."""
    j = np.arange(S)[None, :]
    i = np.arange(S)[:, None]
    allowed = np.broadcast_to(j < length, (S, S)).copy()
    if causal:
        allowed &= j <= i
    return allowed


def softmax_masked(A: np.ndarray, allowed: np.ndarray) -> np.ndarray:
    """Row softmax with excluded entries at -inf (probability exactly 0), max-subtracted."""
    A = np.where(allowed, A, -np.inf)
    m = A.max(axis=-1, keepdims=True)
    e = np.where(allowed, np.exp(A - m), 0.0)
    return e / e.sum(axis=-1, keepdims=True)


def attention_core(Q, K, V, heads: int, lengths, causal: bool = False, dk: int | None = None,
                   return_probs: bool = False):
    """Steps 2-6 of Fig. 3(a): per (b, h) Z_h = softmax(Q_h K_h^T / sqrt(d_k), masked) V_h.

    Q, K: [B, S, H*dq]; V: [B, S, H*dv] (dv may differ from dq under row pruning of
    W_V only through zero columns; here V keeps its full width).  d_k defaults to
    Q's per-head width.  Returns Z [B, S, H*dv] (and P [B, H, S, S] if asked).
    """
    Q = np.asarray(Q, np.float64)
    K = np.asarray(K, np.float64)
    V = np.asarray(V, np.float64)
    B, S, dq_all = Q.shape
    dq = dq_all // heads
    dv = V.shape[2] // heads
    dk = dq if dk is None else dk
    Z = np.zeros((B, S, heads * dv))
    P_all = np.zeros((B, heads, S, S)) if return_probs else None
    for b in range(B):
        allowed = key_mask(S, int(lengths[b]), causal)
        for h in range(heads):
            Qh = Q[b, :, h * dq:(h + 1) * dq]
            Kh = K[b, :, h * dq:(h + 1) * dq]
            Vh = V[b, :, h * dv:(h + 1) * dv]
            A = (Qh @ Kh.T) / math.sqrt(dk)              # Eq. 3: scale after Q.K^T
            P = softmax_masked(A, allowed)
            Z[b, :, h * dv:(h + 1) * dv] = P @ Vh
            if return_probs:
                P_all[b, h] = P
    return (Z, P_all) if return_probs else Z


def attention_block(X, w: dict, heads: int, lengths, causal: bool = False, return_all: bool = False):
    """Self-attention block: projections + attention core + output projection (Eq. 3-4).

    `w` holds pruned weights as float arrays: wq, wk, wv, wo ([d, d]) and biases
    bq, bk, bv, bo.  Returns attn [B, S, d] (and every intermediate if asked).
    """
    X = np.asarray(X, np.float64)
    B, S, d = X.shape
    Q = linear(X, w["wq"], w["bq"])
    K = linear(X, w["wk"], w["bk"])
    V = linear(X, w["wv"], w["bv"])
    Z, P = attention_core(Q, K, V, heads, lengths, causal, dk=d // heads, return_probs=True)
    attn = linear(Z, w["wo"], w["bo"])                   # Eq. 4: Z . W_O^T
    if return_all:
        return attn, {"Q": Q, "K": K, "V": V, "P": P, "Z": Z, "attn": attn}
    return attn


def encoder_layer(X, w: dict, heads: int, lengths, causal: bool, act: str, eps: float,
                  return_all: bool = False):
    """One post-LN encoder layer (§2.1)."""
    X = np.asarray(X, np.float64)
    attn, inter = attention_block(X, w, heads, lengths, causal, return_all=True)
    Y1 = layer_norm(X + attn, w["ln1_g"], w["ln1_b"], eps)
    U = activation(act)(linear(Y1, w["w1"], w["b1"]))
    F = linear(U, w["w2"], w["b2"])
    Y2 = layer_norm(Y1 + F, w["ln2_g"], w["ln2_b"], eps)
    if return_all:
        inter.update({"Y1": Y1, "U": U, "F": F, "Y2": Y2})
        return Y2, inter
    return Y2


def encoder(X, layers: list, heads: int, lengths, causal: bool, act: str, eps: float,
            return_all: bool = False):
    """Stack of L encoder layers (line 57: an encoder stack of identical structure)."""
    h = np.asarray(X, np.float64)
    inters = []
    for w in layers:
        h, inter = encoder_layer(h, w, heads, lengths, causal, act, eps, return_all=True)
        inters.append(inter)
    return (h, inters) if return_all else h


# --------------------------------------------------------------------------
# glue: prune a whole layer with the per-matrix pattern
# --------------------------------------------------------------------------

def prune_layer(raw: dict, scheme: str, ratio: float, tile: int = 16) -> tuple[dict, dict]:
    """Apply the scheme's pattern to each of the six matrices; biases / LN params untouched (C-6).

    Returns (pruned float64 weights, per-matrix prune records).
    """
    from oracle.prune import prune
    from et_synth import MATRICES, matrix_pattern

    w = {k: np.asarray(v, np.float64) for k, v in raw.items()}
    recs = {}
    for name in MATRICES:
        pat = matrix_pattern(scheme, name)
        rec = prune(raw[name], pat, ratio, tile, tile)
        w[name] = rec["W_pruned"]
        recs[name] = rec
    return w, recs
