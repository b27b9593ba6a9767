"""Oracle: independent formulations of the same attention (used ONLY as pins).

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

These restate the paper's alternative derivations so the main oracle
(oracle/encoder.py) can be checked against something other than itself:

  * otf_rowwise      -- Fig. 3(a) steps 2-6 literally, one row of one head at
                        a time, with the scale moved BEFORE Q.K^T (PAPER.md
                        lines 111-113 §3.1, line 159 §3.3);
  * precomputed_attn -- Eq. 5 (lines 124-131): Output = sum_h S_h (X W_VO,h)
                        with W_VO,h = W_V,h^T W_O,h^T, plus the bias fold
                        b_O + sum_h W_O,h b_V,h (reading C-6);
  * brute_force_layer -- scalar triple loops, no BLAS, for tiny shapes (C1).
"""
from __future__ import annotations

import math

import numpy as np


def otf_rowwise(Q, K, V, heads: int, lengths, causal: bool = False):
    """Per row i of per head h: q~ = q_i / sqrt(d_k) (step 2, scale first), s = q~ K_h^T (3),
    mask (4), softmax via max / exp / sum (5), z_i = s V_h (6)."""
    Q = np.asarray(Q, np.float64)
    K = np.asarray(K, np.float64)
    V = np.asarray(V, np.float64)
    B, S, dall = Q.shape
    dk = dall // heads
    Z = np.zeros_like(V)
    for b in range(B):
        L = int(lengths[b])
        for h in range(heads):
            sl = slice(h * dk, (h + 1) * dk)
            for i in range(S):
                q = Q[b, i, sl] / math.sqrt(dk)                   # step 2 (reordered, §3.3)
                row = np.array([q @ K[b, j, sl] for j in range(S)])  # step 3
                ok = np.array([(j < L) and (not causal or j <= i) for j in range(S)])
                row = np.where(ok, row, -np.inf)                  # step 4
                mx = row.max()
                e = np.where(ok, np.exp(row - mx), 0.0)           # step 5
                s = e / e.sum()
                Z[b, i, sl] = s @ V[b, :, sl]                     # step 6
    return Z


def precomputed_attn(X, w: dict, heads: int, lengths, causal: bool = False):
    """Eq. 5: attn = sum_h S_h . X . (W_V,h^T . W_O,h^T)  + b_O + sum_h W_O,h b_V,h."""
    X = np.asarray(X, np.float64)
    B, S, d = X.shape
    dk = d // heads
    Q = X @ w["wq"].T + w["bq"]
    K = X @ w["wk"].T + w["bk"]
    out = np.zeros((B, S, d))
    bias = np.asarray(w["bo"], np.float64).copy()
    for h in range(heads):
        sl = slice(h * dk, (h + 1) * dk)
        Wvo = w["wv"][sl, :].T @ w["wo"][:, sl].T           # offline: W_V,h^T W_O,h^T  [d, d]
        bias = bias + w["wo"][:, sl] @ w["bv"][sl]          # rows of P sum to 1 => bias fold
        XW = X @ Wvo                                         # step 1 with the pre-computed matrix
        for b in range(B):
            L = int(lengths[b])
            A = Q[b, :, sl] @ K[b, :, sl].T / math.sqrt(dk)
            j = np.arange(S)[None, :]
            i = np.arange(S)[:, None]
            ok = (j < L) & ((j <= i) if causal else True)
            A = np.where(ok, A, -np.inf)
            E = np.where(ok, np.exp(A - A.max(axis=1, keepdims=True)), 0.0)
            Sh = E / E.sum(axis=1, keepdims=True)
            out[b] += Sh @ XW[b]                             # step 8: sum over heads
    return out + bias


def _matvec_loops(x, W, b):
    out = []
    for o in range(len(W)):
        acc = 0.0
        for k in range(len(x)):
            acc += float(x[k]) * float(W[o][k])
        out.append(acc + (float(b[o]) if b is not None else 0.0))
    return out


def brute_force_layer(X, w: dict, heads: int, lengths, causal: bool, act: str, eps: float):
    """Scalar-loop encoder layer (no BLAS, no numpy reductions) for tiny shapes."""
    X = np.asarray(X, np.float64)
    B, S, d = X.shape
    dk = d // heads
    lst = lambda a: np.asarray(a, np.float64).tolist()
    WQ, WK, WV, WO = lst(w["wq"]), lst(w["wk"]), lst(w["wv"]), lst(w["wo"])
    W1, W2 = lst(w["w1"]), lst(w["w2"])
    bq, bk, bv, bo, b1, b2 = (lst(w[k]) for k in ("bq", "bk", "bv", "bo", "b1", "b2"))

    def ln(v, g, be):
        n = len(v)
        mu = sum(v) / n
        var = sum((x - mu) ** 2 for x in v) / n
        return [float(g[i]) * (v[i] - mu) / math.sqrt(var + eps) + float(be[i]) for i in range(n)]

    def f_act(x):
        return 0.5 * x * (1.0 + math.erf(x / math.sqrt(2.0))) if act == "gelu" else max(x, 0.0)

    Y = np.zeros((B, S, d))
    for b in range(B):
        L = int(lengths[b])
        xs = [lst(X[b, i]) for i in range(S)]
        q = [_matvec_loops(x, WQ, bq) for x in xs]
        k = [_matvec_loops(x, WK, bk) for x in xs]
        v = [_matvec_loops(x, WV, bv) for x in xs]
        for i in range(S):
            z = [0.0] * d
            for h in range(heads):
                sc = []
                for j in range(S):
                    if j < L and (not causal or j <= i):
                        dot = 0.0
                        for t in range(h * dk, (h + 1) * dk):
                            dot += q[i][t] * k[j][t]
                        sc.append((j, dot / math.sqrt(dk)))
                mx = max(s for _, s in sc)
                ex = [(j, math.exp(s - mx)) for j, s in sc]
                tot = sum(e for _, e in ex)
                for j, e in ex:
                    for t in range(h * dk, (h + 1) * dk):
                        z[t] += (e / tot) * v[j][t]
            attn = _matvec_loops(z, WO, bo)
            y1 = ln([xs[i][t] + attn[t] for t in range(d)], lst(w["ln1_g"]), lst(w["ln1_b"]))
            u = [f_act(a) for a in _matvec_loops(y1, W1, b1)]
            f = _matvec_loops(u, W2, b2)
            Y[b, i] = ln([y1[t] + f[t] for t in range(d)], lst(w["ln2_g"]), lst(w["ln2_b"]))
    return Y
