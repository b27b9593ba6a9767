"""Fit g(t) = -log2(erfc(t)) on [0, 4] (g(0) = 0) for the GEMM epilogue's GELU (tsgemm.cu gelu_erf)
and report the float32 error of GELU(x) = x * Phi(x) against the exact erf form."""
import numpy as np
from scipy.special import erf, erfc

T, deg = 4.0, 5   # number of coefficients of q (degree deg - 1); tsgemm.cu uses 5
t = np.cos(np.linspace(0, np.pi, 4000)) * T / 2 + T / 2
y = -np.log2(erfc(t))
A = np.stack([t ** (k + 1) for k in range(deg)], axis=1)
w = 2.0 ** (-y)
c, *_ = np.linalg.lstsq(A * w[:, None], y * w, rcond=None)
print("coefficients of q (t^0..):", [float(f"{v:.10f}") for v in c])
x = np.linspace(-12, 12, 2000001).astype(np.float32)
cf = c.astype(np.float32)
tt = np.minimum(np.abs(x) * np.float32(0.70710678118654752), np.float32(T))
q = cf[-1]
for k in range(deg - 2, -1, -1):
    q = q * tt + cf[k]
e = np.exp2(-(tt * q + 1)).astype(np.float32)
gelu = x * np.where(x >= 0, 1 - e, e)
ref = 0.5 * x.astype(np.float64) * (1 + erf(x.astype(np.float64) / np.sqrt(2)))
print("max |GELU error| = %.3e" % np.abs(gelu - ref).max())
