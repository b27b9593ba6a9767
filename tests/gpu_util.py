"""Helpers shared by the -m gpu parity tests (no method arithmetic here)."""
import numpy as np
import torch

TOL_MAX_ABS = 2e-2     # north_star: FP16/BF16 max-abs vs the float64 oracle
TOL_REL_FRO = 5e-3     # north_star: relative Frobenius


def dev_tensor(a: np.ndarray, dtype: str) -> torch.Tensor:
    tdt = {"fp16": torch.float16, "bf16": torch.bfloat16, "fp32": torch.float32}[dtype]
    return torch.from_numpy(np.ascontiguousarray(a, dtype=np.float32)).to("cuda").to(tdt).contiguous()


def to64(t: torch.Tensor) -> np.ndarray:
    return t.detach().float().cpu().numpy().astype(np.float64)


def errors(gpu: np.ndarray, ref: np.ndarray):
    d = gpu - ref
    return float(np.abs(d).max()), float(np.linalg.norm(d) / max(np.linalg.norm(ref), 1e-300))


def assert_close(gpu: np.ndarray, ref: np.ndarray, max_abs=TOL_MAX_ABS, rel_fro=TOL_REL_FRO, what=""):
    assert np.all(np.isfinite(gpu)), f"{what}: non-finite values"
    ma, rf = errors(gpu, ref)
    assert ma <= max_abs and rf <= rel_fro, f"{what}: max-abs {ma:.3e} (<= {max_abs}), rel-fro {rf:.3e} (<= {rel_fro})"
    return ma, rf
