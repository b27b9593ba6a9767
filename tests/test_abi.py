"""The C-ABI library loads on a CPU-only host and exports every function include/et.h declares;
host-only entry points (size query, argument validation) behave as documented."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "et.h")


def _declared():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(et_[a-z0-9_]+)\s*\(", src)))


@pytest.fixture(scope="module")
def et():
    import paper_conf_sc_chenhplg0d021_b200 as m   # builds nothing; fails loudly if libet.so is absent
    return m


def test_every_declared_symbol_is_exported(et):
    names = _declared()
    assert len(names) >= 14
    missing = [n for n in names if not hasattr(et._lib, n)]
    assert not missing, f"missing exports: {missing}"
    assert set(names) <= set(et.SYMBOLS)
    assert not hasattr(et._lib, "et_diag_mma_probe")   # probes live in libet_diag.so


def test_version_and_error_string(et):
    assert "sm_100a" in et.version()


def _query(et, rows, cols, dtype, pat, ratio, r=16, c=16, group=0):
    sizes = [ctypes.c_size_t() for _ in range(8)]
    nnz = ctypes.c_int32()
    st = et._q(rows, cols, dtype, pat, ratio, r, c, group, None, ctypes.byref(nnz), *[ctypes.byref(s) for s in sizes])
    return st, nnz.value, [s.value for s in sizes]


def test_prune_pack_query_counts(et):
    # keep 461 of 2304 tiles (768x768) and 1843 of 9216 (3072x768) at 80 %
    st, nnz, sz = _query(et, 768, 768, et.FP16, et.PRUNE_TILE, 0.8)
    assert st == 0 and nnz == 461
    assert sz[0] == 72 * 4                    # mask: ceil(2304 / 32) words
    assert sz[2] == 49 * 4                    # row_ptr
    assert sz[6] == 2304 * 512                # values: worst case (all tiles) x 512 B
    st, nnz, _ = _query(et, 3072, 768, et.FP16, et.PRUNE_TILE, 0.8)
    assert st == 0 and nnz == 1843
    st, nnz, _ = _query(et, 768, 768, et.FP16, et.PRUNE_ROW, 0.8, group=64)
    assert st == 0 and nnz == 154             # C4 W_V rows
    st, nnz, _ = _query(et, 64, 64, et.FP32, et.PRUNE_TILE, 0.5)
    assert st == 0 and nnz == 8               # C1


def test_prune_pack_query_rejects_bad_arguments(et):
    assert _query(et, 768, 768, et.FP16, et.PRUNE_TILE, 1.5)[0] == 1       # ratio outside [0, 1]
    assert "ratio" in et._lib.et_last_error().decode()
    assert _query(et, 770, 768, et.FP16, et.PRUNE_TILE, 0.5)[0] == 1       # tile does not divide
    assert _query(et, 768, 768, et.FP16, 9, 0.5)[0] == 1                   # bad pattern
    assert _query(et, 768, 768, et.FP16, et.PRUNE_ROW, 0.5, group=100)[0] == 1


def test_gather_cols_validates_before_launch(et):
    # et_gather_cols (column pruning, X_adjusted): argument errors return before any
    # CUDA call, so they are checkable on a CPU-only host
    g = et._gather
    assert g(None, 4, 64, None, 10, 12, et.FP16, None, None) == 1          # nk_pad % 8 != 0
    assert "multiple" in et._lib.et_last_error().decode()
    assert g(None, 4, 64, None, 10, 8, et.FP16, None, None) == 1           # nk_pad < nk
    assert g(None, 4, 64, None, 4, 8, 7, None, None) == 1                  # bad dtype
    assert g(None, 4, 64, None, 4, 8, et.FP16, None, None) == 1            # null pointers
    assert g(None, 0, 64, None, 0, 8, et.FP16, None, None) == 0            # empty: nothing to do


def test_product_has_no_cpu_fallback(et):
    import torch
    if torch.cuda.is_available():
        pytest.skip("CPU-only check")
    with pytest.raises(Exception):
        et.prune_pack(torch.zeros(64, 64), "tile", 0.5)        # host tensor: no silent CPU path
