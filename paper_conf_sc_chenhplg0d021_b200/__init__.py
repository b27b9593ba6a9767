"""Python binding of libet.so — the B200-native (sm_100a) hot path of E.T. (SC'21).

Argument marshalling only: every step of the path runs in the CUDA kernels of libet.so
(include/et.h).  PyTorch is used for device memory and streams; there is no CPU fallback:
loading fails loudly if the library is missing, and every call raises on a non-OK status.

Names follow the C ABI: prune_pack, unpack, linear_fwd, layernorm_fwd, attn_core_fwd,
attention_fwd, encoder_fwd (+ the *_workspace_size queries).
"""
from __future__ import annotations

import ctypes
import os

import torch

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("ET_LIB_PATH") or os.path.join(_HERE, "libet.so")

# enums (include/et.h)
FP16, BF16, FP32 = 0, 1, 2
PRUNE_NONE, PRUNE_TILE, PRUNE_ROW, PRUNE_COL = 0, 1, 2, 3
ATTN_AUTO, ATTN_SHORT, ATTN_LONG, ATTN_SHORT_GENERIC = 0, 1, 2, 3
ACT_GELU_ERF, ACT_RELU = 0, 1
EPI_BIAS, EPI_BIAS_SCALE, EPI_BIAS_GELU, EPI_BIAS_RELU, EPI_F32, EPI_PART16 = 0, 1, 2, 3, 4, 5

_DT = {"fp16": FP16, "bf16": BF16, "fp32": FP32}
_TORCH_DT = {FP16: torch.float16, BF16: torch.bfloat16, FP32: torch.float32}
_PAT = {"none": PRUNE_NONE, "tile": PRUNE_TILE, "row": PRUNE_ROW, "col": PRUNE_COL}
_MODE = {"auto": ATTN_AUTO, "short": ATTN_SHORT, "long": ATTN_LONG, "short_generic": ATTN_SHORT_GENERIC}
_ACT = {"gelu": ACT_GELU_ERF, "relu": ACT_RELU}


class EtError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"et status {status}: {msg}")
        self.status = status


def _load():
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing: build it with `python paper_conf_sc_chenhplg0d021_b200/build.py` "
                          "(there is no CPU fallback)")
    return ctypes.CDLL(LIB_PATH)


_lib = _load()
_vp, _i32, _sz, _f32, _f64 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_size_t, ctypes.c_float, ctypes.c_double


class PackedWeightC(ctypes.Structure):
    _fields_ = [("pattern", ctypes.c_int), ("dtype", ctypes.c_int), ("rows", _i32), ("cols", _i32),
                ("tile_r", _i32), ("tile_c", _i32), ("group_rows", _i32), ("nnz", _i32), ("rows_padded", _i32),
                ("ntiles", _i32), ("kparts", _i32), ("mask", _vp), ("idx", _vp), ("row_ptr", _vp),
                ("tile_col", _vp), ("row_map", _vp), ("part_row_ptr", _vp), ("values", _vp)]


class AttnDescC(ctypes.Structure):
    _fields_ = [("batch", _i32), ("seq_len", _i32), ("heads", _i32), ("d_model", _i32), ("dtype", ctypes.c_int),
                ("lengths_dev", _vp), ("causal", _i32), ("mode", ctypes.c_int), ("head_begin", _i32),
                ("head_end", _i32)]


class LayerC(ctypes.Structure):
    _fields_ = [("wq", PackedWeightC), ("wk", PackedWeightC), ("wv", PackedWeightC), ("wo", PackedWeightC),
                ("w1", PackedWeightC), ("w2", PackedWeightC), ("bq", _vp), ("bk", _vp), ("bv", _vp), ("bo", _vp),
                ("b1", _vp), ("b2", _vp), ("ln1_g", _vp), ("ln1_b", _vp), ("ln2_g", _vp), ("ln2_b", _vp),
                ("v_col", _vp), ("v_width", _vp), ("bv_packed", _vp), ("bo_folded", _vp)]


def _sig(name, res, args):
    f = getattr(_lib, name)
    f.restype = res
    f.argtypes = args
    return f


_lib.et_last_error.restype = ctypes.c_char_p
_lib.et_version.restype = ctypes.c_char_p
_sz_p = ctypes.POINTER(_sz)
_q = _sig("et_prune_pack_query", ctypes.c_int,
          [_i32, _i32, ctypes.c_int, ctypes.c_int, _f64, _i32, _i32, _i32, _vp, ctypes.POINTER(_i32)] + [_sz_p] * 8)
_pack = _sig("et_prune_pack", ctypes.c_int,
             [_vp, _i32, _i32, ctypes.c_int, ctypes.c_int, _f64, _i32, _i32, _i32, _vp,
              ctypes.POINTER(PackedWeightC), _vp, _sz, _vp])
_unpack = _sig("et_unpack", ctypes.c_int, [ctypes.POINTER(PackedWeightC), _vp, _vp])
_linear = _sig("et_linear_fwd", ctypes.c_int,
               [ctypes.POINTER(PackedWeightC), _vp, _i32, _vp, ctypes.c_int, _f32, _i32, _vp, _vp])
_ln = _sig("et_layernorm_fwd", ctypes.c_int,
           [_vp, ctypes.c_int, _i32, _i32, _i32, _vp, ctypes.c_int, _vp, ctypes.c_int, _vp, _vp, _f32, _vp, _vp, _vp])
_short_max = _sig("et_attn_short_max", _i32, [_i32])

SYMBOLS = ["et_last_error", "et_version", "et_prune_pack_query", "et_prune_pack", "et_unpack", "et_linear_fwd",
           "et_layernorm_fwd", "et_attn_short_max", "et_attn_core_fwd", "et_attention_workspace_size",
           "et_attention_fwd", "et_encoder_workspace_size", "et_encoder_fwd"]


def _check(st: int):
    if st != 0:
        raise EtError(st, _lib.et_last_error().decode())


def version() -> str:
    return _lib.et_version().decode()


def _stream(stream=None) -> int:
    s = stream if stream is not None else torch.cuda.current_stream()
    return s.cuda_stream


def _ptr(t):
    return None if t is None else t.data_ptr()


def dtype_code(dt) -> int:
    if isinstance(dt, int):
        return dt
    if isinstance(dt, torch.dtype):
        return {torch.float16: FP16, torch.bfloat16: BF16, torch.float32: FP32}[dt]
    return _DT[dt]


def torch_dtype(code) -> torch.dtype:
    return _TORCH_DT[dtype_code(code)]


# ------------------------------------------------------------------------------------------ packing
class Packed:
    """A packed pruned weight: the device buffers (torch tensors) + the C struct pointing at them."""

    def __init__(self, c: PackedWeightC, bufs: dict):
        self.c = c
        self.bufs = bufs

    @property
    def nnz(self):
        return self.c.nnz

    @property
    def rows_padded(self):
        return self.c.rows_padded

    def mask(self):
        return self.bufs["mask"]

    def units(self):
        c = self.c
        if c.pattern == PRUNE_TILE:
            return (c.rows // c.tile_r) * (c.cols // c.tile_c)
        return c.rows if c.pattern == PRUNE_ROW else c.cols

    def csr(self):
        """(row_ptr, col_idx) of a TILE weight (the bit-exact contract)."""
        p = self.c.rows // self.c.tile_r
        return self.bufs["row_ptr"][:p + 1], self.bufs["idx"][:self.c.nnz]

    def kept_index(self):
        return self.bufs["idx"][:self.c.nnz]


def prune_pack(W: torch.Tensor, pattern: str = "tile", ratio: float = 0.8, tile=(16, 16), group_rows: int = 0,
               mask_in: torch.Tensor | None = None, stream=None) -> Packed:
    """et_prune_pack: prune and pack a device weight W [rows, cols] (fp16 / bf16 / fp32)."""
    assert W.is_cuda and W.dim() == 2 and W.is_contiguous()
    rows, cols = W.shape
    dt = dtype_code(W.dtype)
    pat = _PAT[pattern] if isinstance(pattern, str) else pattern
    sizes = [_sz() for _ in range(8)]
    nnz = _i32()
    # with mask_in the kept count is its popcount: the size query needs a host copy of the bitmap
    host_mask = None
    if mask_in is not None:
        host_mask = mask_in.detach().to("cpu", torch.int32).contiguous()
    _check(_q(rows, cols, dt, pat, ratio, tile[0], tile[1], group_rows, _ptr(host_mask), ctypes.byref(nnz),
              *[ctypes.byref(s) for s in sizes]))
    names = ["mask", "idx", "row_ptr", "tile_col", "row_map", "part_row_ptr", "values", "ws"]
    dev = W.device
    bufs = {}
    for n, s in zip(names, sizes):
        nb = max(int(s.value), 16)
        bufs[n] = torch.empty(((nb + 15) // 16) * 16, dtype=torch.uint8, device=dev)
    c = PackedWeightC()
    c.mask = bufs["mask"].data_ptr()
    c.idx = bufs["idx"].data_ptr()
    c.row_ptr = bufs["row_ptr"].data_ptr()
    c.tile_col = bufs["tile_col"].data_ptr()
    c.row_map = bufs["row_map"].data_ptr()
    c.part_row_ptr = bufs["part_row_ptr"].data_ptr()
    c.values = bufs["values"].data_ptr() if sizes[6].value > 0 else None
    _check(_pack(W.data_ptr(), rows, cols, dt, pat, ratio, tile[0], tile[1], group_rows,
                 _ptr(mask_in), ctypes.byref(c), bufs["ws"].data_ptr(), bufs["ws"].numel(), _stream(stream)))
    del bufs["ws"]
    views = {
        "mask": bufs["mask"].view(torch.int32),
        "idx": bufs["idx"].view(torch.int32),
        "row_ptr": bufs["row_ptr"].view(torch.int32),
        "tile_col": bufs["tile_col"].view(torch.int32),
        "row_map": bufs["row_map"].view(torch.int32),
        "part_row_ptr": bufs["part_row_ptr"].view(torch.int32),
        "values": bufs["values"],
    }
    return Packed(c, views)


def unpack(w: Packed, stream=None) -> torch.Tensor:
    """et_unpack: dense W' = mask (.) W [rows, cols] from the packed values."""
    out = torch.empty(w.c.rows, w.c.cols, dtype=torch_dtype(w.c.dtype), device=w.bufs["values"].device)
    _check(_unpack(ctypes.byref(w.c), out.data_ptr(), _stream(stream)))
    return out


# ------------------------------------------------------------------------------------------ linear / LN
def linear_fwd(w: Packed, X: torch.Tensor, bias: torch.Tensor | None = None, epi: int = EPI_BIAS,
               scale: float = 1.0, scale_cols: int = 0, out: torch.Tensor | None = None, stream=None):
    """et_linear_fwd: Y = epilogue(X . W'^T + b) skipping pruned tiles."""
    M = X.shape[0]
    N = w.c.rows if w.c.pattern == PRUNE_TILE else w.c.rows_padded
    if out is None:
        if epi == EPI_F32:
            out = torch.empty(w.c.kparts, M, N, dtype=torch.float32, device=X.device)
        elif epi == EPI_PART16:
            out = torch.empty(w.c.kparts, M, N, dtype=X.dtype, device=X.device)
        else:
            out = torch.empty(M, N, dtype=X.dtype, device=X.device)
    _check(_linear(ctypes.byref(w.c), X.data_ptr(), M, _ptr(bias), epi, scale, scale_cols, out.data_ptr(),
                   _stream(stream)))
    return out


_gather = _sig("et_gather_cols", ctypes.c_int, [_vp, _i32, _i32, _vp, _i32, _i32, ctypes.c_int, _vp, _vp])
SYMBOLS += ["et_gather_cols"]


def gather_cols(A: torch.Tensor, idx: torch.Tensor, nk_pad: int, out: torch.Tensor | None = None, stream=None):
    """et_gather_cols: out[r, j] = A[r, idx[j]] (j < len(idx)), 0 up to nk_pad (X_adjusted)."""
    assert A.is_cuda and A.dim() == 2 and A.is_contiguous() and idx.dtype == torch.int32
    if out is None:
        out = torch.empty(A.shape[0], nk_pad, dtype=A.dtype, device=A.device)
    _check(_gather(A.data_ptr(), A.shape[0], A.shape[1], _ptr(idx) if idx.numel() else None, idx.numel(), nk_pad,
                   dtype_code(A.dtype), out.data_ptr(), _stream(stream)))
    return out


class ColLinear:
    """Column-pruned linear layer with X_adjusted (Fig. 5(b)).

    pack: et_prune_pack(ET_PRUNE_COL) selects the kept input columns (mask / ascending idx, bit-exact
    with the oracle); W_pruned = W[:, keep] is condensed by et_gather_cols, zero-padded to a multiple
    of 64 columns (the tile GEMM's K granule) and packed as a dense tile weight (ratio 0).
    forward: X_adjusted = et_gather_cols(X, keep) (one gather kernel), then the tcgen05 tile GEMM
    (et_linear_fwd) on the condensed operands.  Padded columns are zero on both sides (exact)."""

    def __init__(self, W: torch.Tensor, ratio: float, stream=None):
        self.rows, self.cols = W.shape
        self.sel = prune_pack(W, "col", ratio, stream=stream)
        self.nk = self.sel.nnz
        self.keep = self.sel.kept_index()
        self.nk_pad = max(64, (self.nk + 63) // 64 * 64)
        Wc = gather_cols(W, self.keep, self.nk_pad, stream=stream)
        self.dense = prune_pack(Wc, "tile", 0.0, stream=stream)

    def __call__(self, X: torch.Tensor, bias: torch.Tensor | None = None, epi: int = EPI_BIAS, stream=None,
                 x_adj: torch.Tensor | None = None):
        Xa = gather_cols(X, self.keep, self.nk_pad, out=x_adj, stream=stream)
        return linear_fwd(self.dense, Xa, bias, epi, stream=stream)


def layernorm_fwd(part: torch.Tensor, bias, resid, gamma, beta, eps: float, dtype, resid_dtype,
                  out_act=None, out_resid=None, stream=None):
    """et_layernorm_fwd: LN(sum(part) + bias + resid)."""
    nparts, M, N = part.shape
    _check(_ln(part.data_ptr(), dtype_code(part.dtype), nparts, M, N, _ptr(bias), dtype_code(dtype), _ptr(resid), dtype_code(resid_dtype),
               gamma.data_ptr(), beta.data_ptr(), eps, _ptr(out_act), _ptr(out_resid), _stream(stream)))
    return out_act, out_resid


def attn_short_max(d_k: int) -> int:
    return int(_short_max(d_k))


# ------------------------------------------------------------------------------------------ attention
_core = _sig("et_attn_core_fwd", ctypes.c_int,
             [ctypes.POINTER(AttnDescC), _vp, _i32, _i32, _i32, _i32, _vp, _vp, _i32, _f32, _vp, _i32, _vp, _vp])
_attn_ws = _sig("et_attention_workspace_size", ctypes.c_int,
                [ctypes.POINTER(AttnDescC), ctypes.POINTER(PackedWeightC), ctypes.POINTER(_sz)])
_attn = _sig("et_attention_fwd", ctypes.c_int,
             [ctypes.POINTER(AttnDescC), _vp] + [ctypes.POINTER(PackedWeightC)] * 4 + [_vp] * 6 +
             [_f32, _vp, _vp, _sz, _vp])
_enc_ws = _sig("et_encoder_workspace_size", ctypes.c_int,
               [ctypes.POINTER(AttnDescC), _i32, _i32, ctypes.c_int, ctypes.POINTER(LayerC), ctypes.POINTER(_sz)])
_enc = _sig("et_encoder_fwd", ctypes.c_int,
            [ctypes.POINTER(AttnDescC), _i32, _i32, ctypes.c_int, _f32, ctypes.c_int, ctypes.POINTER(LayerC), _vp,
             _vp, _vp, _sz, _vp])

_graph_create = _sig("et_encoder_graph_create", ctypes.c_int,
                     [ctypes.POINTER(AttnDescC), _i32, _i32, ctypes.c_int, _f32, ctypes.c_int, ctypes.POINTER(LayerC),
                      _vp, _vp, _vp, _sz, ctypes.POINTER(ctypes.c_void_p)])
_graph_launch = _sig("et_graph_launch", ctypes.c_int, [ctypes.c_void_p, _vp])
_graph_destroy = _sig("et_graph_destroy", ctypes.c_int, [ctypes.c_void_p])
SYMBOLS += ["et_encoder_graph_create", "et_graph_launch", "et_graph_destroy"]


def attn_desc(batch, seq_len, heads, d_model, dtype, lengths=None, causal=False, mode="auto",
              head_begin=0, head_end=None) -> AttnDescC:
    d = AttnDescC()
    d.batch, d.seq_len, d.heads, d.d_model = batch, seq_len, heads, d_model
    d.dtype = dtype_code(dtype)
    d.lengths_dev = _ptr(lengths)
    d.causal = 1 if causal else 0
    d.mode = _MODE[mode] if isinstance(mode, str) else mode
    d.head_begin = head_begin
    d.head_end = heads if head_end is None else head_end
    return d


def attn_core_fwd(qkv: torch.Tensor, batch: int, seq_len: int, heads: int, d_model: int, q_off: int, k_off: int,
                  v_off: int, lengths=None, causal=False, mode="auto", scale: float = 1.0, v_col=None,
                  v_width=None, v_width_max: int = 0, Z=None, z_map=None, stream=None):
    """et_attn_core_fwd: on-the-fly attention on a [batch*seq_len, ld] QKV buffer."""
    d = attn_desc(batch, seq_len, heads, d_model, qkv.dtype, lengths, causal, mode)
    if Z is None:
        Z = torch.zeros(batch * seq_len, d_model, dtype=qkv.dtype, device=qkv.device)
    _check(_core(ctypes.byref(d), qkv.data_ptr(), qkv.stride(0), q_off, k_off, v_off, _ptr(v_col), _ptr(v_width),
                 v_width_max, scale, Z.data_ptr(), Z.stride(0), _ptr(z_map), _stream(stream)))
    return Z


_partial_bytes = _sig("et_attn_partial_scores_bytes", ctypes.c_int, [ctypes.POINTER(AttnDescC), ctypes.POINTER(_sz)])
_partial = _sig("et_attn_partial_fwd", ctypes.c_int,
                [ctypes.POINTER(AttnDescC), _vp, _i32, _i32, _i32, _i32, _f32, _vp, _i32, _vp, _sz, _vp])
SYMBOLS += ["et_attn_partial_scores_bytes", "et_attn_partial_fwd"]


def attn_partial_scores_bytes(batch: int, seq_len: int, heads: int, d_model: int, dtype="fp16",
                              head_begin: int = 0, head_end: int | None = None) -> int:
    d = attn_desc(batch, seq_len, heads, d_model, dtype, head_begin=head_begin, head_end=head_end)
    n = _sz(0)
    _check(_partial_bytes(ctypes.byref(d), ctypes.byref(n)))
    return int(n.value)


def attn_partial_fwd(qkv: torch.Tensor, batch: int, seq_len: int, heads: int, d_model: int, q_off: int, k_off: int,
                     v_off: int, lengths=None, causal=False, scale: float = 1.0, Z=None, scores=None, stream=None):
    """et_attn_partial_fwd: the paper's partial OTF (Fig. 8) — Q.K^T materialised
    in a 16-bit score buffer, then mask + softmax + x V per row.  Returns (Z, scores)."""
    d = attn_desc(batch, seq_len, heads, d_model, qkv.dtype, lengths, causal)
    if Z is None:
        Z = torch.zeros(batch * seq_len, d_model, dtype=qkv.dtype, device=qkv.device)
    if scores is None:
        nbytes = attn_partial_scores_bytes(batch, seq_len, heads, d_model, qkv.dtype)
        scores = torch.empty(nbytes // 2, dtype=qkv.dtype, device=qkv.device)
    _check(_partial(ctypes.byref(d), qkv.data_ptr(), qkv.stride(0), q_off, k_off, v_off, scale, Z.data_ptr(),
                    Z.stride(0), scores.data_ptr(), scores.numel() * scores.element_size(), _stream(stream)))
    return Z, scores


# ------------------------------------------------------------------------------------------ layers
class Layer:
    """One packed encoder layer: six packed weights + device biases / LayerNorm parameters."""

    def __init__(self, packed: dict, dense: dict):
        self.packed = packed      # name -> Packed
        self.dense = dense        # biases (dtype) and LN params (fp32) as device tensors
        c = LayerC()
        for n in ("wq", "wk", "wv", "wo", "w1", "w2"):
            setattr(c, n, packed[n].c)
        for n in ("bq", "bk", "bv", "bo", "b1", "b2", "ln1_g", "ln1_b", "ln2_g", "ln2_b"):
            setattr(c, n, dense[n].data_ptr())
        for n in ("v_col", "v_width", "bv_packed", "bo_folded"):   # et_vprep output (attention-aware), optional
            setattr(c, n, dense[n].data_ptr() if n in dense else None)
        self.c = c


_vprep = _sig("et_vprep", ctypes.c_int,
              [ctypes.POINTER(PackedWeightC), ctypes.POINTER(PackedWeightC), _vp, _vp, _i32, _i32, ctypes.c_int,
               _vp, _vp, _vp, _vp, _vp])
SYMBOLS += ["et_vprep"]


def vprep(wv: "Packed", wo: "Packed", bv: torch.Tensor, bo: torch.Tensor | None, heads: int, d_model: int,
          dtype="fp16", stream=None) -> dict:
    """et_vprep: an attention-aware layer's weight-only data (per-head packed V columns / widths, packed
    b_V, folded b_O'), computed once instead of on every forward."""
    tdt = torch_dtype(dtype)
    out = {"v_col": torch.empty(heads, dtype=torch.int32, device="cuda"),
           "v_width": torch.empty(heads, dtype=torch.int32, device="cuda"),
           "bv_packed": torch.empty(max(wv.c.rows_padded, 1), dtype=tdt, device="cuda"),
           "bo_folded": torch.empty(d_model, dtype=tdt, device="cuda")}
    _check(_vprep(ctypes.byref(wv.c), ctypes.byref(wo.c), bv.data_ptr(), _ptr(bo), heads, d_model, dtype_code(dtype),
                  out["v_col"].data_ptr(), out["v_width"].data_ptr(), out["bv_packed"].data_ptr(),
                  out["bo_folded"].data_ptr(), _stream(stream)))
    return out


def pack_layer(raw: dict, scheme: str, ratio: float, heads: int, dtype="fp16", stream=None, precompute=True) -> Layer:
    """Prune + pack the six matrices of one layer (pattern per scheme: PAPER.md line 107, 317).

    raw: name -> float32 numpy/torch array holding storage-dtype values (et_synth.make_layer).
    precompute: for a row-pruned W_V, compute the attention-aware layer data once (et_vprep) so the
    forward skips it; False leaves it to every forward (both paths are tested)."""
    tdt = torch_dtype(dtype)
    dev = torch.device("cuda")
    packed, dense = {}, {}
    d_model = raw["wq"].shape[0]
    for n in ("wq", "wk", "wv", "wo", "w1", "w2"):
        W = torch.as_tensor(raw[n]).to(dev).to(tdt).contiguous()
        if scheme == "none":
            pat, r = "tile", 0.0
        elif scheme == "attention-aware" and n == "wv":
            pat, r = "row", ratio
        else:
            pat, r = "tile", ratio
        packed[n] = prune_pack(W, pat, r, (16, 16), group_rows=d_model // heads if pat == "row" else 0,
                               stream=stream)
    for n in ("bq", "bk", "bv", "bo", "b1", "b2"):
        dense[n] = torch.as_tensor(raw[n]).to(dev).to(tdt).contiguous()
    for n in ("ln1_g", "ln1_b", "ln2_g", "ln2_b"):
        dense[n] = torch.as_tensor(raw[n]).to(dev).to(torch.float32).contiguous()
    if precompute and packed["wv"].c.pattern == PRUNE_ROW and dtype in ("fp16", "bf16"):
        dense.update(vprep(packed["wv"], packed["wo"], dense["bv"], dense["bo"], heads, d_model, dtype, stream))
    return Layer(packed, dense)


def attention_workspace_size(layer: Layer, batch: int, seq_len: int, heads: int, d_model: int, dtype,
                             head_range=None) -> int:
    """et_attention_workspace_size (bytes)."""
    h0, h1 = head_range or (0, heads)
    d = attn_desc(batch, seq_len, heads, d_model, dtype, head_begin=h0, head_end=h1)
    nb = _sz()
    _check(_attn_ws(ctypes.byref(d), ctypes.byref(layer.packed["wv"].c), ctypes.byref(nb)))
    return int(nb.value)


def attention_fwd(X: torch.Tensor, layer: Layer, batch: int, seq_len: int, heads: int, lengths=None,
                  causal=False, mode="auto", ln: bool = True, ln_eps: float = 1e-12, out=None, stream=None,
                  head_range=None, workspace: torch.Tensor | None = None):
    """et_attention_fwd: LN(X + SelfAttn(X)) (ln=True) or SelfAttn(X).

    head_range=(h0, h1) != (0, heads): head-parallel partial (Eq. 4) — `layer` holds the rank's
    slices (dist.pack_head_slice), no LN, out is FP32 [M, d_model]."""
    d_model = X.shape[1]
    h0, h1 = head_range or (0, heads)
    hp = (h0, h1) != (0, heads)
    d = attn_desc(batch, seq_len, heads, d_model, X.dtype, lengths, causal, mode, head_begin=h0, head_end=h1)
    P, D = layer.packed, layer.dense
    if workspace is None:
        workspace = torch.empty(attention_workspace_size(layer, batch, seq_len, heads, d_model, X.dtype, (h0, h1)),
                                dtype=torch.uint8, device=X.device)
    if out is None:
        out = torch.empty(X.shape, dtype=torch.float32 if hp else X.dtype, device=X.device)
    use_ln = ln and not hp
    _check(_attn(ctypes.byref(d), X.data_ptr(), ctypes.byref(P["wq"].c), ctypes.byref(P["wk"].c),
                 ctypes.byref(P["wv"].c), ctypes.byref(P["wo"].c), D["bq"].data_ptr(), D["bk"].data_ptr(),
                 D["bv"].data_ptr(), D["bo"].data_ptr(), D["ln1_g"].data_ptr() if use_ln else None,
                 D["ln1_b"].data_ptr() if use_ln else None, ln_eps, out.data_ptr(), workspace.data_ptr(),
                 workspace.numel(), _stream(stream)))
    return out


# ------------------------------------------------------------------- pre-computed operator (Eq. 5)
_prevo = _sig("et_precompute_vo", ctypes.c_int,
              [_vp, _vp, _vp, _vp, _vp, _i32, _i32, _i32, ctypes.c_int, _vp, _vp, _vp])
_pre_ws = _sig("et_attention_pre_workspace_size", ctypes.c_int, [ctypes.POINTER(AttnDescC), _i32, ctypes.POINTER(_sz)])
_pre = _sig("et_attention_pre_fwd", ctypes.c_int,
            [ctypes.POINTER(AttnDescC), _vp] + [ctypes.POINTER(PackedWeightC)] * 3 + [_vp, _i32, _vp, _vp, _vp, _vp, _vp,
                                                                                    _f32, _vp, _vp, _sz, _vp])
SYMBOLS += ["et_precompute_vo", "et_attention_pre_workspace_size", "et_attention_pre_fwd"]


class PreLayer:
    """Attention block in the pre-computed form (Fig. 3(b)): W_Q / W_K tile
    pruned, W_O row pruned (kept output features), W_V dense; W_VO = ||_h W_V,h^T W_O,h^T and the folded
    bias b' computed on the device by et_precompute_vo, W_VO packed as a dense tile weight."""

    def __init__(self, raw: dict, ratio: float, heads: int, dtype="fp16", stream=None):
        tdt = torch_dtype(dtype)
        dev = torch.device("cuda")
        d = raw["wq"].shape[0]
        self.heads, self.d_model, self.dtype = heads, d, tdt
        T = {n: torch.as_tensor(raw[n]).to(dev).to(tdt).contiguous() for n in ("wq", "wk", "wv", "wo")}
        self.wq = prune_pack(T["wq"], "tile", ratio, stream=stream)
        self.wk = prune_pack(T["wk"], "tile", ratio, stream=stream)
        self.wo_sel = prune_pack(T["wo"], "row", ratio, stream=stream)    # kept W_O rows = output features
        self.n_kept = int(self.wo_sel.c.nnz)
        self.kept = self.wo_sel.kept_index().contiguous()
        self.Dv = (self.n_kept + 15) // 16 * 16
        self.dense = {n: torch.as_tensor(raw[n]).to(dev).to(tdt).contiguous() for n in ("bq", "bk", "bv", "bo")}
        self.dense["ln1_g"] = torch.as_tensor(raw["ln1_g"]).to(dev).to(torch.float32).contiguous()
        self.dense["ln1_b"] = torch.as_tensor(raw["ln1_b"]).to(dev).to(torch.float32).contiguous()
        self.wvo_dense = torch.empty(heads * self.Dv, d, dtype=tdt, device=dev)
        self.bias_fold = torch.empty(d, dtype=tdt, device=dev)
        _check(_prevo(T["wv"].data_ptr(), T["wo"].data_ptr(), self.dense["bv"].data_ptr(), self.dense["bo"].data_ptr(),
                      self.kept.data_ptr(), self.n_kept, heads, d, dtype_code(tdt), self.wvo_dense.data_ptr(),
                      self.bias_fold.data_ptr(), _stream(stream)))
        self.wvo = prune_pack(self.wvo_dense, "tile", 0.0, stream=stream)

    def workspace_size(self, batch: int, seq_len: int) -> int:
        d = attn_desc(batch, seq_len, self.heads, self.d_model, self.dtype)
        nb = _sz()
        _check(_pre_ws(ctypes.byref(d), self.n_kept, ctypes.byref(nb)))
        return int(nb.value)

    def __call__(self, X: torch.Tensor, batch: int, seq_len: int, lengths=None, causal=False, ln: bool = True,
                 ln_eps: float = 1e-12, out=None, workspace=None, stream=None):
        """et_attention_pre_fwd: LN(X + SelfAttn(X)) (ln=True) or SelfAttn(X)."""
        d = attn_desc(batch, seq_len, self.heads, self.d_model, X.dtype, lengths, causal)
        if workspace is None:
            workspace = torch.empty(self.workspace_size(batch, seq_len), dtype=torch.uint8, device=X.device)
        if out is None:
            out = torch.empty(X.shape, dtype=X.dtype, device=X.device)
        D = self.dense
        _check(_pre(ctypes.byref(d), X.data_ptr(), ctypes.byref(self.wq.c), ctypes.byref(self.wk.c),
                    ctypes.byref(self.wvo.c), self.kept.data_ptr(), self.n_kept, D["bq"].data_ptr(), D["bk"].data_ptr(),
                    self.bias_fold.data_ptr(), D["ln1_g"].data_ptr() if ln else None,
                    D["ln1_b"].data_ptr() if ln else None, ln_eps, out.data_ptr(), workspace.data_ptr(),
                    workspace.numel(), _stream(stream)))
        return out


class Encoder:
    """A packed encoder stack bound to a fixed problem shape: owns the C layer array and workspace."""

    def __init__(self, layers: list, batch: int, seq_len: int, heads: int, d_ff: int, act="gelu", ln_eps=1e-12,
                 dtype="fp16", resid_dtype=None, causal=False, mode="auto", lengths=None):
        self.layers = layers
        self.arr = (LayerC * len(layers))(*[l.c for l in layers])
        d_model = layers[0].packed["wq"].c.rows
        self.d_model = d_model
        self.desc = attn_desc(batch, seq_len, heads, d_model, dtype, lengths, causal, mode)
        self.lengths = lengths
        self.d_ff, self.act, self.eps = d_ff, _ACT[act], ln_eps
        # residual stream dtype (reading C-22): the operand dtype unless given (FP32 is the other choice)
        self.dtype = dtype_code(dtype)
        self.resid_dtype = self.dtype if resid_dtype is None else dtype_code(resid_dtype)
        nb = _sz()
        _check(_enc_ws(ctypes.byref(self.desc), len(layers), d_ff, self.resid_dtype, self.arr, ctypes.byref(nb)))
        self.ws = torch.empty(nb.value, dtype=torch.uint8, device="cuda")

    def set_lengths(self, lengths):
        self.lengths = lengths
        self.desc.lengths_dev = _ptr(lengths)

    def __call__(self, X: torch.Tensor, out: torch.Tensor | None = None, stream=None) -> torch.Tensor:
        """et_encoder_fwd: X, out [batch*seq_len, d_model] in resid_dtype."""
        if out is None:
            out = torch.empty_like(X)
        _check(_enc(ctypes.byref(self.desc), len(self.layers), self.d_ff, self.act, self.eps, self.resid_dtype,
                    self.arr, X.data_ptr(), out.data_ptr(), self.ws.data_ptr(), self.ws.numel(), _stream(stream)))
        return out


    def capture(self, X: torch.Tensor, out: torch.Tensor) -> "Graph":
        """et_encoder_graph_create: the whole forward on (X, out) as one CUDA graph (X is read in place
        at every launch; X, out, the workspace and the layers must outlive the graph)."""
        g = ctypes.c_void_p()
        _check(_graph_create(ctypes.byref(self.desc), len(self.layers), self.d_ff, self.act, self.eps,
                             self.resid_dtype, self.arr, X.data_ptr(), out.data_ptr(), self.ws.data_ptr(),
                             self.ws.numel(), ctypes.byref(g)))
        return Graph(g, keep=(self, X, out))


class Graph:
    """A captured forward (et_graph*): launch() enqueues one replay on the current stream."""

    def __init__(self, handle: ctypes.c_void_p, keep=()):
        self.h = handle
        self._keep = keep

    def launch(self, stream=None):
        _check(_graph_launch(self.h, _stream(stream)))

    def __del__(self):
        if getattr(self, "h", None) is not None and self.h.value:
            _graph_destroy(self.h)
            self.h = None


def encoder_fwd(X: torch.Tensor, layers: list, batch: int, seq_len: int, heads: int, d_ff: int, **kw):
    """One-shot et_encoder_fwd (allocates the workspace; use Encoder for repeated calls)."""
    return Encoder(layers, batch, seq_len, heads, d_ff, **kw)(X)


# ------------------------------------------------------------------------------------------ tracing
_sig("et_trace_begin", ctypes.c_int, [_i32, _vp])
_sig("et_trace_end", ctypes.c_int, [ctypes.POINTER(_i32)])
_sig("et_trace_get", ctypes.c_int, [_i32, ctypes.POINTER(_i32), ctypes.POINTER(_f32)])
_sig("et_launch_count", ctypes.c_int64, [])
if hasattr(_lib, "et_diag_gemm_timeline"):
    _sig("et_diag_gemm_timeline", ctypes.c_int, [_vp])
SYMBOLS += ["et_trace_begin", "et_trace_end", "et_trace_get", "et_launch_count"]
