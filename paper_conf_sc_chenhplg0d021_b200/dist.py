"""Multi-GPU plumbing (sequences — and heads, and rows — are independent units).

Batch sharding: rank r of N processes owns a contiguous slice of the global batch; there is no
collective on the data path.  The only collectives are outside the timed region: a barrier and a
MAX all-reduce of each rank's device time (throughput = all sequences / slowest rank), plus a
check that every rank packed bit-identical masks.  Works with the nccl (GPU) and gloo (CPU tests)
backends of torch.distributed.
"""
from __future__ import annotations

import hashlib
import os

import torch


def env_rank_world():
    return int(os.environ.get("RANK", "0")), int(os.environ.get("WORLD_SIZE", "1")), \
        int(os.environ.get("LOCAL_RANK", "0"))


def shard_range(global_batch: int, world: int, rank: int) -> tuple[int, int]:
    """Contiguous, near-equal shard [b0, b1) of the global batch for `rank` (sizes differ by <= 1)."""
    if world <= 0 or not (0 <= rank < world):
        raise ValueError("bad world / rank")
    base, rem = divmod(global_batch, world)
    b0 = rank * base + min(rank, rem)
    return b0, b0 + base + (1 if rank < rem else 0)


def max_over_ranks(value: float, device=None) -> float:
    """MAX all-reduce of a scalar (no-op without an initialised process group)."""
    import torch.distributed as dist
    if not (dist.is_available() and dist.is_initialized()):
        return float(value)
    t = torch.tensor([float(value)], dtype=torch.float64, device=device or "cpu")
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def mask_digest(words) -> str:
    """Digest of a packed mask (bytes-like / tensor / ndarray) for cross-rank agreement checks."""
    if isinstance(words, torch.Tensor):
        words = words.detach().cpu().numpy()
    return hashlib.sha256(memoryview(words).tobytes()).hexdigest()


def layers_digest(layers) -> str:
    """Digest over every packed mask of every layer (et.Layer objects): batch-sharded ranks pack the same
    weights deterministically, and bench.py checks that the digests agree before timing."""
    h = hashlib.sha256()
    for lay in layers:
        for n in ("wq", "wk", "wv", "wo", "w1", "w2"):
            h.update(mask_digest(lay.packed[n].mask()).encode())
    return h.hexdigest()


def all_equal_across_ranks(digest: str) -> bool:
    """True iff every rank passed the same digest."""
    import torch.distributed as dist
    if not (dist.is_available() and dist.is_initialized()):
        return True
    out = [None] * dist.get_world_size()
    dist.all_gather_object(out, digest)
    return all(o == out[0] for o in out)


# ------------------------------------------------------------------------------------------------
# Head-parallel mode (optional; Megatron-style split of Eq. 4, PAPER.md line 119:
# Output = sum_h Z_h W_O,h^T).  Rank r owns heads [h0, h1): the rows h0*d_k .. h1*d_k of W_Q, W_K,
# W_V (and their biases) and the same columns of W_O.  Each rank computes its partial sum with
# et_attention_fwd on those slices, the partials are summed by an all-reduce (NCCL over NVLink on
# GPUs; gloo in the CPU tests), then residual + LayerNorm and the (replicated) FFN follow.
# Pruning stays per matrix (reading C-3): every rank packs the FULL matrices deterministically,
# restricts the masks to its slices and packs the slices with that mask (et_prune_pack mask_in).
# ------------------------------------------------------------------------------------------------

def head_range(heads: int, world: int, rank: int) -> tuple[int, int]:
    """Contiguous near-equal head range [h0, h1) of `rank` (H = 12 over 8 ranks: 2/1 imbalance)."""
    if world > heads:
        raise ValueError(f"head-parallel needs world <= heads ({world} > {heads})")
    return shard_range(heads, world, rank)


def mask_to_bits(words: torch.Tensor, n: int) -> torch.Tensor:
    """Bitmap (int32 words, unit t at bit t % 32 of word t // 32; include/et.h) -> bool [n]."""
    w = words.to(torch.int64).reshape(-1)[: (n + 31) // 32] & 0xFFFFFFFF
    bits = (w.unsqueeze(1) >> torch.arange(32, device=w.device)) & 1
    return bits.reshape(-1)[:n].to(torch.bool)


def bits_to_mask(bits: torch.Tensor) -> torch.Tensor:
    """bool [n] -> bitmap (int32 words), the inverse of mask_to_bits."""
    n = bits.numel()
    nw = (n + 31) // 32
    b = torch.zeros(nw * 32, dtype=torch.int64, device=bits.device)
    b[:n] = bits.reshape(-1).to(torch.int64)
    w = (b.reshape(nw, 32) << torch.arange(32, device=bits.device)).sum(dim=1)
    return torch.where(w >= 2 ** 31, w - 2 ** 32, w).to(torch.int32)


def tile_mask_rows(words: torch.Tensor, p: int, q: int, r0: int, r1: int) -> torch.Tensor:
    """Mask of the tile-row slice [r0, r1) of a p x q tile grid (row slice of the matrix)."""
    return bits_to_mask(mask_to_bits(words, p * q).reshape(p, q)[r0:r1].reshape(-1))


def tile_mask_cols(words: torch.Tensor, p: int, q: int, c0: int, c1: int) -> torch.Tensor:
    """Mask of the tile-column slice [c0, c1) of a p x q tile grid (column slice of the matrix)."""
    return bits_to_mask(mask_to_bits(words, p * q).reshape(p, q)[:, c0:c1].reshape(-1))


def unit_mask_range(words: torch.Tensor, n: int, u0: int, u1: int) -> torch.Tensor:
    """Mask of the unit range [u0, u1) of a ROW / COL pattern over n units."""
    return bits_to_mask(mask_to_bits(words, n)[u0:u1])


class SliceLayer:
    """A rank's head slice of one layer: packed W_Q/W_K/W_V row slices and the W_O column slice, the
    matching bias slices and the full b_O (the library adds it only on the rank owning head 0)."""

    def __init__(self, packed: dict, dense: dict, h0: int, h1: int):
        self.packed, self.dense, self.h0, self.h1 = packed, dense, h0, h1


def pack_head_slice(raw: dict, full, heads: int, h0: int, h1: int, dtype="fp16") -> SliceLayer:
    """Pack the head slice [h0, h1) of a layer with the masks of the full packed layer `full`
    (a paper_conf_sc_chenhplg0d021_b200.Layer packed from the same `raw`)."""
    import paper_conf_sc_chenhplg0d021_b200 as et
    tdt = et.torch_dtype(dtype)
    d = raw["wq"].shape[0]
    dk = d // heads
    a, b = h0 * dk, h1 * dk
    packed, dense = {}, {}
    for n in ("wq", "wk", "wv"):
        fw = full.packed[n]
        W = torch.as_tensor(raw[n]).to("cuda").to(tdt)[a:b].contiguous()
        if fw.c.pattern == et.PRUNE_ROW:
            m = unit_mask_range(fw.mask(), d, a, b)
            packed[n] = et.prune_pack(W, "row", 0.0, (16, 16), group_rows=dk, mask_in=m.to("cuda"))
        else:
            m = tile_mask_rows(fw.mask(), d // 16, d // 16, a // 16, b // 16)
            packed[n] = et.prune_pack(W, "tile", 0.0, (16, 16), mask_in=m.to("cuda"))
    fo = full.packed["wo"]
    Wo = torch.as_tensor(raw["wo"]).to("cuda").to(tdt)[:, a:b].contiguous()
    packed["wo"] = et.prune_pack(Wo, "tile", 0.0, (16, 16),
                                 mask_in=tile_mask_cols(fo.mask(), d // 16, d // 16, a // 16, b // 16).to("cuda"))
    for n in ("bq", "bk", "bv"):
        dense[n] = full.dense[n][a:b].contiguous()
    dense["bo"] = full.dense["bo"]
    return SliceLayer(packed, dense, h0, h1)


class HeadParallelEncoder:
    """Post-LN encoder stack in head-parallel mode on this rank (one process per GPU).

    Per layer: et_attention_fwd on the FULL packed weights with the rank's head range (the library
    slices them) -> FP32 partial [M, d] -> all-reduce(sum) over `group` (skipped at
    world size 1) -> et_layernorm_fwd (residual + LN, Y1) -> FFN1 / FFN2 (et_linear_fwd, replicated on
    every rank) -> et_layernorm_fwd (Y2).  Every rank processes the whole batch; the outputs are
    identical on all ranks.  Residual stream in the operand dtype.  `capture()` records the whole
    forward, NCCL all-reduces included, as one CUDA graph (torch.cuda.graph on the current stream).
    slices=True: the caller-sliced form instead (dist.pack_head_slice re-packs each rank's slices)."""

    def __init__(self, raws: list, full_layers: list, heads: int, batch: int, seq_len: int, d_ff: int,
                 act="gelu", ln_eps=1e-12, dtype="fp16", causal=False, mode="auto", lengths=None,
                 rank: int = 0, world: int = 1, group=None, slices: bool = False):
        import paper_conf_sc_chenhplg0d021_b200 as et
        self.et = et
        self.h0, self.h1 = head_range(heads, world, rank)
        self.full = full_layers
        self.slices = ([pack_head_slice(r, f, heads, self.h0, self.h1, dtype) for r, f in zip(raws, full_layers)]
                       if slices else list(full_layers))
        self.heads, self.batch, self.seq_len, self.d_ff = heads, batch, seq_len, d_ff
        self.act_epi = et.EPI_BIAS_GELU if act == "gelu" else et.EPI_BIAS_RELU
        self.eps, self.dtype, self.causal, self.mode, self.lengths = ln_eps, dtype, causal, mode, lengths
        self.world, self.group = world, group
        d = raws[0]["wq"].shape[0]
        self.d_model = d
        M = batch * seq_len
        tdt = et.torch_dtype(dtype)
        nb = max(et.attention_workspace_size(s, batch, seq_len, heads, d, dtype, (self.h0, self.h1))
                 for s in self.slices)
        self.ws = torch.empty(nb, dtype=torch.uint8, device="cuda")
        full_range = (self.h0, self.h1) == (0, heads)   # one rank owns every head: plain block output
        self.part = torch.empty(M, d, dtype=tdt if full_range else torch.float32, device="cuda")
        self.y1 = torch.empty(M, d, dtype=tdt, device="cuda")
        self.u = torch.empty(M, d_ff, dtype=tdt, device="cuda")
        kp = full_layers[0].packed["w2"].c.kparts
        self.p2 = torch.empty(kp, M, d, dtype=tdt if dtype == "fp16" else torch.float32, device="cuda")
        self.p2_epi = et.EPI_PART16 if dtype == "fp16" else et.EPI_F32

    def _allreduce(self, t: torch.Tensor):
        import torch.distributed as dist
        if self.group is not None or (self.world > 1 and dist.is_available() and dist.is_initialized()):
            dist.all_reduce(t, op=dist.ReduceOp.SUM, group=self.group)

    def attn_partial(self, l: int, cur: torch.Tensor) -> torch.Tensor:
        """This rank's O-projection partial of layer l (FP32 [M, d]; the full SelfAttn output in the
        operand dtype when the rank owns every head)."""
        return self.et.attention_fwd(cur, self.slices[l], self.batch, self.seq_len, self.heads, self.lengths,
                                     self.causal, self.mode, ln=False, out=self.part,
                                     head_range=(self.h0, self.h1), workspace=self.ws)

    def finish_layer(self, l: int, cur: torch.Tensor, attn: torch.Tensor, dst: torch.Tensor):
        """Given the all-reduced attention output: Y1 = LN(cur + attn); Y2 = LN(Y1 + FFN(Y1)) -> dst."""
        et, f = self.et, self.full[l]
        D = f.dense
        et.layernorm_fwd(attn.unsqueeze(0), None, cur, D["ln1_g"], D["ln1_b"], self.eps, self.dtype, self.dtype,
                         out_act=self.y1)
        et.linear_fwd(f.packed["w1"], self.y1, D["b1"], epi=self.act_epi, out=self.u)
        et.linear_fwd(f.packed["w2"], self.u, None, epi=self.p2_epi, out=self.p2)
        et.layernorm_fwd(self.p2, D["b2"], self.y1, D["ln2_g"], D["ln2_b"], self.eps, self.dtype, self.dtype,
                         out_act=dst)

    def capture(self, X: torch.Tensor, out: torch.Tensor):
        """The whole forward on (X, out) as one CUDA graph, the per-layer NCCL all-reduce included
        (torch captures NCCL collectives on the capture stream); replay with g.replay()."""
        self._tmp = torch.empty_like(X) if len(self.full) > 1 else None
        s = torch.cuda.Stream()
        s.wait_stream(torch.cuda.current_stream())
        with torch.cuda.stream(s):   # warm-up on a side stream (NCCL communicator init, lazy state)
            self(X, out)
        torch.cuda.current_stream().wait_stream(s)
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g):
            self(X, out)
        return g

    def __call__(self, X: torch.Tensor, out: torch.Tensor | None = None) -> torch.Tensor:
        cur = X
        if out is None:
            out = torch.empty_like(X)
        tmp = getattr(self, "_tmp", None)
        if tmp is None and len(self.full) > 1:
            tmp = self._tmp = torch.empty_like(X)
        for l in range(len(self.full)):
            part = self.attn_partial(l, cur)
            self._allreduce(part)                                   # NCCL over NVLink on GPUs
            dst = out if (len(self.full) - 1 - l) % 2 == 0 else tmp   # the last layer lands in out
            self.finish_layer(l, cur, part, dst)
            cur = dst
        return out
