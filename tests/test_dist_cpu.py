"""Multi-process host logic of batch sharding on CPU (gloo, world_size 2): shards partition the
global batch, the MAX reduction picks the slowest rank, every rank agrees on packed-mask digests."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_sc_chenhplg0d021_b200.dist import (all_equal_across_ranks, mask_digest, max_over_ranks,
                                                   shard_range)


def test_shard_range_partitions_the_batch():
    for gb in (1, 7, 32, 256):
        for world in (1, 2, 3, 8):
            if world > gb:
                continue
            spans = [shard_range(gb, world, r) for r in range(world)]
            assert spans[0][0] == 0 and spans[-1][1] == gb
            assert all(a[1] == b[0] for a, b in zip(spans, spans[1:]))
            sizes = [b - a for a, b in spans]
            assert max(sizes) - min(sizes) <= 1
    with pytest.raises(ValueError):
        shard_range(8, 2, 2)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        b0, b1 = shard_range(64, world, rank)
        t = max_over_ranks(1.0 + rank)                      # rank 1 is the slowest
        from oracle.prune import prune_tile                 # same weights on every rank -> same mask
        from et_synth import make_matrix
        W = make_matrix(5, (64, 64), 0.02, "fp16")
        dig = mask_digest(prune_tile(W.astype(np.float64), 0.8)["mask"])
        ok = all_equal_across_ranks(dig)
        bad = all_equal_across_ranks(dig + ("x" if rank == 1 else ""))
        q.put((rank, b0, b1, t, ok, bad))
    finally:
        dist.destroy_process_group()


def test_gloo_world2_sharding_and_reductions():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = sorted(q.get(timeout=120) for _ in procs)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert [(r[1], r[2]) for r in res] == [(0, 32), (32, 64)]
    assert all(r[3] == 2.0 for r in res)                  # MAX over ranks
    assert all(r[4] for r in res) and not any(r[5] for r in res)


# ---------------------------------------------------------------- head-parallel mode
from paper_conf_sc_chenhplg0d021_b200.dist import (bits_to_mask, head_range, mask_to_bits, tile_mask_cols,
                                                   tile_mask_rows, unit_mask_range)


def test_head_range_partitions_heads():
    for H in (1, 4, 12):
        for world in range(1, H + 1):
            spans = [head_range(H, world, r) for r in range(world)]
            assert spans[0][0] == 0 and spans[-1][1] == H
            assert all(a[1] == b[0] for a, b in zip(spans, spans[1:]))
    assert [head_range(12, 8, r) for r in range(8)][:4] == [(0, 2), (2, 4), (4, 6), (6, 8)]
    with pytest.raises(ValueError):
        head_range(4, 5, 0)


def test_mask_slices_equal_the_global_selection_restricted():
    """A rank's slice keeps exactly the tiles / rows the whole-matrix ranking kept (reading C-3):
    the sliced bitmaps equal the oracle's bitmap of the restricted keep grid, bit for bit."""
    from et_synth import make_matrix
    from oracle.prune import bitmap, prune_row, prune_tile
    W = make_matrix(11, (128, 128), 0.02, "fp16").astype(np.float64)
    rec = prune_tile(W, 0.8)
    words = torch.from_numpy(rec["mask"].view(np.int32).copy())
    assert torch.equal(bits_to_mask(mask_to_bits(words, 64)), words)
    g = rec["tile_mask"]
    for r0, r1 in ((0, 2), (2, 6), (6, 8)):
        assert np.array_equal(tile_mask_rows(words, 8, 8, r0, r1).numpy().view(np.uint32), bitmap(g[r0:r1]))
        assert np.array_equal(tile_mask_cols(words, 8, 8, r0, r1).numpy().view(np.uint32), bitmap(g[:, r0:r1]))
    rr = prune_row(W, 0.8)
    rw = torch.from_numpy(rr["mask"].view(np.int32).copy())
    for a, b in ((0, 32), (32, 96), (96, 128)):
        assert np.array_equal(unit_mask_range(rw, 128, a, b).numpy().view(np.uint32), bitmap(rr["keep"][a:b]))


def _hp_case():
    from et_synth import CONFIGS, make_layer, make_lengths, make_x
    from oracle import encoder as oe
    cfg = CONFIGS["C2"].with_(d_model=128, heads=4, d_ff=512, seq_len=16, batch=2, ratio=0.5)
    raw = make_layer(cfg, 0)
    w = oe.prune_layer(raw, cfg.scheme, cfg.ratio)[0]      # attention-aware: W_V row pruned
    return cfg, w, make_x(cfg).astype(np.float64), make_lengths(cfg)


def _hp_partial(cfg, w, X, lens, h0, h1):
    """Oracle partial of heads [h0, h1) on the rank's slices (Eq. 4), b_O on the rank owning head 0."""
    from oracle import encoder as oe
    dk = cfg.d_model // cfg.heads
    a, b = h0 * dk, h1 * dk
    Q = oe.linear(X, w["wq"][a:b], w["bq"][a:b])
    K = oe.linear(X, w["wk"][a:b], w["bk"][a:b])
    V = oe.linear(X, w["wv"][a:b], w["bv"][a:b])
    Z = oe.attention_core(Q, K, V, h1 - h0, lens, cfg.causal, dk=dk)
    return oe.linear(Z, w["wo"][:, a:b], w["bo"] if h0 == 0 else None)


def _hp_worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        cfg, w, X, lens = _hp_case()
        h0, h1 = head_range(cfg.heads, world, rank)
        part = torch.from_numpy(_hp_partial(cfg, w, X, lens, h0, h1))
        dist.all_reduce(part, op=dist.ReduceOp.SUM)        # the head-parallel exchange step
        q.put((rank, h0, h1, part.numpy()))
    finally:
        dist.destroy_process_group()


def test_gloo_world2_head_parallel_allreduce_equals_full_attention():
    """World size 2 over gloo: each rank's oracle partial over its heads, summed by all-reduce,
    equals the oracle's full self-attention output (b_O counted once) on every rank."""
    from oracle import encoder as oe
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_hp_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = sorted((q.get(timeout=120) for _ in procs), key=lambda r: r[0])
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert [(r[1], r[2]) for r in res] == [(0, 2), (2, 4)]
    cfg, w, X, lens = _hp_case()
    ref = oe.attention_block(X, w, cfg.heads, lens, cfg.causal)
    for r in res:
        assert np.max(np.abs(r[3] - ref)) <= 1e-12 * max(1.0, np.max(np.abs(ref)))
    # a dropped / doubled bias would be caught: the partials alone are far from the full output
    assert np.max(np.abs(_hp_partial(cfg, w, X, lens, 2, 4) - ref)) > 1e-3
