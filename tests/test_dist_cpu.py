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
