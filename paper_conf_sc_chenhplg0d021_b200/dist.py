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


def all_equal_across_ranks(digest: str) -> bool:
    """True iff every rank passed the same digest."""
    import torch.distributed as dist
    if not (dist.is_available() and dist.is_initialized()):
        return True
    out = [None] * dist.get_world_size()
    dist.all_gather_object(out, digest)
    return all(o == out[0] for o in out)
