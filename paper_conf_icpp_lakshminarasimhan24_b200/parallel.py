"""Multi-GPU plumbing: one process per GPU, batch sharding with no data-path collective.

Merged execution never crosses images (bricks block the batch only within a brick, PAPER.md
L374-376, L738-739), so an inference batch shards trivially across ranks: rank r runs the whole
merged plan on its contiguous slice of images.  The only collectives are the timing barrier and the
max-over-ranks reduction in bench.py (plumbing, not the data path).
"""
from __future__ import annotations

import os


def shard(n_total: int, rank: int, world: int) -> tuple[int, int]:
    """Contiguous image range [lo, hi) of `rank`; sizes differ by at most one image."""
    if world <= 0 or not (0 <= rank < world):
        raise ValueError("bad rank/world")
    base, extra = divmod(n_total, world)
    lo = rank * base + min(rank, extra)
    hi = lo + base + (1 if rank < extra else 0)
    return lo, hi


def env_rank():
    """(rank, local_rank, world) from the torchrun environment (defaults: single process)."""
    return (int(os.environ.get("RANK", "0")), int(os.environ.get("LOCAL_RANK", "0")),
            int(os.environ.get("WORLD_SIZE", "1")))
