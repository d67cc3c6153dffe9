"""Parameter sharding of the Adam workload across ranks (north_star:
"Adam over parameter partitions with no collective").

Adam is elementwise (DESIGN.md R-adam-1), so rank r of P updates a contiguous slice
[lo, hi) of p, m, v, g with no exchange at all; the only cross-rank operations are the
barriers that bracket timing.  Shard starts are multiples of 4 elements (16 B), so each
shard's p/m/v/g views keep the float4 alignment the kernels' 128-bit accesses need, and
the last rank takes the ragged tail.  Every rank holds its own JIT cache; all ranks but
the last share n/P, hence one specialization (the tail rank's n differs when P does not
divide n into multiples of 4).
"""
from __future__ import annotations


def shard_range(n: int, world: int, rank: int, align: int = 4) -> tuple[int, int]:
    """[lo, hi) of rank `rank`: contiguous, disjoint, covering [0, n), lo % align == 0 (an
    empty shard of a rank past the end is [n, n): callers skip it),
    sizes ceil(n / world) rounded up to `align`, the remainder on the last ranks."""
    if world < 1 or not 0 <= rank < world:
        raise ValueError(f"rank {rank} of world {world}")
    if n < 0:
        raise ValueError("n < 0")
    per = -(-n // world)
    per = -(-per // align) * align
    lo = min(rank * per, n)
    hi = min(lo + per, n)
    return lo, hi


def shard_views(tensors, n: int, world: int, rank: int):
    """Views of this rank's slice of each [n] tensor (no copy)."""
    lo, hi = shard_range(n, world, rank)
    return [t[lo:hi] for t in tensors], (lo, hi)
