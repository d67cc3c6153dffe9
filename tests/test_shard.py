"""Host logic of the Adam parameter sharding: shard bounds, and a gloo
world-2 run in which each rank updates its shard with the fp64 oracle and the gathered
result equals the single-process update bit for bit (Adam is elementwise, R-adam-1)."""
import os

import numpy as np
import pytest

import synthetic
from paper_conf_cgo_georgakoudispb25_b200.shard import shard_range


@pytest.mark.parametrize("n", [0, 1, 3, 4, 5, 1000, 1000003, 10 ** 6])
@pytest.mark.parametrize("world", [1, 2, 3, 4, 8])
def test_shards_partition_and_align(n, world):
    rs = [shard_range(n, world, r) for r in range(world)]
    assert rs[0][0] == 0 and rs[-1][1] == n
    for (a, b), (c, d) in zip(rs, rs[1:]):
        assert b == c                       # contiguous, disjoint
    for lo, hi in rs:
        assert (lo % 4 == 0 or lo == hi == n) and 0 <= lo <= hi <= n   # empty tail shards sit at n
    sizes = [hi - lo for lo, hi in rs]
    full = [s for s in sizes if s]
    assert max(sizes) - min(full or [0]) <= max(sizes)  # non-negative sizes
    assert all(s == sizes[0] for s in full[:-1])         # equal except the tail shard


def test_shard_rejects_bad_rank():
    with pytest.raises(ValueError):
        shard_range(10, 2, 2)


def _worker(rank, world, port, out):
    import torch.distributed as dist
    import torch
    import oracle
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    n = 1003
    S = synthetic.ADAM_SCALARS
    f = lambda x: float(np.float32(x))
    p, m, v, g = synthetic.adam_inputs(n)
    lo, hi = shard_range(n, world, rank)
    res = oracle.adam(p[lo:hi], m[lo:hi], v[lo:hi], g[lo:hi], lr=f(S["lr"]), b1=f(S["b1"]),
                      b2=f(S["b2"]), eps=f(S["eps"]), grad_scale=f(S["grad_scale"]),
                      decay=f(S["decay"]), steps=7)[0]
    parts = [None] * world
    dist.all_gather_object(parts, (lo, hi, res))
    if rank == 0:
        full = np.empty(n)
        for a, b, x in parts:
            full[a:b] = x
        np.save(out, full)
    dist.barrier()
    dist.destroy_process_group()


def test_gloo_world2_sharded_equals_single(tmp_path):
    import socket

    import torch.multiprocessing as mp

    import oracle
    oracle.build()
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    out = str(tmp_path / "full.npy")
    mp.spawn(_worker, args=(2, port, out), nprocs=2, join=True)
    S = synthetic.ADAM_SCALARS
    f = lambda x: float(np.float32(x))
    p, m, v, g = synthetic.adam_inputs(1003)
    want = oracle.adam(p, m, v, g, lr=f(S["lr"]), b1=f(S["b1"]), b2=f(S["b2"]), eps=f(S["eps"]),
                       grad_scale=f(S["grad_scale"]), decay=f(S["decay"]), steps=7)[0]
    np.testing.assert_array_equal(np.load(out), want)
