"""The N > 1 host path of the stencil (z-slab halo exchange, halo.exchange_halos) run
with the gloo backend in world_size 2 and 4 CPU processes (-m "not gpu").

Each rank sweeps its slab with the oracle (test-only compute; the product path uses the
CUDA kernel), re-applies the global Dirichlet planes, and exchanges halos through the
same code the GPU bench uses.  The gathered result must equal the single-domain oracle
bit-exactly (pin P3, decomposition invariance).
"""
import os
import socket
import sys

import numpy as np
import pytest
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, shape, T, out_q):
    sys.path.insert(0, ROOT)
    import torch
    import torch.distributed as dist

    import oracle
    import synthetic
    from paper_conf_cgo_georgakoudispb25_b200 import halo

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    nx, ny, nz = shape
    nzl = nz // world
    u0 = synthetic.stencil_inputs(nx, ny, nz)
    co = synthetic.STENCIL_COEFFS
    slab = np.zeros((nzl + 4, ny, nx))
    lo = rank * nzl - 2
    s0, s1 = max(lo, 0), min(lo + nzl + 4, nz)
    slab[s0 - lo:s1 - lo] = u0[s0:s1]
    u = torch.from_numpy(slab)
    zg = np.arange(nzl + 4) + lo
    frozen = (zg < 2) | (zg > nz - 3)
    for _ in range(T):
        w = torch.from_numpy(oracle.stencil(u.numpy(), *co, T=1))
        w[frozen] = u[frozen]                # global Dirichlet planes (the kernel does this)
        halo.exchange_halos(w, nzl, rank, world)
        u = w
    owned = u[2:nzl + 2].contiguous()
    gathered = [torch.empty_like(owned) for _ in range(world)] if rank == 0 else None
    dist.gather(owned, gathered, dst=0)
    if rank == 0:
        out_q.put(torch.cat(gathered).numpy())
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world,shape,T", [(2, (12, 10, 16), 5), (4, (9, 11, 24), 4)])
def test_halo_exchange_gloo_matches_single_domain(world, shape, T):
    import oracle
    import synthetic
    oracle.build()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, shape, T, q)) for r in range(world)]
    for p in procs:
        p.start()
    got = q.get(timeout=120)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    nx, ny, nz = shape
    want = oracle.stencil(synthetic.stencil_inputs(nx, ny, nz), *synthetic.STENCIL_COEFFS, T=T)
    np.testing.assert_array_equal(got, want)
