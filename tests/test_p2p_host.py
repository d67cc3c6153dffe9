"""Host side of the fused stencil + halo exchange (NEXT-2) on the CPU box (-m "not gpu"):
the peer-address arithmetic against an independent slab model, the C-ABI peer-memory
entry points on the fake backend (host memory), and the gloo world-2 handle exchange."""
import ctypes
import os

import numpy as np
import pytest

from paper_conf_cgo_georgakoudispb25_b200 import halo
from paper_conf_cgo_georgakoudispb25_b200 import proteus as P


def test_peer_addresses_point_at_the_neighbours_halo_planes():
    nx, ny, nzl = 10, 6, 5
    plane = nx * ny * 8
    slab = (nzl + 4) * plane
    L, R = 1 << 20, 1 << 30
    peers, (sl, sr) = halo.p2p_peer_addresses(L, R, nx=nx, ny=ny, nzl=nzl)
    # rank r-1's halo above its owned planes = its local planes nzl+2, nzl+3 of each buffer
    assert peers["u"][0] == L + (nzl + 2) * plane
    assert peers["w"][0] == L + slab + (nzl + 2) * plane
    # rank r+1's halo below = its local planes 0, 1
    assert peers["u"][1] == R and peers["w"][1] == R + slab
    # flags: I write the left rank's "from right" word and the right rank's "from left"
    assert sl == L + 2 * slab + 4 * halo.FLAG_RIGHT
    assert sr == R + 2 * slab + 4 * halo.FLAG_LEFT
    peers, (sl, sr) = halo.p2p_peer_addresses(0, R, nx=nx, ny=ny, nzl=nzl)
    assert peers["u"][0] == 0 and peers["w"][0] == 0 and sl == 0 and sr != 0
    peers, (sl, sr) = halo.p2p_peer_addresses(L, 0, nx=nx, ny=ny, nzl=nzl)
    assert peers["u"][1] == 0 and peers["w"][1] == 0 and sr == 0 and sl != 0


def test_peer_addresses_match_arena_views():
    """The arena layout p2p_arena builds (on CPU tensors here) and the addresses
    p2p_peer_addresses computes agree byte for byte."""
    torch = pytest.importorskip("torch")
    nx, ny, nzl = 8, 4, 6
    arena, u, w, flags = halo.p2p_arena(nx, ny, nzl, torch.device("cpu"))
    base = arena.data_ptr()
    peers, (sl, sr) = halo.p2p_peer_addresses(base, base, nx=nx, ny=ny, nzl=nzl)
    assert peers["u"][0] == u[nzl + 2].data_ptr() and peers["w"][0] == w[nzl + 2].data_ptr()
    assert peers["u"][1] == u[0].data_ptr() and peers["w"][1] == w[0].data_ptr()
    assert sl == flags[halo.FLAG_RIGHT:].data_ptr() and sr == flags[halo.FLAG_LEFT:].data_ptr()
    assert flags.numel() == halo.FLAG_WORDS and not flags.any()


@pytest.fixture
def fake(tmp_path):
    P.proteus_finalize()
    P.testing_use_fake_backend(1)
    P.proteus_init(device=0, cache_dir=str(tmp_path))
    yield P
    P.proteus_finalize()
    P.testing_use_fake_backend(0)


def test_abi_peer_memory_roundtrip_on_fake_backend(fake):
    buf = (ctypes.c_uint32 * 64)()
    addr = ctypes.addressof(buf)
    h, off = P.proteus_ipc_get_handle(addr + 16)
    assert len(h) == 64 and off == 0
    assert P.proteus_ipc_open_handle(h) == addr + 16
    P.proteus_ipc_close_handle(addr)
    P.proteus_stream_write_u32(0, addr + 4, 7)
    assert buf[1] == 7
    P.proteus_stream_wait_u32(0, addr + 4, 7)          # satisfied: 7 >= 7
    P.proteus_stream_wait_u32(0, addr + 4, 3)
    with pytest.raises(P.ProteusError):
        P.proteus_stream_wait_u32(0, addr + 4, 8)      # would block on the fake backend
    with pytest.raises(P.ProteusError) as e:
        P.proteus_stream_write_u32(0, addr + 2, 1)     # misaligned
    assert e.value.status == 1
    with pytest.raises(P.ProteusError):
        P.proteus_ipc_open_handle(b"\0" * 64)


def test_abi_peer_memory_needs_init():
    P.proteus_finalize()
    with pytest.raises(P.ProteusError) as e:
        P.proteus_stream_write_u32(0, 64, 1)
    assert e.value.status == 2


def _exchange_worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    import tempfile

    import torch
    import torch.distributed as dist
    dist.init_process_group("gloo", rank=rank, world_size=world)
    P.testing_use_fake_backend(1)
    P.proteus_init(device=0, cache_dir=tempfile.mkdtemp())
    arena = torch.zeros(100, dtype=torch.float64)
    left, right, opened = halo.connect_ipc(arena, rank, world)
    # the fake handle carries the exporter's pointer: each rank must have mapped exactly
    # its neighbours' arenas
    ptrs = [None] * world
    dist.all_gather_object(ptrs, arena.data_ptr())
    q.put((rank, left == (ptrs[rank - 1] if rank > 0 else 0),
           right == (ptrs[rank + 1] if rank < world - 1 else 0), len(opened)))
    P.proteus_finalize()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_connect_ipc_exchanges_neighbour_handles_gloo(world):
    import multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = 29400 + os.getpid() % 500 + world
    ps = [ctx.Process(target=_exchange_worker, args=(r, world, port, q)) for r in range(world)]
    for p in ps:
        p.start()
    res = sorted(q.get(timeout=120) for _ in range(world))
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    for rank, ok_l, ok_r, n in res:
        assert ok_l and ok_r
        assert n == (rank > 0) + (rank < world - 1)
