"""z-slab decomposition of the CFG 2 stencil across GPUs (one process per GPU).

Rank r of P owns global planes [r*nzl, (r+1)*nzl) of an nzg-plane field (nzl = nzg/P),
stored as a slab of nzl + 4 planes: 0-1 lower halo, 2..nzl+1 owned, nzl+2..nzl+3 upper
halo.  One sweep:

    1. w <- stencil(u) on the owned boundary planes {2,3} and {nzl, nzl+1}
    2. NCCL group (torch.distributed.batch_isend_irecv): send w{2,3} -> r-1 and
       w{nzl,nzl+1} -> r+1, receive into w{0,1} <- r-1 and w{nzl+2,nzl+3} <- r+1
       (2 planes = 2*nx*ny*8 B contiguous per neighbour per direction)
    3. w <- stencil(u) on the interior planes {4 .. nzl-1}, overlapping step 2
    4. wait for the receives; swap(u, w)

The stencil kernel itself applies the global Dirichlet frame (planes with global z < 2
or > nzg-3 are copied), so ranks 0 and P-1 need no special casing beyond skipping the
missing neighbour.  Only the halo exchange is a collective; the Adam workload shards
with no data-path collective at all.
"""
from __future__ import annotations

import numpy as np

from . import workloads as W


def neighbour_ops(w, nzl, rank, world, group=None):
    """P2P ops of one halo exchange on slab tensor w ([nzl+4, ny, nx], any device)."""
    import torch.distributed as dist
    ops = []
    if rank > 0:
        ops.append(dist.P2POp(dist.isend, w[2:4], rank - 1, group))
        ops.append(dist.P2POp(dist.irecv, w[0:2], rank - 1, group))
    if rank < world - 1:
        ops.append(dist.P2POp(dist.isend, w[nzl:nzl + 2], rank + 1, group))
        ops.append(dist.P2POp(dist.irecv, w[nzl + 2:nzl + 4], rank + 1, group))
    return ops


def exchange_halos(w, nzl, rank, world, group=None, wait=True):
    """Blocking (or asynchronous when wait=False) exchange of w's boundary planes."""
    import torch.distributed as dist
    if w.is_cuda and dist.get_backend(group) == "gloo":
        # gloo moves host memory only: stage the slab's boundary planes through the host
        # (used when several test ranks share one GPU; the product path is NCCL)
        h = w.cpu()
        exchange_halos(h, nzl, rank, world, group, wait=True)
        w[0:2].copy_(h[0:2])
        w[nzl + 2:nzl + 4].copy_(h[nzl + 2:nzl + 4])
        return []
    ops = neighbour_ops(w, nzl, rank, world, group)
    if not ops:
        return []
    works = dist.batch_isend_irecv(ops)
    if wait:
        for wk in works:
            wk.wait()
    return works


class ZSlabStencil:
    """Distributed stencil: this rank's slab pair + prepared launches (JIT or AOT)."""

    def __init__(self, kernel, u0_slab, *, nx, ny, nzl, nzg, rank, world, coeffs,
                 tile=None, group=None, variant="jit"):
        import torch
        assert nzl >= 4, "each rank needs >= 4 owned planes (2 boundary + 2 halo source)"
        self.nx, self.ny, self.nzl, self.nzg = nx, ny, nzl, nzg
        self.rank, self.world, self.group, self.variant = rank, world, group, variant
        self.u = u0_slab
        self.w = torch.empty_like(u0_slab)
        self.w.copy_(u0_slab)
        kg0 = rank * nzl
        common = dict(nx=nx, ny=ny, nzl=nzl, kg0=kg0, nzg=nzg, coeffs=coeffs, tile=tile)
        self.launch = {}
        for name, (a, b) in (("uw", (self.u, self.w)), ("wu", (self.w, self.u))):
            if world == 1:
                self.launch[name] = [W.stencil_launch(kernel, a, b, **common)]
            else:
                self.launch[name] = [
                    W.stencil_launch(kernel, a, b, k_begin=2, k_end=4, zchunks=1, **common),
                    W.stencil_launch(kernel, a, b, k_begin=nzl, k_end=nzl + 2, zchunks=1, **common),
                    W.stencil_launch(kernel, a, b, k_begin=4, k_end=nzl, **common)]
        self.parity = 0
        if world > 1:
            exchange_halos(self.u, nzl, rank, world, group)   # halos of u0 once

    def sweep(self, events=None):
        """One sweep; `events` = (start, end) CUDA events bracketing the compute launches."""
        name = "uw" if self.parity == 0 else "wu"
        dst = self.w if self.parity == 0 else self.u
        Ls = self.launch[name]
        if events:
            events[0].record()
        if self.world == 1:
            Ls[0](self.variant)
            if events:
                events[1].record()
        else:
            Ls[0](self.variant)
            Ls[1](self.variant)
            works = exchange_halos(dst, self.nzl, self.rank, self.world, self.group, wait=False)
            Ls[2](self.variant)                 # interior overlaps the NCCL transfer
            if events:
                events[1].record()
            for wk in works:
                wk.wait()                       # current stream waits for the receives
        self.parity ^= 1

    @property
    def current(self):
        return self.u if self.parity == 0 else self.w


def run_slabs_serial(kernel, u0, T, P, coeffs, variant="jit", tile=None):
    """Single-GPU emulation of the P-slab decomposition (halos copied on device between
    slabs).  Used by the decomposition-invariance test (pin P3)."""
    import torch
    nz, ny, nx = u0.shape
    assert nz % P == 0
    nzl = nz // P
    slabs = []
    for r in range(P):
        s = np.zeros((nzl + 4, ny, nx))
        lo, hi = max(0, r * nzl - 2), min(nz, (r + 1) * nzl + 2)
        s[lo - (r * nzl - 2):hi - (r * nzl - 2)] = u0[lo:hi]
        a = torch.from_numpy(s).cuda()
        slabs.append([a, a.clone()])
    launches = []
    for r in range(P):
        a, b = slabs[r]
        common = dict(nx=nx, ny=ny, nzl=nzl, kg0=r * nzl, nzg=nz, coeffs=coeffs, tile=tile)
        launches.append([W.stencil_launch(kernel, a, b, **common),
                         W.stencil_launch(kernel, b, a, **common)])
    for t in range(T):
        for r in range(P):
            launches[r][t % 2](variant)
        dst = (t + 1) % 2
        for r in range(P):
            if r > 0:
                slabs[r][dst][0:2].copy_(slabs[r - 1][dst][nzl:nzl + 2])
            if r < P - 1:
                slabs[r][dst][nzl + 2:nzl + 4].copy_(slabs[r + 1][dst][2:4])
    torch.cuda.synchronize()
    cur = T % 2
    return np.concatenate([slabs[r][cur][2:nzl + 2].cpu().numpy() for r in range(P)])
