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


def _init_slab(self, kernel, u0_slab, *, nx, ny, nzl, nzg, rank, world, coeffs, tile, group,
               variant):
    """ZSlabStencil state: the slab pair and its prepared launches (one full launch per
    sweep at world 1; boundary {2,3}, boundary {nzl, nzl+1}, interior at world > 1)."""
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


class ZSlabStencil:
    """Distributed stencil: this rank's slab pair + prepared launches (JIT or AOT)."""

    def __init__(self, kernel, u0_slab, *, nx, ny, nzl, nzg, rank, world, coeffs,
                 tile=None, group=None, variant="jit"):
        _init_slab(self, kernel, u0_slab, nx=nx, ny=ny, nzl=nzl, nzg=nzg, rank=rank,
                   world=world, coeffs=coeffs, tile=tile, group=group, variant=variant)
        if world > 1:
            exchange_halos(self.u, nzl, rank, world, group)   # halos of u0 once

    # One sweep in phases (sweep() runs them in order; run_slabs_split_local interleaves
    # the phases of several slabs in one process, exchanging halos with device copies).
    def _launches(self):
        return self.launch["uw" if self.parity == 0 else "wu"]

    @property
    def dst(self):
        """The buffer this sweep writes."""
        return self.w if self.parity == 0 else self.u

    def phase_boundary(self):
        """World > 1: the owned boundary planes {2,3} and {nzl, nzl+1} of dst."""
        Ls = self._launches()
        Ls[0](self.variant)
        Ls[1](self.variant)

    def phase_interior(self):
        """World > 1: planes {4 .. nzl-1} of dst (they read no halo plane of u)."""
        self._launches()[2](self.variant)

    def sweep(self, events=None):
        """One sweep; `events` = (start, end) CUDA events bracketing the compute launches."""
        if events:
            events[0].record()
        if self.world == 1:
            self._launches()[0](self.variant)
            if events:
                events[1].record()
        else:
            self.phase_boundary()
            works = exchange_halos(self.dst, self.nzl, self.rank, self.world, self.group,
                                   wait=False)
            self.phase_interior()               # interior overlaps the NCCL transfer
            if events:
                events[1].record()
            for wk in works:
                wk.wait()                       # current stream waits for the receives
        self.parity ^= 1

    @property
    def current(self):
        return self.u if self.parity == 0 else self.w


def _slab_of(u0, r, nzl):
    """Rank r's slab (nzl owned planes + 2 halo planes per side, zeros past the field)."""
    nz, ny, nx = u0.shape
    s = np.zeros((nzl + 4, ny, nx))
    lo, hi = max(0, r * nzl - 2), min(nz, (r + 1) * nzl + 2)
    s[lo - (r * nzl - 2):hi - (r * nzl - 2)] = u0[lo:hi]
    return s


def copy_halos_local(slabs, bufname):
    """The halo exchange of P in-process slabs (ZSlabStencil objects): buffer `bufname`
    ("dst" or "current") of rank r receives its neighbours' boundary planes, exactly the
    planes neighbour_ops sends and receives (device-to-device copies on the stream)."""
    P_ = len(slabs)
    for r in range(P_):
        me = getattr(slabs[r], bufname)
        nzl = slabs[r].nzl
        if r > 0:
            me[0:2].copy_(getattr(slabs[r - 1], bufname)[nzl:nzl + 2])
        if r < P_ - 1:
            me[nzl + 2:nzl + 4].copy_(getattr(slabs[r + 1], bufname)[2:4])


def run_slabs_split_local(kernel, u0, T, P_, coeffs, variant="jit", tile=None):
    """Single-GPU run of ZSlabStencil's N > 1 sweep: P_ slabs in one process, each sweep
    in ZSlabStencil's three launches per slab (boundary planes, then -- after the halo
    exchange, here device copies between the slabs -- the interior).  Returns the owned
    planes of all slabs after T sweeps, [nz][ny][nx]."""
    import torch
    nz, ny, nx = u0.shape
    assert nz % P_ == 0 and P_ > 1
    nzl = nz // P_
    slabs = []
    for r in range(P_):
        st = ZSlabStencil.__new__(ZSlabStencil)
        _init_slab(st, kernel, torch.from_numpy(_slab_of(u0, r, nzl)).cuda(), nx=nx, ny=ny,
                   nzl=nzl, nzg=nz, rank=r, world=P_, coeffs=coeffs, tile=tile, group=None,
                   variant=variant)
        slabs.append(st)
    for _ in range(T):
        for st in slabs:
            st.phase_boundary()
        copy_halos_local(slabs, "dst")
        for st in slabs:
            st.phase_interior()
        for st in slabs:
            st.parity ^= 1
    torch.cuda.synchronize()
    return np.concatenate([st.current[2:nzl + 2].cpu().numpy() for st in slabs])


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


# ------------------------------------------------------------------------------------
# NEXT-2: the halo exchange fused into the stencil kernel over peer memory.
#
# Each rank keeps its slab pair and a small flag block in ONE device allocation (the
# "arena", one CUDA IPC handle).  Ranks exchange handles once (torch.distributed object
# collective: host-side plumbing only), map their neighbours' arenas, and from then on a
# sweep s on rank r is, all on r's stream:
#     wait  flag_from_left >= s and flag_from_right >= s     (neighbours finished s-1:
#           my halo planes of `cur` are written, and their `dst` is no longer read)
#     stencil4_p2p(cur -> dst): owned planes to dst, boundary planes {2,3} also into
#           rank r-1's dst plane nzl+2.., {nzl, nzl+1} into rank r+1's dst plane 0..
#     write rank r-1's flag_from_right = s+1 and rank r+1's flag_from_left = s+1
#           (stream write ordered after the kernel, with a memory fence)
# so the only data movement between ranks is the kernel's own stores, overlapped with
# its compute, and no NCCL kernel or copy sits between sweeps.  The waits and writes are
# executed by the GPU front end (proteus_stream_wait_u32 / proteus_stream_write_u32).
# ------------------------------------------------------------------------------------
FLAG_LEFT, FLAG_RIGHT = 0, 32     # int32 indices in the flag block (separate 128-B lines)
FLAG_WORDS = 64


def p2p_arena(nx, ny, nzl, device):
    """(arena, u, w, flags): one allocation holding both slabs and the zeroed flags."""
    import torch
    slab = (nzl + 4) * ny * nx
    arena = torch.zeros(2 * slab + FLAG_WORDS // 2, dtype=torch.float64, device=device)
    u = arena[:slab].view(nzl + 4, ny, nx)
    w = arena[slab:2 * slab].view(nzl + 4, ny, nx)
    flags = arena[2 * slab:].view(torch.int32)
    return arena, u, w, flags


def p2p_peer_addresses(arena_ptr_left, arena_ptr_right, *, nx, ny, nzl):
    """Peer addresses for rank r given the neighbours' arena base addresses (0 = none):
    {"u": (lo, hi), "w": (lo, hi)} halo targets per buffer and (sig_left, sig_right)
    flag words to write.  lo = plane nzl+2 of the left rank's buffer, hi = plane 0 of the
    right rank's buffer (the arena layout of p2p_arena)."""
    plane = ny * nx * 8
    slab = (nzl + 4) * plane
    out = {}
    for i, name in enumerate(("u", "w")):
        lo = arena_ptr_left + i * slab + (nzl + 2) * plane if arena_ptr_left else 0
        hi = arena_ptr_right + i * slab if arena_ptr_right else 0
        out[name] = (lo, hi)
    flag_base = lambda a: a + 2 * slab
    sig_left = flag_base(arena_ptr_left) + 4 * FLAG_RIGHT if arena_ptr_left else 0
    sig_right = flag_base(arena_ptr_right) + 4 * FLAG_LEFT if arena_ptr_right else 0
    return out, (sig_left, sig_right)


def connect_ipc(arena, rank, world, group=None):
    """Exchange arena IPC handles with the neighbours; -> (left base, right base,
    mapped bases to close).  Collective over all ranks (all_gather_object)."""
    import torch.distributed as dist

    from . import proteus as P
    h, off = P.proteus_ipc_get_handle(arena.data_ptr())
    allh = [None] * world
    dist.all_gather_object(allh, (h, off), group=group)
    opened, bases = [], {}
    for nb in (rank - 1, rank + 1):
        if 0 <= nb < world:
            hh, oo = allh[nb]
            if hh not in bases:
                bases[hh] = P.proteus_ipc_open_handle(hh)
                opened.append(bases[hh])
    left = bases[allh[rank - 1][0]] + allh[rank - 1][1] if rank > 0 else 0
    right = bases[allh[rank + 1][0]] + allh[rank + 1][1] if rank < world - 1 else 0
    return left, right, opened


class P2PZSlabStencil:
    """This rank's slabs (in a p2p_arena) + stencil4_p2p launches + flag protocol.
    `left`/`right` = neighbour arena base addresses in THIS process (connect_ipc across
    processes, or plain device pointers when several slabs live in one process)."""

    def __init__(self, kernel, arena_parts, *, nx, ny, nzl, nzg, rank, world, coeffs, left,
                 right, variant="jit", stream=None, tile=None):
        import torch
        assert kernel.entry == "stencil4_p2p"
        assert nzl >= 4, "each rank needs >= 4 owned planes"
        self.arena, self.u, self.w, self.flags = arena_parts
        self.rank, self.world, self.nzl, self.variant = rank, world, nzl, variant
        self.stream = stream if stream is not None else torch.cuda.current_stream().cuda_stream
        peers, (self.sig_left, self.sig_right) = p2p_peer_addresses(left, right, nx=nx, ny=ny,
                                                                    nzl=nzl)
        fbase = self.flags.data_ptr()
        self.wait_left = fbase + 4 * FLAG_LEFT if left else 0
        self.wait_right = fbase + 4 * FLAG_RIGHT if right else 0
        common = dict(nx=nx, ny=ny, nzl=nzl, kg0=rank * nzl, nzg=nzg, coeffs=coeffs, tile=tile,
                      stream=self.stream)
        self.launch = {
            "uw": W.stencil_launch(kernel, self.u, self.w, peer_lo=peers["w"][0],
                                   peer_hi=peers["w"][1], **common),
            "wu": W.stencil_launch(kernel, self.w, self.u, peer_lo=peers["u"][0],
                                   peer_hi=peers["u"][1], **common)}
        self.s = 0          # sweeps issued so far (flag values count completed sweeps)

    def sweep(self, events=None):
        from . import proteus as P
        s = self.s
        if s > 0:
            if self.wait_left:
                P.proteus_stream_wait_u32(self.stream, self.wait_left, s)
            if self.wait_right:
                P.proteus_stream_wait_u32(self.stream, self.wait_right, s)
        if events:
            events[0].record()
        self.launch["uw" if s % 2 == 0 else "wu"](self.variant)
        if events:
            events[1].record()
        if self.sig_left:
            P.proteus_stream_write_u32(self.stream, self.sig_left, s + 1)
        if self.sig_right:
            P.proteus_stream_write_u32(self.stream, self.sig_right, s + 1)
        self.s = s + 1

    @property
    def current(self):
        return self.u if self.s % 2 == 0 else self.w


def run_slabs_p2p_local(kernel, u0, T, P_, coeffs, variant="jit"):
    """P_ "ranks" in ONE process on one GPU, each with its own arena and stream, wired
    with plain device pointers: the kernel's peer stores and the flag protocol run exactly
    as across processes (IPC only changes how the addresses are obtained)."""
    import torch
    nz, ny, nx = u0.shape
    assert nz % P_ == 0
    nzl = nz // P_
    dev = torch.device("cuda", torch.cuda.current_device())
    parts = []
    for r in range(P_):
        arena, u, w, flags = p2p_arena(nx, ny, nzl, dev)
        lo, hi = max(0, r * nzl - 2), min(nz, (r + 1) * nzl + 2)
        u[lo - (r * nzl - 2):hi - (r * nzl - 2)] = torch.from_numpy(u0[lo:hi]).to(dev)
        w.copy_(u)
        parts.append((arena, u, w, flags))
    streams = [torch.cuda.Stream() for _ in range(P_)]
    torch.cuda.synchronize()
    sts = [P2PZSlabStencil(kernel, parts[r], nx=nx, ny=ny, nzl=nzl, nzg=nz, rank=r, world=P_,
                           coeffs=coeffs,
                           left=parts[r - 1][0].data_ptr() if r > 0 else 0,
                           right=parts[r + 1][0].data_ptr() if r < P_ - 1 else 0,
                           variant=variant, stream=streams[r].cuda_stream)
           for r in range(P_)]
    for _ in range(T):
        for st in sts:
            st.sweep()
    torch.cuda.synchronize()
    out = np.concatenate([st.current[2:nzl + 2].cpu().numpy() for st in sts])
    flags = [st.flags.cpu().numpy()[[FLAG_LEFT, FLAG_RIGHT]].tolist() for st in sts]
    return out, flags
