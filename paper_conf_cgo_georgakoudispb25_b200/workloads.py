"""The four workload kernels (+ the paper's daxpy example) registered with libproteus,
with launch helpers over torch CUDA tensors.  Argument marshalling only: every step
of every workload runs in the CUDA kernels under csrc/kernels/.

Each kernel is registered once with
  * its CUDA source (the same text nvcc compiled into libproteus_aot.so),
  * its parameter types and 1-based annotated indices (annotate("jit", ...), P@12394),
  * its generic AOT sm_100a CUfunction from libproteus_aot.so (proteus_aot_function).
`variant="jit"` launches through proteus_launch (key -> cache -> specialized cubin);
`variant="aot"` launches the nvcc-built generic kernel through proteus_launch_aot.
"""
from __future__ import annotations

import ctypes
import math
import os

from . import proteus as P

_PKG = os.path.dirname(os.path.abspath(__file__))
KERNEL_DIR = os.path.join(_PKG, "csrc", "kernels")

# name -> (parameter types, annotated 1-based indices, extra NVRTC/nvcc options)
SPECS = {
    # Fig. 2 daxpy(a, N, x, y), annotated 1, 2 (P@12394-12699)
    "daxpy": ([P.F64, P.I64, P.PTR, P.PTR], [1, 2], ""),
    # adam_step(p, m, v, g, n, lr, b1, b2, eps, grad_scale, decay, mode, bc1, bc2)
    "adam_step": ([P.PTR] * 4 + [P.U64] + [P.F32] * 6 + [P.I32, P.F32, P.F32],
                  [5, 6, 7, 8, 9, 10, 11], ""),
    # adam_run(p, m, v, g, n, lr, b1, b2, eps, grad_scale, decay, mode, steps, bc)  [the time
    # loop in-kernel; steps annotated like the paper's time_step]
    "adam_run": ([P.PTR] * 4 + [P.U64] + [P.F32] * 6 + [P.I32, P.I32, P.PTR],
                 [5, 6, 7, 8, 9, 10, 11, 13], ""),
    # stencil4(tmap(u), w, nx, ny, nzl, k_begin, k_end, kg0, nzg, a0, a1, a2)  [TMA-fed]
    "stencil4": ([P.OPAQUE, P.PTR] + [P.I32] * 7 + [P.F64] * 3, [3, 4, 5, 9, 10, 11, 12], ""),
    # stencil4_ws(tmap(u), w, ...same...)  [TMA ring, producer warp + empty/full mbarriers]
    "stencil4_ws": ([P.OPAQUE, P.PTR] + [P.I32] * 7 + [P.F64] * 3, [3, 4, 5, 9, 10, 11, 12], ""),
    # stencil4_p2p(...stencil4_ws..., peer_lo, peer_hi)  [+ halo stores into peer memory]
    "stencil4_p2p": ([P.OPAQUE, P.PTR] + [P.I32] * 7 + [P.F64] * 3 + [P.PTR, P.PTR],
                     [3, 4, 5, 9, 10, 11, 12], ""),
    # stencil4_smem(u, w, ...same...)   [per-thread loads + smem plane; any nx]
    "stencil4_smem": ([P.PTR, P.PTR] + [P.I32] * 7 + [P.F64] * 3, [3, 4, 5, 9, 10, 11, 12], ""),
    # xs_lookup(egrid, recs, mat_nuc, mat_off, mat_cnt, conc, cum, seed, L, n_nuc, n_grid,
    #           n_mat, macro_out, idx_out, perm, gidx)
    "xs_lookup": ([P.PTR] * 7 + [P.U64, P.U64, P.I32, P.I32, P.I32, P.PTR, P.PTR, P.PTR, P.PTR],
                  [9, 10, 11, 12], ""),
    # xs_index(egrid, n_nuc, n_grid, gidx): energy-bin search index, built once per table
    "xs_index": ([P.PTR, P.I32, P.I32, P.PTR], [2, 3], ""),
    # xs_bin(seed, L, n_mat, cum, counts); xs_scan(n_blk, n_mat, counts, prefix, totals);
    # xs_scatter(seed, L, n_mat, cum, totals, prefix, perm)   [per-block counting sort]
    "xs_bin": ([P.U64, P.U64, P.I32, P.PTR, P.PTR], [2, 3], ""),
    "xs_scan": ([P.I32, P.I32, P.PTR, P.PTR, P.PTR], [1, 2], ""),
    "xs_scatter": ([P.U64, P.U64, P.I32, P.PTR, P.PTR, P.PTR, P.PTR], [2, 3], ""),
    # micro_column(th, qv, qc, qr, rho, pk, p, precip, ncol, nz, nsub, dt, dz)
    "micro_column": ([P.PTR] * 8 + [P.U64, P.I32, P.I32, P.F32, P.F32], [10, 11, 13],
                     "-fmad=false"),
    # scale_count(y, n, bias): device-global linking demo (globals_demo.cu)
    "scale_count": ([P.PTR, P.I64, P.F64], [2, 3], ""),
    # micro_spec_sweep(start, count, fn, b, chunk_hash): exhaustive pin of exp_s/log_s/pow_s
    "micro_spec_sweep": ([P.U64, P.U64, P.I32, P.F32, P.PTR], [3, 4], "-fmad=false"),
}

_aot = None


def aot_function(entry: str) -> int:
    """CUfunction of the nvcc-built generic kernel (libproteus_aot.so)."""
    global _aot
    if _aot is None:
        if not os.path.exists(P.AOT_PATH):
            raise ImportError(f"{P.AOT_PATH} missing: run __graft_entry__.build()")
        _aot = ctypes.CDLL(P.AOT_PATH)
        _aot.proteus_aot_function.argtypes = [ctypes.c_char_p, ctypes.POINTER(ctypes.c_void_p)]
        _aot.proteus_aot_function.restype = ctypes.c_int
    fn = ctypes.c_void_p()
    rc = _aot.proteus_aot_function(entry.encode(), ctypes.byref(fn))
    if rc != 0 or not fn.value:
        raise RuntimeError(f"proteus_aot_function({entry}) failed with {rc}")
    return fn.value


SOURCE_FILE = {"stencil4_p2p": "stencil4_ws", "adam_run": "adam_step", "micro_spec_sweep": "micro_column",
               "scale_count": "globals_demo", "xs_bin": "xs_lookup", "xs_scan": "xs_lookup",
               "xs_scatter": "xs_lookup",
               "xs_index": "xs_lookup"}


def aot_global(name: str) -> int:
    """Device address of a __device__ global of the nvcc-built AOT module."""
    aot_function("daxpy")   # loads the library
    _aot.proteus_aot_global.argtypes = [ctypes.c_char_p, ctypes.POINTER(ctypes.c_void_p)]
    _aot.proteus_aot_global.restype = ctypes.c_int
    p = ctypes.c_void_p()
    rc = _aot.proteus_aot_global(name.encode(), ctypes.byref(p))
    if rc != 0 or not p.value:
        raise RuntimeError(f"proteus_aot_global({name}) failed with {rc}")
    return p.value


def kernel_source(entry: str) -> str:
    with open(os.path.join(KERNEL_DIR, SOURCE_FILE.get(entry, entry) + ".cu")) as f:
        return f.read()


# Launch-bounds minBlocks hint per kernel (proteus_kernel_set_min_blocks), tuned on B200
# (profiles/r01/tune_min_blocks.txt; micro_column 10 at 128-thread blocks for its
# warp-per-column layout, profiles/r01/ab_micro_lpl.txt, ab_micro_block.txt; adam_run 4 since the folded step of r02bp
# (48 registers either way; at 5 ptxas scheduled the folded loop worse, 0.0530 vs 0.0479 ms,
# profiles/r02/ab_adam_minb_r02br.txt; 5 for the r01 form, profiles/r01/ab_adam_rcp.txt); xs_lookup 9 at
# its 128-thread blocks since the r02 event-order kernel: 56 registers, no spill, 0.956 ms vs
# 1.034 at 8 and 1.009 for the generic build; large table 3.24 vs 3.43 ms,
# profiles/r02/tune_xs_minblocks_r02g.txt); kernels not listed use the config default (1, the
# paper's value, P@23207).
# stencil4_ws/_p2p: 4 resident 160-thread blocks per SM keep the 512-block sweep in one
# wave (with minBlocks 1 ptxas took 98 registers -> 3 blocks/SM -> 2 waves, 63 us vs 46).
MIN_BLOCKS = {"adam_run": 4, "micro_column": 10, "xs_lookup": 9, "stencil4_ws": 4, "stencil4_p2p": 4}
# Kernels launched with programmatic dependent launch (their sources call PROTEUS_PDL_WAIT
# before any global access): back-to-back launches overlap launch gap and prologue.
# PROTEUS_PDL=0 in the environment turns it off (A/B).
PDL_KERNELS = {"stencil4_ws", "adam_step"}


def register(entry: str, with_generic: bool = True, min_blocks: int | None = None,
             pdl: bool | None = None, generic_entry: str | None = None,
             options: str = "") -> P.Kernel:
    """generic_entry: another nvcc build of the same kernel to use as the generic AOT
    variant (e.g. "stencil4_ws_aotlb", the static-launch-bounds baseline).  options: extra
    NVRTC options for the specializations (e.g. "-DPROTEUS_CHECK", the device bounds
    checks of proteus_device.h); they are part of the kernel's identity."""
    types, ann, opts = SPECS[entry]
    opts = " ".join(o for o in (opts, options) if o)
    gen = aot_function(generic_entry or entry) if with_generic else None
    k = P.proteus_register_kernel(entry, kernel_source(entry), types, ann, gen, opts)
    mb = MIN_BLOCKS.get(entry, 0) if min_blocks is None else min_blocks
    if mb:
        k.set_min_blocks(mb)
    if pdl is None:
        pdl = entry in PDL_KERNELS and os.environ.get("PROTEUS_PDL", "1") != "0"
    if pdl:
        k.set_launch_attrs(P.LAUNCH_PDL)
    return k


class Launch:
    """A prepared launch: ctypes argument block built once, scalars updated in place,
    so the per-launch Python cost is one ctypes call.  Launch.override_stream (a CUstream
    int) redirects every launch, e.g. into a stream being captured into a CUDA graph."""

    override_stream = None

    def __init__(self, k: P.Kernel, grid, block, args, shmem=0, stream=0):
        self.k = k
        self.dims = P._dims(grid, block)
        self.arr, self.holders = k.pack(args)
        self.shmem = shmem
        self.stream = ctypes.c_void_p(stream)
        self._jit = P.lib.proteus_launch
        self._aot = P.lib.proteus_launch_aot

    def set(self, idx0: int, value):
        self.holders[idx0].value = value

    def prefetch(self):
        """Compile (or fetch from the caches) this launch's specialization without launching
        it -- proteus_get_specialization; thread-safe, and ctypes drops the GIL, so several
        prefetches compile concurrently (prefetch_all)."""
        fn, st, n = ctypes.c_void_p(), ctypes.c_int(), ctypes.c_size_t()
        P._check(P.lib.proteus_get_specialization(self.k.handle, *self.dims, self.arr,
                                                  ctypes.byref(fn), ctypes.byref(st), None, 0,
                                                  ctypes.byref(n)))

    def prefetch_async(self):
        """Start compiling this launch's specialization on the library's worker pool and
        return at once (proteus_prefetch); a later jit() launch waits for it if needed."""
        P._check(P.lib.proteus_prefetch(self.k.handle, *self.dims, self.arr))

    def jit(self):
        st = self.stream if Launch.override_stream is None else Launch.override_stream
        s = self._jit(self.k.handle, *self.dims, self.shmem, st, self.arr)
        if s:
            P._check(s)

    def aot(self):
        st = self.stream if Launch.override_stream is None else Launch.override_stream
        s = self._aot(self.k.handle, *self.dims, self.shmem, st, self.arr)
        if s:
            P._check(s)

    def __call__(self, variant="jit"):
        (self.jit if variant == "jit" else self.aot)()


def _stream(stream):
    if stream is not None:
        return stream
    import torch
    return torch.cuda.current_stream().cuda_stream


# ------------------------------------------------------------------------ daxpy (K0)
def daxpy_launch(k, a, x, y, block=256, stream=None):
    n = x.numel()
    grid = max(1, min((n + block - 1) // block, 148 * 16))
    return Launch(k, (grid,), (block,), [a, n, x.data_ptr(), y.data_ptr()], 0, _stream(stream))


# ------------------------------------------------------------------------ Adam (CFG 1)
def adam_bias_corrections(b1: float, b2: float, t: int):
    """fp32(1 - b^t) computed in double on the host (DESIGN.md R-adam-2)."""
    f32 = lambda x: ctypes.c_float(x).value
    b1f, b2f = f32(b1), f32(b2)
    return f32(1.0 - math.pow(b1f, t)), f32(1.0 - math.pow(b2f, t))


def adam_launch(k, p, m, v, g, *, lr, b1, b2, eps, grad_scale, decay, mode=1, block=256,
                stream=None):
    n = p.numel()
    assert p.data_ptr() % 16 == 0 and m.data_ptr() % 16 == 0 and v.data_ptr() % 16 == 0
    assert g.data_ptr() % 16 == 0
    grid = max(1, (n // 4 + block - 1) // block)
    bc1, bc2 = adam_bias_corrections(b1, b2, 1)
    L = Launch(k, (grid,), (block,), [p.data_ptr(), m.data_ptr(), v.data_ptr(), g.data_ptr(), n,
                                      lr, b1, b2, eps, grad_scale, decay, mode, bc1, bc2], 0,
               _stream(stream))
    L.b1, L.b2 = b1, b2
    return L


def adam_bias_table(b1: float, b2: float, t_first: int, steps: int):
    """fp32 [steps][2] of (bc1_t, bc2_t), t = t_first .. t_first+steps-1 (R-adam-2)."""
    import numpy as np
    return np.array([adam_bias_corrections(b1, b2, t) for t in range(t_first, t_first + steps)],
                    dtype=np.float32).reshape(-1)


ADAM_RUN_MAX_STEPS = 6144


# SFU (XU-pipe) operations per element-step of adam_run (adam_step.cu, R-adam-6): mode 1
# sqrt + rcp, with 1 of a float4's 4 reciprocals on the FMA pipe (ADAM_RCP_SPLIT 1) -> 7 per
# float4 and step; mode 0 one rsqrt.  The analytic count matches ncu: 1.75 x 10^8 over the
# 50.7 us launch = 75% of 148 SMs x 16 lanes x clock, ncu XU pipe 75.4% (r02ay).
ADAM_RUN_SFU_PER_ELEMENT_STEP = {1: 1.75, 0: 1.0}


def sfu_peak(sm_mhz):
    """SFU operations / s: 148 SMs x 16 XU lanes x SM clock."""
    return 148 * 16 * sm_mhz * 1e6


def adam_run_launch(k, p, m, v, g, *, lr, b1, b2, eps, grad_scale, decay, steps, t_first=1,
                    mode=1, block=256, stream=None):
    """One adam_run launch = `steps` Adam steps from t_first (the bias-correction table is
    built on the host and kept on the device with the Launch)."""
    import torch
    n = p.numel()
    assert p.data_ptr() % 16 == 0 and m.data_ptr() % 16 == 0 and v.data_ptr() % 16 == 0
    assert g.data_ptr() % 16 == 0
    # the kernel keeps the per-step reciprocals of (bc1, bc2) in 8 * steps bytes of dynamic
    # shared memory (R-adam-5): up to 6144 steps per launch (48 KB, no opt-in needed);
    # longer runs are split into launches with t_first (bit-exact, test_adam_run_split)
    assert 1 <= steps <= ADAM_RUN_MAX_STEPS, f"adam_run: 1..{ADAM_RUN_MAX_STEPS} steps per launch"
    bc = torch.from_numpy(adam_bias_table(b1, b2, t_first, steps)).to(p.device)
    # one float4 per thread (a one-wave grid of SMs x 4 CTAs with ~1.7 float4 per thread
    # measured slower on B200: 0.235 vs 0.203 ms for 100 steps of 10^6)
    grid = max(1, -(-(n // 4) // block))
    L = Launch(k, (grid,), (block,), [p.data_ptr(), m.data_ptr(), v.data_ptr(), g.data_ptr(), n,
                                      lr, b1, b2, eps, grad_scale, decay, mode, steps,
                                      bc.data_ptr()], 8 * steps, _stream(stream))
    L.bc = bc
    return L


def adam_set_step(L: Launch, t: int):
    bc1, bc2 = adam_bias_corrections(L.b1, L.b2, t)
    L.set(12, bc1)
    L.set(13, bc2)


# ------------------------------------------------------------------------ stencil (CFG 2)
STENCIL_TILE = (32, 4)        # threads (x, y) of the TMA kernel; each thread owns 2 x ST_RY points
STENCIL_RY = 2                # = ST_RY in stencil4.cu (tuned, profiles/r01/tune_stencil.txt)
STENCIL_RING = 6              # = ST_S in stencil4.cu
STENCIL_SMEM_TILE = (32, 8)   # stencil4_smem
# stencil4_ws: consumer warps, rows/thread (= WS_RY), ring slots (= WS_S), z-chunks
# (B200 sweep, profiles/r01/tune_ws_wide.txt)
STENCIL_WS = dict(ty=4, ry=2, ring=6, zchunks=4)


def stencil_config(entry: str) -> dict:
    """Default launch configuration of a stencil kernel (for reports)."""
    if entry in ("stencil4_ws", "stencil4_p2p"):
        return dict(STENCIL_WS, tile_points=[64, STENCIL_WS["ty"] * STENCIL_WS["ry"]],
                    block=[32, STENCIL_WS["ty"] + 1])
    if entry == "stencil4":
        return dict(tile=list(STENCIL_TILE), ry=STENCIL_RY, ring=STENCIL_RING)
    return dict(tile=list(STENCIL_SMEM_TILE))


def stencil_launch(k, u, w, *, nx, ny, nzl, kg0, nzg, coeffs, k_begin=None, k_end=None,
                   tile=None, zchunks=None, stream=None, ry=None, ring=None, peer_lo=0,
                   peer_hi=0):
    """One sweep over local planes [k_begin, k_end) of a (nzl+4)-plane slab u -> w.
    k.entry selects the kernel: "stencil4_ws" (warp-specialized TMA ring), "stencil4_p2p"
    (the same + boundary planes stored into the neighbours' halos at peer_lo / peer_hi:
    device addresses of plane nzl+2 of rank r-1's slab / plane 0 of rank r+1's, 0 = none),
    "stencil4" (TMA ring, v3) or "stencil4_smem"."""
    k_begin = 2 if k_begin is None else k_begin
    k_end = nzl + 2 if k_end is None else k_end
    assert 2 <= k_begin <= k_end <= nzl + 2
    a0, a1, a2 = coeffs
    nplanes = max(1, k_end - k_begin)
    if k.entry in ("stencil4_ws", "stencil4_p2p"):
        # tile = (32, consumer warps); block = 32 x (warps + 1): the last warp is the producer
        ty = (tile or (32, STENCIL_WS["ty"]))[1]
        tx = 32
        ry = ry or STENCIL_WS["ry"]
        ring = ring or STENCIL_WS["ring"]
        rows, cols = ty * ry, 64
        assert (nx * 8) % 16 == 0, "stencil4_ws (TMA) needs an even nx; use stencil4_smem"
        gx, gy = (nx + cols - 1) // cols, (ny + rows - 1) // rows
        if zchunks is None:
            # 4 z-chunks (512 blocks, one wave) down to 8 planes per chunk: best for every
            # per-rank slab of the 256^3 decomposition (nzl 256..32; at nzl 32: 7.4 us vs
            # 8.6 us with 2 chunks, profiles/r01/tune_slab_zchunks.txt)
            zchunks = max(1, min(STENCIL_WS["zchunks"], nplanes // 8))
        plane = -(-(cols + 4) * (rows + 4) // 16) * 16
        shmem = ring * plane * 8 + 2 * ring * 8
        tmap = P.proteus_encode_tensor_map(P.TMA_F64, u.data_ptr(), (nx, ny, nzl + 4),
                                           (nx * 8, nx * ny * 8), (cols + 4, rows + 4, 1))
        args = [tmap, w.data_ptr(), nx, ny, nzl, k_begin, k_end, kg0, nzg, a0, a1, a2]
        if k.entry == "stencil4_p2p":
            args += [peer_lo, peer_hi]
        else:
            assert not (peer_lo or peer_hi), "peer stores need the stencil4_p2p kernel"
        L = Launch(k, (gx, gy, zchunks), (tx, ty + 1), args, shmem, _stream(stream))
        L.u = u
        return L
    if k.entry == "stencil4":
        tx, ty = tile or STENCIL_TILE
        ry = ry or STENCIL_RY
        ring = ring or STENCIL_RING
        rows, cols = ty * ry, 2 * tx          # each thread: 2 columns x ry rows
        assert (nx * 8) % 16 == 0, "stencil4 (TMA) needs an even nx; use stencil4_smem"
        gx, gy = (nx + cols - 1) // cols, (ny + rows - 1) // rows
        if zchunks is None:   # ~512 blocks, >= 32 planes per chunk (profiles/r01/tune_stencil_v3.txt)
            zchunks = max(1, min(round(512 / (gx * gy)), nplanes // 32))
        plane = -(-(cols + 4) * (rows + 4) // 16) * 16     # 128-B aligned slots
        shmem = ring * plane * 8 + ring * 8
        tmap = P.proteus_encode_tensor_map(P.TMA_F64, u.data_ptr(), (nx, ny, nzl + 4),
                                           (nx * 8, nx * ny * 8), (cols + 4, rows + 4, 1))
        first = tmap
    else:
        tx, ty = tile or STENCIL_SMEM_TILE
        gx, gy = (nx + tx - 1) // tx, (ny + ty - 1) // ty
        if zchunks is None:   # ~ 2 waves of 8 resident 256-thread blocks per SM on 148 SMs
            zchunks = max(1, min(nplanes, (148 * 16) // (gx * gy)))
        shmem = (tx + 4) * (ty + 4) * 8
        first = u.data_ptr()
    L = Launch(k, (gx, gy, zchunks), (tx, ty), [first, w.data_ptr(), nx, ny, nzl, k_begin, k_end,
                                               kg0, nzg, a0, a1, a2], shmem, _stream(stream))
    L.u = u   # keep the source alive with its descriptor
    return L


# ------------------------------------------------------------------------ XS lookup (CFG 3)
def xs_device_tables(t: dict, device="cuda", index_kernel=None, variant="aot"):
    """Tables to the device; with `index_kernel` (registered "xs_index") also build the
    energy-bin search index gidx[n_nuc][XS_EBINS+1] on the device (once per table).  The
    index kernel runs its generic build by default: it runs once per table, so a
    specialization would be compiled for nothing (and a JIT job and an AOT job must do
    the same set-up work)."""
    import torch
    # xs_lookup indexes egrid / recs rows with 32-bit flat offsets (record element n_nuc *
    # n_grid * 6 must fit), and packs the material into perm's top 4 bits
    # n_nuc * n_grid < 2^26: the lookup's pipelined loop shuffles a bracket's flat start row
    # and its width in one word (XS_PACK, 26 + 6 bits)
    if t["n_nuc"] * t["n_grid"] >= 2 ** 26 or t["n_mat"] > 16:
        raise ValueError("xs tables too large: n_nuc * n_grid < 2^26 and n_mat <= 16 required")
    d = {}
    for name in ("egrid", "recs", "conc", "cum"):
        d[name] = torch.from_numpy(t[name].reshape(-1).copy()).to(device)
    for name in ("mat_nuc", "mat_off", "mat_cnt"):
        d[name] = torch.from_numpy(t[name].astype("int32")).to(device)
    d.update(n_nuc=t["n_nuc"], n_grid=t["n_grid"], n_mat=t["n_mat"], gidx=None)
    if index_kernel is not None:
        xs_build_index(d, index_kernel, variant)
    return d


def xs_build_index(d: dict, index_kernel, variant="aot"):
    """The energy-bin search index of tables already on the device (d from
    xs_device_tables): gidx[n][b] = lower(e_n, b / XS_EBINS), one xs_index launch."""
    import torch
    n = d["n_nuc"] * (XS_EBINS + 1)
    d["gidx"] = torch.empty(n, dtype=torch.int32, device=d["egrid"].device)
    Launch(index_kernel, ((n + 255) // 256,), (256,),
           [d["egrid"].data_ptr(), d["n_nuc"], d["n_grid"], d["gidx"].data_ptr()], 0,
           _stream(None))(variant)
    return d


XS_EBINS = 4096   # = XS_EBINS in xs_lookup.cu (profiles/r01/ab_xs_ebins.txt)
XS_BLOCK = 128    # xs_lookup threads per block (with minBlocks 9: <= 56 registers)
XS_SORT_BLOCK = 1024   # xs_bin / xs_scatter threads per block (one block per SM)
XS_BIN_SMEM_MAX = 200 * 1024   # = XS_BIN_SMEM_MAX in xs_lookup.cu


def xs_launch(k, d: dict, L: int, seed: int, macro_out, idx_out, block=XS_BLOCK, grid=None,
              stream=None, perm=None):
    """The lookup kernel alone; `perm` (from xs_bin/xs_scan/xs_scatter) selects sorted mode
    (slot t = lookup perm[t] & 0x0FFFFFFF); without it slot t = lookup t."""
    assert d["n_grid"] >= 3
    if grid is None:
        grid = max(1, (L + block - 1) // block)
    return Launch(k, (grid,), (block,), [d["egrid"].data_ptr(), d["recs"].data_ptr(),
                                         d["mat_nuc"].data_ptr(), d["mat_off"].data_ptr(),
                                         d["mat_cnt"].data_ptr(), d["conc"].data_ptr(),
                                         d["cum"].data_ptr(), seed, L, d["n_nuc"], d["n_grid"],
                                         d["n_mat"], macro_out.data_ptr(), idx_out.data_ptr(),
                                         perm.data_ptr() if perm is not None else 0,
                                         d["gidx"].data_ptr() if d.get("gidx") is not None else 0],
                  0, _stream(stream))


class XSStep:
    """One event-based lookup step = xs_bin -> xs_scan -> xs_scatter -> xs_lookup, sorted by
    (material, energy bin).  kernels: dict with the four registered entries.  Results go
    to macro_out / idx_out in event order: slot t holds lookup slot_lookups()[t]."""

    # The kernels of the step that are specialized (the others always run their generic AOT
    # build, as un-annotated kernels do in the paper): xs_scan gains nothing from folding
    # (16.6 vs 15.4 us, profiles/r02/xs_step_breakdown_r02as.txt), so it is not compiled.
    JIT_ENTRIES = ("xs_bin", "xs_scatter", "xs_lookup")

    def __init__(self, kernels, d, L, seed, macro_out, idx_out, block=XS_BLOCK, stream=None):
        import torch
        assert L < (1 << 28) and d["n_mat"] <= 16
        dev = macro_out.device
        nb = d["n_mat"] * XS_EBINS
        # the counting sort's blocks: one per SM (xs_bin and xs_scatter hold the 192 KB
        # bucket table in shared memory), each owning a contiguous chunk of the lookups
        self.n_blk = torch.cuda.get_device_properties(dev).multi_processor_count \
            if dev.type == "cuda" else 148
        self.perm = torch.empty(L, dtype=torch.int32, device=dev)
        self.counts = torch.empty(self.n_blk * nb, dtype=torch.int32, device=dev)
        self.prefix = torch.empty(self.n_blk * nb, dtype=torch.int32, device=dev)
        self.totals = torch.empty(nb, dtype=torch.int32, device=dev)
        stream = _stream(stream)
        smem = nb * 4 if nb * 4 <= XS_BIN_SMEM_MAX else 0
        self.launches = [
            Launch(kernels["xs_bin"], (self.n_blk,), (XS_SORT_BLOCK,),
                   [seed, L, d["n_mat"], d["cum"].data_ptr(), self.counts.data_ptr()],
                   smem, stream),
            Launch(kernels["xs_scan"], ((nb + 127) // 128,), (128,),
                   [self.n_blk, d["n_mat"], self.counts.data_ptr(), self.prefix.data_ptr(),
                    self.totals.data_ptr()], 0, stream),
            Launch(kernels["xs_scatter"], (self.n_blk,), (XS_SORT_BLOCK,),
                   [seed, L, d["n_mat"], d["cum"].data_ptr(), self.totals.data_ptr(),
                    self.prefix.data_ptr(), self.perm.data_ptr()], smem, stream),
            xs_launch(kernels["xs_lookup"], d, L, seed, macro_out, idx_out, block=block,
                      stream=stream, perm=self.perm)]

    def __call__(self, variant="jit"):
        for L_ in self.launches:
            L_(variant if L_.k.entry in self.JIT_ENTRIES else "aot")

    def slot_lookups(self):
        """Lookup index of each result slot after a step: results are written in event
        (sorted) order, slot t holding lookup perm[t] & 0x0FFFFFFF (DESIGN.md R-xs-3)."""
        return self.perm & 0x0FFFFFFF

    def prefetch(self, wait=False):
        """The step's specializations compiled concurrently in the background (a cold
        synchronous first step would otherwise compile them one after another); without
        `wait` the step's launches then wait for their own compile only, so xs_bin runs
        while the later kernels still compile."""
        prefetch_all([L_ for L_ in self.launches if L_.k.entry in self.JIT_ENTRIES], wait=wait)


def prefetch_all(launches, wait=True):
    """Specializations of several launches compiled concurrently on the library's worker
    pool (proteus_prefetch); `wait`: return once every queued compile is done."""
    for L_ in launches:
        L_.prefetch_async()
    if wait:
        P.proteus_wait_idle()


# ------------------------------------------------------------------------ microphysics (CFG 4)
MICRO_LANES = 32   # lanes per column = 64 / MICRO_LPL of micro_column.cu (a warp per column)


def micro_launch(k, s: dict, precip, *, nz, nsub, dt, dz, block=128, stream=None,
                 lanes=MICRO_LANES):
    """s: dict of [ncol][nz] fp32 CUDA tensors th, qv, qc, qr, rho, pk, p."""
    assert nz % 4 == 0 and 4 <= nz <= 128, "micro_column: nz must be a multiple of 4, <= 128"
    ncol = s["th"].shape[0]
    threads = ncol * lanes
    assert threads < (1 << 32), "micro_column indexes threads in 32 bits"
    grid = max(1, (threads + block - 1) // block)
    return Launch(k, (grid,), (block,), [s[n].data_ptr() for n in ("th", "qv", "qc", "qr", "rho",
                                                                    "pk", "p")]
                  + [precip.data_ptr(), ncol, nz, nsub, dt, dz], 0, _stream(stream))
