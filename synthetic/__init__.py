"""Seeded synthetic inputs shared by the oracle tests, the GPU tests and bench.py.

This module holds ONLY input generation: the counter-based generator and the
recipes that turn it into the four workloads' inputs.
It contains none of the method's arithmetic (no specialization, no workload
update rule), so it may serve both the CPU oracle (oracle/) and the CUDA path
without coupling them.

Counter-based RNG:
    rng(stream, i) = splitmix64_next(S0 + (stream << 40) + i)      (mod 2**64)
    S0 = 0x50524F54455553 ("PROTEUS")
    splitmix64_next(x) = first output of SplitMix64 seeded with x
    u01_f64(r) = (r >> 11) * 2**-53        u01_f32(r) = (r >> 40) * 2**-24
Both conversions are exact.  The XS-lookup kernel and the oracle each draw the
per-lookup (E, r) pair from this same generator (streams 34/35) independently.

Shapes and value ranges follow the paper's workloads as reshaped by
BASELINE.json configs (Table 1 @29055-29432).
"""
from __future__ import annotations

import numpy as np

S0 = 0x50524F54455553
_M64 = (1 << 64) - 1
_GOLDEN = np.uint64(0x9E3779B97F4A7C15)
_C1 = np.uint64(0xBF58476D1CE4E5B9)
_C2 = np.uint64(0x94D049BB133111EB)


def splitmix64_next(x):
    """First SplitMix64 output for state x (numpy uint64 array or int)."""
    with np.errstate(over="ignore"):
        z = np.asarray(x, dtype=np.uint64) + _GOLDEN
        z = (z ^ (z >> np.uint64(30))) * _C1
        z = (z ^ (z >> np.uint64(27))) * _C2
        return z ^ (z >> np.uint64(31))


def rng(stream: int, idx, seed: int = S0):
    """rng(stream, i) for an int or an integer array of counters i."""
    base = np.uint64((seed + (stream << 40)) & _M64)
    with np.errstate(over="ignore"):
        return splitmix64_next(base + np.asarray(idx, dtype=np.uint64))


def u01_f64(r):
    return (np.asarray(r, dtype=np.uint64) >> np.uint64(11)).astype(np.float64) * (2.0 ** -53)


def u01_f32(r):
    # (r >> 40) has 24 bits: exact in fp32; the scale is a power of two.
    return ((np.asarray(r, dtype=np.uint64) >> np.uint64(40)).astype(np.float32)
            * np.float32(2.0 ** -24))


# --------------------------------------------------------------------------------------
# CFG 1: fused Adam (SURVEY.md §8c-1 inputs)
# --------------------------------------------------------------------------------------
ADAM_SCALARS = dict(lr=1e-3, b1=0.9, b2=0.999, eps=1e-8, grad_scale=1024.0, decay=0.01, mode=1)


def adam_inputs(n: int, seed: int = S0):
    """p0 in +-[0.5, 1), g in [-16, 16), m = v = 0, all fp32 [n]."""
    i = np.arange(n, dtype=np.uint64)
    s = np.where((rng(12, i, seed) & np.uint64(1)) == 0, 1.0, -1.0)
    p = (s * (1.0 + u01_f32(rng(10, i, seed)).astype(np.float64)) / 2.0).astype(np.float32)
    g = ((2.0 * u01_f32(rng(11, i, seed)).astype(np.float64) - 1.0) * 16.0).astype(np.float32)
    m = np.zeros(n, np.float32)
    v = np.zeros(n, np.float32)
    return p, m, v, g


# --------------------------------------------------------------------------------------
# CFG 2: 4th-order 3D stencil (SURVEY.md §8c-2 inputs)
# --------------------------------------------------------------------------------------
STENCIL_COEFFS = (1.0 - 90.0 / 128.0, 16.0 / 128.0, -1.0 / 128.0)   # kappa = 12/128, dyadic


def stencil_inputs(nx: int, ny: int, nz: int, seed: int = S0):
    """u0 = 1 + 0.5*U(0,1) as fp64 [nz][ny][nx], global index (k*ny + j)*nx + i."""
    idx = np.arange(nx * ny * nz, dtype=np.uint64)
    return (1.0 + 0.5 * u01_f64(rng(20, idx, seed))).reshape(nz, ny, nx)


def polynomial_field(nx, ny, nz, coefs):
    """Integer polynomial sum c * x^a y^b z^c in centred coords, returned as fp64.

    coefs: list of (c, a, b, cc) with integer c.  Used by pins P1/P2 only."""
    x = np.arange(nx, dtype=np.int64) - nx // 2
    y = np.arange(ny, dtype=np.int64) - ny // 2
    z = np.arange(nz, dtype=np.int64) - nz // 2
    Z, Y, X = np.meshgrid(z, y, x, indexing="ij")
    out = np.zeros((nz, ny, nx), dtype=np.int64)
    for c, a, b, d in coefs:
        out += c * X ** a * Y ** b * Z ** d
    return out


# --------------------------------------------------------------------------------------
# CFG 3: Monte-Carlo cross-section lookup (SURVEY.md §8c-3 inputs)
# --------------------------------------------------------------------------------------
XS_MAT_COUNTS = [34, 5, 4, 4, 27, 21, 21, 21, 21, 21, 9, 9]
# NEXT-3: XSBench-"large"-shaped table, 355 nuclides with a 321-nuclide
# fuel material (outside knowledge, like the small constants; DESIGN.md R-xs-large):
# 355 x 11303 x (8 + 48) B = 225 MB of energies + records, beyond the 126 MB L2.
XS_NUC_LARGE = 355
XS_MAT_COUNTS_LARGE = [321, 5, 4, 4, 27, 21, 21, 21, 21, 21, 9, 9]
XS_MAT_PROBS = [0.140, 0.052, 0.275, 0.134, 0.154, 0.064, 0.066, 0.055, 0.008, 0.015, 0.025, 0.013]
XS_NCHAN = 5          # sigma_t, sigma_el, sigma_abs, sigma_f, nu*sigma_f
XS_REC = 6            # record = {E, 5 channels} fp64


def xs_tables(n_nuc: int = 68, n_grid: int = 11303, seed: int = S0, mat_counts=None):
    """Returns dict with
      egrid  fp64 [n_nuc][n_grid]   strictly increasing per nuclide, values in (0,1)
      recs   fp64 [n_nuc][n_grid][6] {E, s_t, s_el, s_abs, s_f, nu_s_f}
      mat_nuc i32 [sum counts], mat_off i32 [n_mat], mat_cnt i32 [n_mat]
      conc   fp64 [sum counts]
      cum    fp64 [n_mat] prefix sums of the selection probabilities (index order)
    mat_counts: nuclides per material (default XS_MAT_COUNTS; material 0 = nuclides
    0..counts[0]-1, the others sampled without replacement).
    """
    counts = list(XS_MAT_COUNTS if mat_counts is None else mat_counts)
    assert len(counts) == len(XS_MAT_PROBS) and counts[0] <= n_nuc and max(counts) <= n_nuc
    egrid = np.empty((n_nuc, n_grid), np.float64)
    for n in range(n_nuc):
        # draws in counter order; drop zeros and repeats (keep first occurrence),
        # extend the counter range until n_grid distinct values exist, then sort.
        base = np.uint64(n << 24)
        c1 = n_grid
        while True:
            draw = u01_f64(rng(30, np.arange(c1, dtype=np.uint64) + base, seed))
            draw = draw[draw > 0.0]
            _, first = np.unique(draw, return_index=True)
            if first.size >= n_grid:
                break
            c1 += n_grid - first.size + 8
        keep = np.sort(first)[:n_grid]
        egrid[n] = np.sort(draw[keep])
    recs = np.empty((n_nuc, n_grid, XS_REC), np.float64)
    recs[:, :, 0] = egrid
    ridx = np.arange(n_nuc * n_grid * XS_NCHAN, dtype=np.uint64)
    recs[:, :, 1:] = u01_f64(rng(31, ridx, seed)).reshape(n_nuc, n_grid, XS_NCHAN)
    mats = [np.arange(counts[0], dtype=np.int32)]
    for m in range(1, len(counts)):
        perm = np.arange(n_nuc, dtype=np.int64)
        for t in range(n_nuc - 1, 0, -1):   # Fisher-Yates, stream 32
            j = int(rng(32, (m << 16) + t, seed) % np.uint64(t + 1))
            perm[t], perm[j] = perm[j], perm[t]
        mats.append(np.sort(perm[:counts[m]]).astype(np.int32))
    mat_cnt = np.array(counts, np.int32)
    mat_off = np.concatenate([[0], np.cumsum(mat_cnt)[:-1]]).astype(np.int32)
    mat_nuc = np.concatenate(mats).astype(np.int32)
    conc = u01_f64(rng(33, np.arange(mat_nuc.size, dtype=np.uint64), seed))
    cum = np.cumsum(np.array(XS_MAT_PROBS, np.float64))
    return dict(egrid=egrid, recs=recs, mat_nuc=mat_nuc, mat_off=mat_off, mat_cnt=mat_cnt,
                conc=conc, cum=cum, n_nuc=n_nuc, n_grid=n_grid, n_mat=len(counts))


def xs_tables_large(n_grid: int = 11303, seed: int = S0):
    """NEXT-3: the XSBench-large-shaped table (355 nuclides, 321 in the fuel)."""
    return xs_tables(XS_NUC_LARGE, n_grid, seed, XS_MAT_COUNTS_LARGE)


# --------------------------------------------------------------------------------------
# CFG 4: column microphysics (SURVEY.md §8c-4 inputs; layout [col][k], fp32)
# --------------------------------------------------------------------------------------
MICRO_DT = 20.0
MICRO_NSUB = 2
MICRO_DZ = 250.0


def micro_inputs(ncol: int, nz: int = 64, seed: int = S0, dry: bool = False):
    """Returns dict of fp32 [ncol][nz] arrays th, qv, qc, qr, rho, pk, p.

    Background: z_k = 125 + 250 k, p = 1e5 exp(-z/8000), pk = (p/1e5)^0.2875,
    rho = 1.2 exp(-z/8000)(1 + 0.01 u), theta = 300 + 0.004 z + (u - 0.5).
    Moisture uses a Magnus/Bolton saturation (NOT the scheme's formula) so the
    generator shares no arithmetic with the method:
        e_s = 611.2 exp(17.67 (T-273.15)/(T-29.65)),  q_s = 0.622 e_s/(p - e_s)
        qv = RH q_s with RH ~ U(0.5, 1.05)  (dry=True: RH = 0.3, qc = qr = 0)
        qc ~ U(0, 1e-3) where RH > 0.95 else 0;  qr ~ U(0, 2e-3) in 30% of columns.
    """
    out = {k: np.empty((ncol, nz), np.float32) for k in ("th", "qv", "qc", "qr", "rho", "pk", "p")}
    # per-level background, identical in every column (computed once, broadcast)
    z = 125.0 + 250.0 * np.arange(nz, dtype=np.float64)[None, :]
    p = 1e5 * np.exp(-z / 8000.0)
    pk = (p / 1e5) ** 0.2875
    rho0 = 1.2 * np.exp(-z / 8000.0)
    rainy_all = u01_f64(rng(44, np.arange(ncol, dtype=np.uint64), seed)) < 0.3
    CH = 16384   # columns per chunk: the element-wise recipe below in cache-sized pieces

    def chunk(c0):
        c1 = min(ncol, c0 + CH)
        idx = (np.arange(c0 * nz, c1 * nz, dtype=np.uint64)).reshape(c1 - c0, nz)
        rho = rho0 * (1.0 + 0.01 * u01_f64(rng(40, idx, seed)))
        th = 300.0 + 0.004 * z + (u01_f64(rng(41, idx, seed)) - 0.5)
        T = pk * th
        es = 611.2 * np.exp(17.67 * (T - 273.15) / (T - 29.65))
        qs = 0.622 * es / (p - es)
        if dry:
            rh = np.full((c1 - c0, nz), 0.3)
            qc = np.zeros((c1 - c0, nz))
            qr = np.zeros((c1 - c0, nz))
        else:
            rh = 0.5 + 0.55 * u01_f64(rng(42, idx, seed))
            qc = np.where(rh > 0.95, 1e-3 * u01_f64(rng(43, idx, seed)), 0.0)
            qr = np.where(rainy_all[c0:c1, None], 2e-3 * u01_f64(rng(45, idx, seed)), 0.0)
        qv = rh * qs
        for k, v in (("th", th), ("qv", qv), ("qc", qc), ("qr", qr), ("rho", rho)):
            out[k][c0:c1] = v

    # chunks are independent (counter-based draws): numpy releases the GIL in its loops,
    # so threads split the work; the result does not depend on the thread count
    starts = range(0, ncol, CH)
    if len(starts) > 4:
        from concurrent.futures import ThreadPoolExecutor
        import os
        with ThreadPoolExecutor(max_workers=min(16, len(os.sched_getaffinity(0)))) as ex:
            list(ex.map(chunk, starts))
    else:
        for c0 in starts:
            chunk(c0)
    out["pk"][:] = pk
    out["p"][:] = p
    return out

