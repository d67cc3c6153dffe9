"""CPU oracle (TEST INFRASTRUCTURE ONLY).

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference
legs may import this package.  The product package never imports it.  It shares no
code with the CUDA path: liboracle.so is built from oracle/oracle.c alone, and the
Python key oracle (oracle/key.py) is an independent implementation of the
specialization-key layout.

Functions and the passage each follows are documented in oracle/oracle.c.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
CFLAGS = ["-O2", "-fno-fast-math", "-ffp-contract=off", "-fopenmp", "-fPIC", "-shared",
          "-std=c11", "-Wall"]


def build(force: bool = False) -> str:
    """Compile liboracle.so with gcc (plain C, no contraction)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < max(
            os.path.getmtime(_SRC), os.path.getmtime(os.path.join(_HERE, "oracle.h"))):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", *CFLAGS, "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB)
        u64, i32, f32, f64 = ctypes.c_uint64, ctypes.c_int, ctypes.c_float, ctypes.c_double
        P = ctypes.c_void_p
        L.oracle_splitmix64.restype = u64
        L.oracle_splitmix64.argtypes = [u64]
        L.oracle_rng.restype = u64
        L.oracle_rng.argtypes = [u64, u64, u64]
        L.oracle_fnv1a64.restype = u64
        L.oracle_fnv1a64.argtypes = [ctypes.c_char_p, u64]
        L.oracle_set_threads.argtypes = [i32]
        L.oracle_get_threads.restype = i32
        L.oracle_adam.argtypes = [P, P, P, P, u64, f32, f32, f32, f32, f32, f32, i32, i32, i32]
        L.oracle_stencil_sweep.argtypes = [P, P, i32, i32, i32, f64, f64, f64]
        L.oracle_stencil_run.argtypes = [P, P, i32, i32, i32, f64, f64, f64, i32]
        L.oracle_stencil_run.restype = i32
        L.oracle_xs_lower.argtypes = [P, i32, f64]
        L.oracle_xs_lower.restype = i32
        L.oracle_xs_lookup.argtypes = [P, P, P, P, P, P, P, u64, u64, u64, i32, i32, i32, P, P, P]
        L.oracle_exp_s.argtypes = [f32]
        L.oracle_exp_s.restype = f32
        L.oracle_log_s.argtypes = [f32]
        L.oracle_log_s.restype = f32
        L.oracle_pow_s.argtypes = [f32, f32]
        L.oracle_pow_s.restype = f32
        L.oracle_micro.argtypes = [P, P, P, P, P, P, P, P, u64, i32, i32, f32, f32, i32]
        L.oracle_spec_sweep.argtypes = [u64, u64, i32, f32, P]
        _lib = L
    return _lib


def _p(a: np.ndarray):
    assert a.flags["C_CONTIGUOUS"]
    return a.ctypes.data_as(ctypes.c_void_p)


def set_threads(n: int) -> int:
    lib().oracle_set_threads(int(n))
    return lib().oracle_get_threads()


def splitmix64(x: int) -> int:
    return lib().oracle_splitmix64(x)


def rng(seed: int, stream: int, i: int) -> int:
    return lib().oracle_rng(seed, stream, i)


def fnv1a64(data: bytes) -> int:
    return lib().oracle_fnv1a64(data, len(data))


def adam(p, m, v, g, *, lr, b1, b2, eps, grad_scale, decay, mode=1, t_first=1, steps=1):
    """fp64 Adam over `steps` steps from t_first; returns new (p, m, v) fp64 arrays."""
    p = np.ascontiguousarray(p, np.float64).copy()
    m = np.ascontiguousarray(m, np.float64).copy()
    v = np.ascontiguousarray(v, np.float64).copy()
    g = np.ascontiguousarray(g, np.float64)
    lib().oracle_adam(_p(p), _p(m), _p(v), _p(g), p.size, lr, b1, b2, eps, grad_scale,
                      decay, mode, t_first, steps)
    return p, m, v


def stencil(u, a0, a1, a2, T=1):
    """T sweeps of the 13-point operator over a full [nz][ny][nx] fp64 field."""
    a = np.ascontiguousarray(u, np.float64).copy()
    b = np.empty_like(a)
    nz, ny, nx = a.shape
    which = lib().oracle_stencil_run(_p(a), _p(b), nx, ny, nz, a0, a1, a2, int(T))
    return a if which == 0 else b


def xs_lower(e, E) -> int:
    e = np.ascontiguousarray(e, np.float64)
    return lib().oracle_xs_lower(_p(e), e.size, float(E))


def xs_lookup(t: dict, L: int, seed: int, i0: int = 0, want_mat=False):
    macro = np.empty((L, 5), np.float64)
    idx = np.empty(L, np.uint32)
    mat = np.empty(L, np.int32) if want_mat else None
    c = {k: np.ascontiguousarray(t[k]) for k in ("egrid", "recs", "mat_nuc", "mat_off",
                                                    "mat_cnt", "conc", "cum")}
    assert c["mat_nuc"].dtype == np.int32 and c["recs"].dtype == np.float64
    lib().oracle_xs_lookup(_p(c["egrid"]), _p(c["recs"]), _p(c["mat_nuc"]), _p(c["mat_off"]),
                           _p(c["mat_cnt"]), _p(c["conc"]), _p(c["cum"]), seed, i0, L,
                           t["n_nuc"], t["n_grid"], t["n_mat"], _p(macro), _p(idx),
                           _p(mat) if want_mat else None)
    return (macro, idx, mat) if want_mat else (macro, idx)


def exp_s(x: float) -> float:
    return lib().oracle_exp_s(x)


def log_s(x: float) -> float:
    return lib().oracle_log_s(x)


def pow_s(a: float, b: float) -> float:
    return lib().oracle_pow_s(a, b)


SWEEP_FN = {"exp_s": 0, "log_s": 1, "pow_s": 2, "div": 3}


def spec_sweep(fn: str, start: int, count: int, b: float = 0.0) -> np.ndarray:
    """Per-65536-pattern chunk hashes of a spec routine over fp32 bit patterns
    [start, start+count) (oracle.h oracle_spec_sweep)."""
    assert count % 65536 == 0
    out = np.zeros(count // 65536, np.uint64)
    lib().oracle_spec_sweep(start, count, SWEEP_FN[fn], b, _p(out))
    return out


def micro(state: dict, *, nsub, dt, dz, ncalls=1):
    """Returns a new dict with th, qv, qc, qr updated and precip [ncol] (all fp32)."""
    out = {k: np.ascontiguousarray(state[k], np.float32).copy() for k in ("th", "qv", "qc", "qr")}
    rho = np.ascontiguousarray(state["rho"], np.float32)
    pk = np.ascontiguousarray(state["pk"], np.float32)
    p = np.ascontiguousarray(state["p"], np.float32)
    ncol, nz = rho.shape
    assert nz <= 256
    precip = np.zeros(ncol, np.float32)
    lib().oracle_micro(_p(out["th"]), _p(out["qv"]), _p(out["qc"]), _p(out["qr"]), _p(rho),
                       _p(pk), _p(p), _p(precip), ncol, nz, int(nsub), float(dt), float(dz),
                       int(ncalls))
    out["precip"] = precip
    return out
