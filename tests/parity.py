"""Comparison rule shared by the parity tests (SURVEY.md §8c-6 / DESIGN.md "Tolerances").

Per element: |x - r| <= rtol * max(|r|, phi * ||r||_inf), phi = 1/16, ||r||_inf per array.
rtol = 1e-5 for fp32 arrays, 1e-12 for fp64 (north_star), 0 for integers (bit-exact).
Alongside pass/fail we report the raw max relative error, the normwise error and the
fraction of bit-identical elements.
"""
import numpy as np

PHI = 1.0 / 16.0
RTOL = {np.dtype(np.float32): 1e-5, np.dtype(np.float64): 1e-12}


def compare(x, r, rtol=None, name=""):
    x = np.asarray(x)
    r = np.asarray(r)
    assert x.shape == r.shape, (name, x.shape, r.shape)
    if np.issubdtype(x.dtype, np.integer):
        bad = np.flatnonzero(x != r)
        assert bad.size == 0, f"{name}: {bad.size} integer mismatches, first at {bad[:5]}"
        return dict(name=name, bit_identical=1.0)
    if rtol is None:
        rtol = RTOL[x.dtype]
    xd = x.astype(np.float64)
    rd = r.astype(np.float64)
    inf = np.abs(rd).max() if rd.size else 0.0
    err = np.abs(xd - rd)
    lim = rtol * np.maximum(np.abs(rd), PHI * inf)
    ok = err <= lim
    with np.errstate(divide="ignore", invalid="ignore"):
        rel = np.where(rd != 0, err / np.abs(rd), np.where(err == 0, 0.0, np.inf))
    stats = dict(name=name, max_rel=float(rel.max()) if rel.size else 0.0,
                 normwise=float(err.max() / inf) if inf > 0 else float(err.max()),
                 bit_identical=float(np.mean(x == r.astype(x.dtype))) if x.size else 1.0)
    if not ok.all():
        idx = np.flatnonzero(~ok)[:5]
        raise AssertionError(f"{name}: {np.count_nonzero(~ok)} elements out of tolerance "
                             f"rtol={rtol}; first {idx}: got {xd.flat[idx]} want {rd.flat[idx]}; {stats}")
    return stats
