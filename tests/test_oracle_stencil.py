"""Pins for the 13-point stencil oracle (-m "not gpu").

P1: with (a0, a1, a2) = (-90, 16, -1) one sweep is 12*Laplacian, exact for integer
    polynomials of total degree <= 5 (4th-order central differences are exact there);
    the reference is the analytic Laplacian in int64.
P2: with the dyadic kappa = 12/128 coefficients and u0 = x^2 + y^2 + z^2 every point at
    index distance d >= 2T from the array edge satisfies u_T = u0 + 0.5625 T exactly.
"""
import numpy as np
import pytest

import synthetic


def analytic_12_laplacian(nx, ny, nz, coefs):
    out = np.zeros((nz, ny, nx), np.int64)
    for c, a, b, d in coefs:
        if a >= 2:
            out += synthetic.polynomial_field(nx, ny, nz, [(12 * c * a * (a - 1), a - 2, b, d)])
        if b >= 2:
            out += synthetic.polynomial_field(nx, ny, nz, [(12 * c * b * (b - 1), a, b - 2, d)])
        if d >= 2:
            out += synthetic.polynomial_field(nx, ny, nz, [(12 * c * d * (d - 1), a, b, d - 2)])
    return out


POLYS = [
    [(3, 2, 0, 0), (-2, 0, 2, 0), (5, 0, 0, 2)],
    [(1, 5, 0, 0), (-1, 0, 5, 0), (2, 0, 0, 5)],
    [(7, 2, 2, 1), (-3, 1, 3, 1), (1, 0, 1, 4), (8, 1, 1, 1), (-5, 0, 0, 0)],
    [(2, 3, 1, 1), (-1, 2, 0, 3), (4, 1, 4, 0)],
]


@pytest.mark.parametrize("coefs", POLYS)
@pytest.mark.parametrize("shape", [(20, 17, 13), (9, 40, 11)])
def test_p1_exact_laplacian_of_quintics(orc, coefs, shape):
    nx, ny, nz = shape
    u = synthetic.polynomial_field(nx, ny, nz, coefs)
    assert np.abs(u).max() < 2 ** 40
    w = orc.stencil(u.astype(np.float64), -90.0, 16.0, -1.0, T=1)
    lap = analytic_12_laplacian(nx, ny, nz, coefs)
    interior = (slice(2, nz - 2), slice(2, ny - 2), slice(2, nx - 2))
    np.testing.assert_array_equal(w[interior], lap[interior].astype(np.float64))
    frame = np.ones((nz, ny, nx), bool)
    frame[interior] = False
    np.testing.assert_array_equal(w[frame], u[frame].astype(np.float64))


def test_p1_degree_six_is_not_exact(orc):
    """Negative control: the pin can fail (x^6 has a nonzero 6th derivative)."""
    coefs = [(1, 6, 0, 0)]
    u = synthetic.polynomial_field(16, 9, 9, coefs)
    w = orc.stencil(u.astype(np.float64), -90.0, 16.0, -1.0, T=1)
    lap = analytic_12_laplacian(16, 9, 9, coefs)
    assert not np.array_equal(w[2:-2, 2:-2, 2:-2], lap[2:-2, 2:-2, 2:-2])


@pytest.mark.parametrize("T", [1, 2, 3, 5, 8])
def test_p2_light_cone_closed_form(orc, T):
    n = 48
    u0 = synthetic.polynomial_field(n, n, n, [(1, 2, 0, 0), (1, 0, 2, 0), (1, 0, 0, 2)])
    u0 = u0.astype(np.float64)
    a0, a1, a2 = synthetic.STENCIL_COEFFS
    uT = orc.stencil(u0, a0, a1, a2, T=T)
    i = np.arange(n)
    d1 = np.minimum(i, n - 1 - i)
    D = np.minimum(np.minimum(d1[:, None, None], d1[None, :, None]), d1[None, None, :])
    cone = D >= 2 * T
    np.testing.assert_array_equal(uT[cone], u0[cone] + 0.5625 * T)
    # the Dirichlet frame never changes
    np.testing.assert_array_equal(uT[D < 2], u0[D < 2])
    # the closed form stops holding just outside the cone (tightness, T >= 2)
    if T >= 2:
        ring = (D == 2 * T - 2)
        assert not np.array_equal(uT[ring], u0[ring] + 0.5625 * T)


def test_sweeps_are_thread_count_independent(orc):
    u0 = synthetic.stencil_inputs(24, 20, 18)
    a0, a1, a2 = synthetic.STENCIL_COEFFS
    old = orc.set_threads(1)
    a = orc.stencil(u0, a0, a1, a2, T=4)
    orc.set_threads(4)
    b = orc.stencil(u0, a0, a1, a2, T=4)
    orc.set_threads(old)
    np.testing.assert_array_equal(a, b)
