"""Pins for the Adam oracle against closed forms (-m "not gpu").

Reading (DESIGN.md R-adam-*): m, v from zero; bias corrections bc_t = fp32(1 - b^t);
mode 1 = eps outside the sqrt, mode 0 = eps inside; decay coupled into the update.
"""
import numpy as np
import pytest

import synthetic

S = synthetic.ADAM_SCALARS
f32 = lambda x: float(np.float32(x))


def _scalars():
    return dict(lr=f32(S["lr"]), b1=f32(S["b1"]), b2=f32(S["b2"]), eps=f32(S["eps"]),
                grad_scale=f32(S["grad_scale"]), decay=f32(S["decay"]))


@pytest.mark.parametrize("mode", [0, 1])
def test_one_step_from_zero_moments(orc, mode):
    p0, m0, v0, g = synthetic.adam_inputs(4099)
    sc = _scalars()
    p, m, v = orc.adam(p0, m0, v0, g, mode=mode, steps=1, **sc)
    gs = g.astype(np.float64) / sc["grad_scale"]
    if mode == 1:
        s = gs / (np.abs(gs) + sc["eps"])
    else:
        s = gs / np.sqrt(gs * gs + sc["eps"])
    want = p0 - sc["lr"] * (s + sc["decay"] * p0.astype(np.float64))
    np.testing.assert_allclose(p, want, rtol=1e-13, atol=0)
    np.testing.assert_allclose(m, (1 - sc["b1"]) * gs, rtol=1e-15, atol=0)
    np.testing.assert_allclose(v, (1 - sc["b2"]) * gs * gs, rtol=1e-15, atol=0)


@pytest.mark.parametrize("mode", [0, 1])
@pytest.mark.parametrize("decay", [0.0, 0.01])
def test_constant_gradient_closed_form(orc, mode, decay):
    """mh = gs and vh = gs^2 for every t (real arithmetic), so with a = 1 - lr*decay:
    p_T = a^T p0 - lr*s*(1 - a^T)/(1 - a)   (= p0 - T*lr*s when decay = 0)."""
    n, T = 2048, 100
    p0, m0, v0, _ = synthetic.adam_inputs(n)
    p0 = p0.astype(np.float64)
    # gradients spanning 1e-6..16 so eps matters for the small ones
    g = (np.logspace(-6, np.log10(16.0), n) * np.where(np.arange(n) % 2, 1, -1)).astype(np.float32)
    sc = _scalars()
    sc["decay"] = f32(decay)
    p, _, _ = orc.adam(p0, m0, v0, g, mode=mode, steps=T, **sc)
    gs = g.astype(np.float64) / sc["grad_scale"]
    s = gs / (np.abs(gs) + sc["eps"]) if mode == 1 else gs / np.sqrt(gs * gs + sc["eps"])
    lr = sc["lr"]
    if decay == 0.0:
        want = p0 - T * lr * s
    else:
        a = 1.0 - lr * sc["decay"]
        want = a ** T * p0 - lr * s * (1 - a ** T) / (1 - a)
    # bc_t is rounded to fp32, so mh = gs (1 + d), |d| <= 2^-24 per step; bound the drift
    np.testing.assert_allclose(p, want, rtol=0, atol=T * lr * 4e-7)


def test_zero_gradient_is_pure_decay(orc):
    p0, m0, v0, _ = synthetic.adam_inputs(1000)
    g = np.zeros_like(p0)
    sc = _scalars()
    p, m, v = orc.adam(p0, m0, v0, g, mode=1, steps=37, **sc)
    assert not m.any() and not v.any()
    want = (1 - sc["lr"] * sc["decay"]) ** 37 * p0.astype(np.float64)
    np.testing.assert_allclose(p, want, rtol=1e-13)


def test_steps_compose(orc):
    """100 steps in one call == 60 steps then 40 steps starting at t = 61."""
    p0, m0, v0, g = synthetic.adam_inputs(3000)
    sc = _scalars()
    a = orc.adam(p0, m0, v0, g, steps=100, **sc)
    b = orc.adam(p0, m0, v0, g, steps=60, **sc)
    b = orc.adam(*b, g, t_first=61, steps=40, **sc)
    for x, y in zip(a, b):
        np.testing.assert_array_equal(x, y)
