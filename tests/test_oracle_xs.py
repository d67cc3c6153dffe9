"""Pins for the cross-section lookup oracle (-m "not gpu").

* lower index vs a brute-force linear scan (bit-exact integers), incl. special cases
* material selection vs min{m : r < cum[m]} computed here with numpy
* linear-in-E tables: macro_c = sum conc * (alpha_c E + beta_c) (closed form, the
  interpolation is exact for linear data; extrapolation too)
"""
import numpy as np
import pytest

import synthetic


def brute_lower(e, E):
    G = len(e)
    best = 0
    for g in range(G - 1):        # candidates [0, G-2]
        if e[g] <= E:
            best = g
    return best


def test_lower_matches_linear_scan(orc):
    rs = np.random.default_rng(7)
    for G in (2, 3, 4, 5, 17, 64, 1000):
        e = np.sort(rs.random(G))
        while np.unique(e).size != G:
            e = np.sort(rs.random(G))
        Es = np.concatenate([rs.random(200), e, [e[0] - 1e-3, e[-1] + 1e-3, 0.0, 1.0]])
        for E in Es:
            assert orc.xs_lower(e, E) == brute_lower(e, E), (G, E)


def test_lower_special_cases(orc):
    e = np.linspace(0.1, 0.9, 11)
    for g in range(10):
        assert orc.xs_lower(e, e[g]) == g          # E on a grid point -> lo = g, f = 1
    assert orc.xs_lower(e, e[10]) == 9              # E = last point clamps to G-2
    assert orc.xs_lower(e, 0.05) == 0               # below the grid
    assert orc.xs_lower(e, 0.95) == 9               # above the grid


def _small_tables(n_nuc=68, n_grid=200):
    return synthetic.xs_tables(n_nuc=n_nuc, n_grid=n_grid)


def test_lookup_indices_and_material_vs_brute_force(orc):
    t = _small_tables()
    L = 3000
    macro, idx, mat = orc.xs_lookup(t, L, synthetic.S0, want_mat=True)
    ii = np.arange(L, dtype=np.uint64)
    E = synthetic.u01_f64(synthetic.rng(34, ii))
    r = synthetic.u01_f64(synthetic.rng(35, ii))
    want_mat = np.array([next((m for m in range(12) if rr < t["cum"][m]), 11) for rr in r])
    np.testing.assert_array_equal(mat, want_mat)
    for q in range(0, L, 7):
        m = want_mat[q]
        nucs = t["mat_nuc"][t["mat_off"][m]:t["mat_off"][m] + t["mat_cnt"][m]]
        want = sum(brute_lower(t["egrid"][n], E[q]) for n in nucs)
        assert idx[q] == want


@pytest.mark.parametrize("n_grid", [50, 11303])
def test_linear_tables_closed_form(orc, n_grid):
    t = _small_tables(n_nuc=68, n_grid=n_grid)
    rs = np.random.default_rng(3)
    alpha = rs.uniform(-2, 2, (68, 5))
    beta = rs.uniform(-1, 1, (68, 5))
    E = t["egrid"]
    t["recs"][:, :, 1:] = alpha[:, None, :] * E[:, :, None] + beta[:, None, :]
    L = 4000
    macro, _ = orc.xs_lookup(t, L, synthetic.S0)
    ii = np.arange(L, dtype=np.uint64)
    Eq = synthetic.u01_f64(synthetic.rng(34, ii))
    r = synthetic.u01_f64(synthetic.rng(35, ii))
    for q in range(L):
        m = next((mm for mm in range(12) if r[q] < t["cum"][mm]), 11)
        sl = slice(t["mat_off"][m], t["mat_off"][m] + t["mat_cnt"][m])
        nucs, conc = t["mat_nuc"][sl], t["conc"][sl]
        want = (conc[:, None] * (alpha[nucs] * Eq[q] + beta[nucs])).sum(axis=0)
        np.testing.assert_allclose(macro[q], want, rtol=1e-12, atol=1e-12)


def test_table_generator_invariants():
    t = _small_tables(n_nuc=68, n_grid=300)
    assert (np.diff(t["egrid"], axis=1) > 0).all()
    assert (t["egrid"] > 0).all() and (t["egrid"] < 1).all()
    assert t["mat_cnt"].sum() == 197 and t["mat_nuc"].size == 197
    assert list(t["mat_nuc"][:34]) == list(range(34))
    for m in range(12):
        s = t["mat_nuc"][t["mat_off"][m]:t["mat_off"][m] + t["mat_cnt"][m]]
        assert (np.diff(s) > 0).all() and s.min() >= 0 and s.max() < 68


def test_large_table_generator_and_lookup_vs_brute_force(orc):
    """NEXT-3 table shape (355 nuclides, 321-nuclide fuel) at a reduced grid: generator
    invariants, and the oracle's lo sums vs a linear scan on fuel and non-fuel lookups."""
    t = synthetic.xs_tables(n_nuc=synthetic.XS_NUC_LARGE, n_grid=64,
                            mat_counts=synthetic.XS_MAT_COUNTS_LARGE)
    assert (np.diff(t["egrid"], axis=1) > 0).all()
    assert t["mat_cnt"][0] == 321 and list(t["mat_nuc"][:321]) == list(range(321))
    assert t["mat_nuc"].size == sum(synthetic.XS_MAT_COUNTS_LARGE)
    for m in range(12):
        s = t["mat_nuc"][t["mat_off"][m]:t["mat_off"][m] + t["mat_cnt"][m]]
        assert (np.diff(s) > 0).all() and s.min() >= 0 and s.max() < 355
    L = 600
    _, idx, mat = orc.xs_lookup(t, L, synthetic.S0, want_mat=True)
    E = synthetic.u01_f64(synthetic.rng(34, np.arange(L, dtype=np.uint64)))
    assert (mat == 0).sum() > 30
    for q in range(0, L, 3):
        m = mat[q]
        nucs = t["mat_nuc"][t["mat_off"][m]:t["mat_off"][m] + t["mat_cnt"][m]]
        assert idx[q] == sum(brute_lower(t["egrid"][n], E[q]) for n in nucs)


def test_default_tables_unchanged_by_mat_counts_parameter():
    a = synthetic.xs_tables(n_nuc=68, n_grid=100)
    b = synthetic.xs_tables(n_nuc=68, n_grid=100, mat_counts=synthetic.XS_MAT_COUNTS)
    for k in ("egrid", "recs", "mat_nuc", "mat_off", "mat_cnt", "conc", "cum"):
        np.testing.assert_array_equal(a[k], b[k])


def test_full_table_every_lookup_index_vs_library_search(orc):
    """SURVEY §8c-3 pin at the CFG 3 table (68 x 11303): the oracle's idx (sum of lower
    indices over the lookup's material) for ALL of 10^5 lookups equals an independent
    evaluation of the definition lo = max{g in [0, G-2] : e[g] <= E} (0 if none) through
    numpy's searchsorted (a library binary search: #{g : e[g] <= E} - 1, clamped), and a
    brute-force linear scan agrees on a 1000-lookup subset."""
    t = synthetic.xs_tables()
    L = 10 ** 5
    macro, idx, mat = orc.xs_lookup(t, L, synthetic.S0, want_mat=True)
    E = synthetic.u01_f64(synthetic.rng(34, np.arange(L, dtype=np.uint64)))
    G = t["n_grid"]
    want = np.zeros(L, np.int64)
    for m in range(t["n_mat"]):
        sel = np.flatnonzero(mat == m)
        for n in t["mat_nuc"][t["mat_off"][m]:t["mat_off"][m] + t["mat_cnt"][m]]:
            lo = np.searchsorted(t["egrid"][n], E[sel], side="right") - 1
            want[sel] += np.clip(lo, 0, G - 2)
    np.testing.assert_array_equal(idx.astype(np.int64), want)
    def scan(e, x):        # max over every candidate g in [0, G-2] with e[g] <= x
        hit = np.flatnonzero(e[:G - 1] <= x)
        return int(hit[-1]) if hit.size else 0

    for q in range(0, L, L // 1000):
        m = mat[q]
        nucs = t["mat_nuc"][t["mat_off"][m]:t["mat_off"][m] + t["mat_cnt"][m]]
        assert idx[q] == sum(scan(t["egrid"][n], E[q]) for n in nucs)
