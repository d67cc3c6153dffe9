"""CUDA path vs the CPU oracle, through the C ABI (-m gpu; needs a B200).

Every workload is run as the nvcc generic AOT kernel (proteus_launch_aot) and as the
NVRTC specialization (proteus_launch), on seeded synthetic inputs, and compared element
by element with the oracle under tests/parity.py's rule: fp32 1e-5, fp64 1e-12 relative,
integers bit-exact; the microphysics path is reproducible fp32 and must be bit-exact.
Sizes span several tiles with ragged tails; the BASELINE.json full-size launch
configurations are checked on samples the oracle computes one by one.
"""
import os

import numpy as np
import pytest

import synthetic
from parity import compare

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def rt(tmp_path_factory):
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import oracle
    oracle.build()
    from paper_conf_cgo_georgakoudispb25_b200 import proteus as P
    from paper_conf_cgo_georgakoudispb25_b200 import workloads as W
    torch.cuda.init()
    torch.zeros(1, device="cuda")
    P.proteus_finalize()
    P.testing_use_fake_backend(0)
    P.proteus_init(device=torch.cuda.current_device(),
                   cache_dir=str(tmp_path_factory.mktemp("jitcache")), mode="all")
    ks = {name: W.register(name) for name in W.SPECS}
    yield dict(P=P, W=W, k=ks, oracle=oracle)
    torch.cuda.synchronize()
    P.proteus_finalize()


def run(L, variant):
    L(variant)
    torch.cuda.synchronize()


# ----------------------------------------------------------------------------- daxpy
@pytest.mark.parametrize("n", [1, 1000, (1 << 20) + 3])
def test_daxpy_end_to_end(rt, n):
    W = rt["W"]
    g = torch.Generator().manual_seed(n)
    x = torch.randn(n, dtype=torch.float64, generator=g)
    y0 = torch.randn(n, dtype=torch.float64, generator=g)
    want = 2.5 * x.numpy() + y0.numpy()
    for variant in ("aot", "jit"):
        y = y0.cuda()
        run(W.daxpy_launch(rt["k"]["daxpy"], 2.5, x.cuda(), y), variant)
        compare(y.cpu().numpy(), want, name=f"daxpy-{variant}")


# ----------------------------------------------------------------------------- Adam
def _adam_gpu(rt, n, steps, variant, mode=1):
    W = rt["W"]
    S = synthetic.ADAM_SCALARS
    p0, m0, v0, g = synthetic.adam_inputs(n)
    t = [torch.from_numpy(a).cuda() for a in (p0, m0, v0, g)]
    L = W.adam_launch(rt["k"]["adam_step"], *t, lr=S["lr"], b1=S["b1"], b2=S["b2"], eps=S["eps"],
                      grad_scale=S["grad_scale"], decay=S["decay"], mode=mode)
    for step in range(1, steps + 1):
        W.adam_set_step(L, step)
        L(variant)
    torch.cuda.synchronize()
    return [a.cpu().numpy() for a in t[:3]], (p0, m0, v0, g)


def _adam_oracle(rt, inputs, steps, mode=1):
    S = synthetic.ADAM_SCALARS
    f = lambda x: float(np.float32(x))
    p0, m0, v0, g = inputs
    return rt["oracle"].adam(p0, m0, v0, g, lr=f(S["lr"]), b1=f(S["b1"]), b2=f(S["b2"]),
                             eps=f(S["eps"]), grad_scale=f(S["grad_scale"]),
                             decay=f(S["decay"]), mode=mode, steps=steps)


@pytest.mark.parametrize("n,steps,mode", [(1000003, 100, 1), (4099, 100, 0), (5, 3, 1),
                                          (1 << 20, 20, 1)])
def test_adam_vs_oracle(rt, n, steps, mode):
    outs = {}
    for variant in ("aot", "jit"):
        (p, m, v), inputs = _adam_gpu(rt, n, steps, variant, mode)
        want = _adam_oracle(rt, inputs, steps, mode)
        for name, x, r in zip("pmv", (p, m, v), want):
            compare(x, r, rtol=1e-5, name=f"adam-{variant}-{name}")
        outs[variant] = (p, m, v)
    for a, b, name in zip(outs["aot"], outs["jit"], "pmv"):
        compare(b, a, rtol=1e-5, name=f"adam-jit-vs-aot-{name}")


@pytest.mark.parametrize("n,steps,mode", [(1000003, 100, 1), (4099, 100, 0), (5, 3, 1),
                                          (1 << 20, 20, 1)])
def test_adam_run_vs_oracle_and_per_step_launches(rt, n, steps, mode):
    """adam_run (the time loop in one launch, the paper's kernel form) vs the oracle, and vs
    `steps` adam_step launches (same per-step operations): within 1e-5 (the two kernels
    may contract differently); the bit-identical fraction is reported by compare()."""
    W = rt["W"]
    S = synthetic.ADAM_SCALARS
    p0, m0, v0, g = synthetic.adam_inputs(n)
    want = _adam_oracle(rt, (p0, m0, v0, g), steps, mode)
    for variant in ("aot", "jit"):
        t = [torch.from_numpy(a).cuda() for a in (p0, m0, v0, g)]
        run(W.adam_run_launch(rt["k"]["adam_run"], *t, lr=S["lr"], b1=S["b1"], b2=S["b2"],
                              eps=S["eps"], grad_scale=S["grad_scale"], decay=S["decay"],
                              steps=steps, mode=mode), variant)
        got = [a.cpu().numpy() for a in t[:3]]
        for name, x, r in zip("pmv", got, want):
            compare(x, r, rtol=1e-5, name=f"adam_run-{variant}-{name}")
        chain, _ = _adam_gpu(rt, n, steps, variant, mode)
        for name, x, r in zip("pmv", got, chain):
            compare(x, r, rtol=1e-5, name=f"adam_run-vs-steps-{variant}-{name}")


@pytest.mark.parametrize("lr", [0.0, 1e-30])
@pytest.mark.parametrize("mode", [0, 1])
def test_adam_run_degenerate_lr(rt, lr, mode):
    """lr = 0 and a vanishing lr (1e-30): R-adam-6 keeps L = lr/bc1 as a factor, so the
    folded step stays finite -- p unchanged (bit-exact for lr = 0), m and v still updated,
    no NaN -- in both builds (folding L into den as a divisor gave NaN here)."""
    W = rt["W"]
    S = synthetic.ADAM_SCALARS
    n, steps = 4099, 20
    p0, m0, v0, g = synthetic.adam_inputs(n)
    f = lambda x: float(np.float32(x))
    want = rt["oracle"].adam(p0, m0, v0, g, lr=f(lr), b1=f(S["b1"]), b2=f(S["b2"]),
                             eps=f(S["eps"]), grad_scale=f(S["grad_scale"]),
                             decay=f(S["decay"]), mode=mode, steps=steps)
    for variant in ("aot", "jit"):
        t = [torch.from_numpy(a).cuda() for a in (p0, m0, v0, g)]
        run(W.adam_run_launch(rt["k"]["adam_run"], *t, lr=lr, b1=S["b1"], b2=S["b2"],
                              eps=S["eps"], grad_scale=S["grad_scale"], decay=S["decay"],
                              steps=steps, mode=mode), variant)
        got = [a.cpu().numpy() for a in t[:3]]
        assert all(np.isfinite(x).all() for x in got), variant
        for name, x, r in zip("pmv", got, want):
            compare(x, r, rtol=1e-5, name=f"adam_run-lr{lr}-{variant}-{name}")
        if lr == 0.0:
            np.testing.assert_array_equal(got[0], p0)


def test_adam_run_split_equals_one_run(rt):
    """Two adam_run launches of 40 + 60 steps (t_first 1 and 41) give the 100-step run
    bit-exactly (generic kernel: same binary, same per-step operations)."""
    W = rt["W"]
    S = synthetic.ADAM_SCALARS
    n = 100003
    p0, m0, v0, g = synthetic.adam_inputs(n)
    sc = dict(lr=S["lr"], b1=S["b1"], b2=S["b2"], eps=S["eps"], grad_scale=S["grad_scale"],
              decay=S["decay"])
    a = [torch.from_numpy(x).cuda() for x in (p0, m0, v0, g)]
    run(W.adam_run_launch(rt["k"]["adam_run"], *a, steps=100, **sc), "aot")
    b = [torch.from_numpy(x).cuda() for x in (p0, m0, v0, g)]
    run(W.adam_run_launch(rt["k"]["adam_run"], *b, steps=40, **sc), "aot")
    run(W.adam_run_launch(rt["k"]["adam_run"], *b, steps=60, t_first=41, **sc), "aot")
    for x, y in zip(a[:3], b[:3]):
        np.testing.assert_array_equal(x.cpu().numpy(), y.cpu().numpy())


# ----------------------------------------------------------------------------- stencil
def _stencil_gpu(rt, u0, T, variant, coeffs, tile=None, zchunks=None, entry="stencil4"):
    W = rt["W"]
    nz, ny, nx = u0.shape
    slab = np.zeros((nz + 4, ny, nx))
    slab[2:nz + 2] = u0
    a = torch.from_numpy(slab).cuda()
    b = a.clone()
    Ls = [W.stencil_launch(rt["k"][entry], a, b, nx=nx, ny=ny, nzl=nz, kg0=0, nzg=nz,
                           coeffs=coeffs, tile=tile, zchunks=zchunks),
          W.stencil_launch(rt["k"][entry], b, a, nx=nx, ny=ny, nzl=nz, kg0=0, nzg=nz,
                           coeffs=coeffs, tile=tile, zchunks=zchunks)]
    for t in range(T):
        Ls[t % 2](variant)
    torch.cuda.synchronize()
    out = (a if T % 2 == 0 else b).cpu().numpy()
    return out[2:nz + 2]


@pytest.mark.parametrize("entry,shape,T", [
    ("stencil4", (40, 40, 40), 7), ("stencil4", (70, 37, 19), 4), ("stencil4", (256, 256, 256), 2),
    ("stencil4", (6, 5, 5), 3), ("stencil4", (98, 130, 9), 2), ("stencil4_smem", (45, 40, 40), 5),
    ("stencil4_ws", (40, 40, 40), 7), ("stencil4_ws", (70, 37, 19), 4),
    ("stencil4_ws", (256, 256, 256), 2), ("stencil4_ws", (6, 5, 5), 3),
    ("stencil4_ws", (130, 98, 9), 2),
    ("stencil4_smem", (5, 5, 5), 3), ("stencil4_smem", (256, 256, 256), 1)])
def test_stencil_random_vs_oracle(rt, entry, shape, T):
    nx, ny, nz = shape
    u0 = synthetic.stencil_inputs(nx, ny, nz)
    co = synthetic.STENCIL_COEFFS
    want = rt["oracle"].stencil(u0, *co, T=T)
    res = {}
    for variant in ("aot", "jit"):
        got = _stencil_gpu(rt, u0, T, variant, co, entry=entry)
        compare(got, want, name=f"{entry}-{variant}")
        res[variant] = got
    compare(res["jit"], res["aot"], name=f"{entry}-jit-vs-aot")


@pytest.mark.parametrize("entry,tile,zchunks", [
    ("stencil4", (32, 4), None), ("stencil4", (32, 2), 3), ("stencil4", (64, 2), 1),
    ("stencil4", (32, 8), 23), ("stencil4_ws", (32, 7), None), ("stencil4_ws", (32, 4), 3),
    ("stencil4_ws", (32, 1), 23), ("stencil4_ws", (32, 11), 2), ("stencil4_smem", (32, 8), None), ("stencil4_smem", (64, 4), 2),
    ("stencil4_smem", (32, 16), 7)])
def test_stencil_polynomial_exact(rt, entry, tile, zchunks):
    """Pin P1 on the GPU: 12*Laplacian of a quintic, bit-exact, any tile shape/z-split."""
    nx, ny, nz = (45 if entry == "stencil4_smem" else 46), 38, 23
    coefs = [(1, 5, 0, 0), (-2, 0, 3, 2), (3, 1, 1, 3), (7, 2, 0, 0)]
    u = synthetic.polynomial_field(nx, ny, nz, coefs).astype(np.float64)
    want = rt["oracle"].stencil(u, -90.0, 16.0, -1.0, T=1)
    for variant in ("aot", "jit"):
        got = _stencil_gpu(rt, u, 1, variant, (-90.0, 16.0, -1.0), tile=tile, zchunks=zchunks,
                           entry=entry)
        np.testing.assert_array_equal(got, want)


def test_stencil_light_cone(rt):
    n, T = 48, 6
    u0 = synthetic.polynomial_field(n, n, n, [(1, 2, 0, 0), (1, 0, 2, 0), (1, 0, 0, 2)]).astype(float)
    got = _stencil_gpu(rt, u0, T, "jit", synthetic.STENCIL_COEFFS)
    i = np.arange(n)
    d1 = np.minimum(i, n - 1 - i)
    D = np.minimum(np.minimum(d1[:, None, None], d1[None, :, None]), d1[None, None, :])
    np.testing.assert_array_equal(got[D >= 2 * T], u0[D >= 2 * T] + 0.5625 * T)


def test_stencil_slab_decomposition_matches_single(rt):
    """Pin P3 (host side of the z-slab decomposition): running the P=4 slabs one after
    another with halos copied between them equals the P=1 sweep bit-exactly (generic)."""
    from paper_conf_cgo_georgakoudispb25_b200 import halo
    nx = ny = 36
    nz, T, P_ = 32, 5, 4
    u0 = synthetic.stencil_inputs(nx, ny, nz)
    co = synthetic.STENCIL_COEFFS
    full = _stencil_gpu(rt, u0, T, "aot", co)
    got = halo.run_slabs_serial(rt["k"]["stencil4"], u0, T, P_, co, variant="aot")
    np.testing.assert_array_equal(got, full)
    got = halo.run_slabs_serial(rt["k"]["stencil4"], u0, T, P_, co, variant="jit")
    compare(got, full, name="slabs-jit")


# ----------------------------------------------------------------------------- XS lookup
@pytest.fixture(scope="module")
def xs_full(rt):
    t = synthetic.xs_tables()
    return t, rt["W"].xs_device_tables(t, index_kernel=rt["k"]["xs_index"])


def _noindex(d):
    d = dict(d)
    d["gidx"] = None
    return d


def test_xs_index_is_lower_of_bin_edges(rt, xs_full):
    """gidx[n][b] = lower(e_n, b/EBINS) -- checked against the oracle's bisection."""
    t, d = xs_full
    nb = rt["W"].XS_EBINS
    g = d["gidx"].cpu().numpy().reshape(t["n_nuc"], nb + 1)
    for n in (0, 7, 33, 67):
        for b in (0, 1, nb // 2 - 1, nb - 1, nb):
            assert g[n, b] == rt["oracle"].xs_lower(t["egrid"][n], b / float(nb))


def _xs_gpu(rt, d, L, variant, seed=synthetic.S0, block=None, grid=None, sorted_=False, steps=1):
    block = block or rt["W"].XS_BLOCK
    macro = torch.empty((L, 5), dtype=torch.float64, device="cuda")
    idx = torch.empty(L, dtype=torch.int32, device="cuda")
    if sorted_:
        step = rt["W"].XSStep(rt["k"], d, L, seed, macro, idx, block=block)
        for _ in range(steps):     # both counter parities are exercised for steps >= 2
            step(variant)
        torch.cuda.synchronize()
        raw = step.perm.cpu().numpy().view(np.uint32)
        assert np.array_equal(np.sort(raw & 0x0FFFFFFF), np.arange(L)), "perm is not a permutation"
        # the sort key is non-decreasing along perm: (material, EBINS-bin of E)
        nb = rt["W"].XS_EBINS
        ii = (raw & 0x0FFFFFFF).astype(np.uint64)
        E = synthetic.u01_f64(synthetic.rng(34, ii, seed))
        key = (raw >> 28).astype(np.int64) * nb + np.minimum((E * nb).astype(np.int64), nb - 1)
        assert (np.diff(key) >= 0).all(), "perm is not sorted by (material, energy bin)"
        # the bucket totals of the per-block counting sort add up to the lookups
        assert int(step.totals.sum().item()) == L
        # results are in event order (DESIGN R-xs-3): slot t holds lookup ii[t]
        m_s, i_s = macro.cpu().numpy(), idx.cpu().numpy().view(np.uint32)
        m, i = np.empty_like(m_s), np.empty_like(i_s)
        m[ii.astype(np.int64)] = m_s
        i[ii.astype(np.int64)] = i_s
        return m, i
    run(rt["W"].xs_launch(rt["k"]["xs_lookup"], d, L, seed, macro, idx, block=block,
                          grid=grid), variant)
    return macro.cpu().numpy(), idx.cpu().numpy().view(np.uint32)


@pytest.mark.parametrize("index", [False, True])
@pytest.mark.parametrize("sorted_", [False, True])
@pytest.mark.parametrize("L", [1, 1000, 100003])
def test_xs_vs_oracle(rt, xs_full, L, sorted_, index):
    t, d = xs_full
    d = d if index else _noindex(d)
    want_m, want_i = rt["oracle"].xs_lookup(t, L, synthetic.S0)
    for variant in ("aot", "jit"):
        m, i = _xs_gpu(rt, d, L, variant, sorted_=sorted_, steps=3)
        compare(i, want_i, name=f"xs-idx-{variant}")
        compare(m, want_m, name=f"xs-macro-{variant}")


def _xs_more_materials(t, n_mat):
    """t with materials 12 .. n_mat-1 added (copies of materials 1, 2, ... nuclide lists and
    concentrations), selection probabilities rescaled so the new ones get 4% each."""
    t = dict(t)
    extra = list(range(1, n_mat - len(t["mat_cnt"]) + 1))
    nuc = [t["mat_nuc"]] + [t["mat_nuc"][t["mat_off"][m]:t["mat_off"][m] + t["mat_cnt"][m]]
                            for m in extra]
    conc = [t["conc"]] + [t["conc"][t["mat_off"][m]:t["mat_off"][m] + t["mat_cnt"][m]]
                          for m in extra]
    t["mat_cnt"] = np.concatenate([t["mat_cnt"], t["mat_cnt"][extra]]).astype(np.int32)
    t["mat_off"] = np.concatenate([[0], np.cumsum(t["mat_cnt"])[:-1]]).astype(np.int32)
    t["mat_nuc"] = np.concatenate(nuc).astype(np.int32)
    t["conc"] = np.concatenate(conc)
    probs = np.diff(np.concatenate([[0.0], t["cum"]])) * (1.0 - 0.04 * len(extra))
    t["cum"] = np.cumsum(np.concatenate([probs, np.full(len(extra), 0.04)]))
    t["n_mat"] = n_mat
    return t


@pytest.mark.parametrize("n_mat", [13, 16])
def test_xs_sort_global_bucket_rows(rt, n_mat):
    """n_mat * XS_EBINS * 4 B > XS_BIN_SMEM_MAX (13..16 materials): xs_bin counts and
    xs_scatter places in their global rows instead of shared memory -- a product path the
    12-material configs never take.  Ragged L, both variants, vs the oracle."""
    t = _xs_more_materials(synthetic.xs_tables(n_grid=2000), n_mat)
    assert n_mat * rt["W"].XS_EBINS * 4 > rt["W"].XS_BIN_SMEM_MAX
    d = rt["W"].xs_device_tables(t, index_kernel=rt["k"]["xs_index"])
    L = 200003
    want_m, want_i, want_mat = rt["oracle"].xs_lookup(t, L, synthetic.S0, want_mat=True)
    assert (want_mat >= 12).sum() > 0.03 * (n_mat - 12) * L   # the new materials are drawn
    for variant in ("aot", "jit"):
        m, i = _xs_gpu(rt, d, L, variant, sorted_=True, steps=2)
        compare(i, want_i, name=f"xs-{n_mat}mat-idx-{variant}")
        compare(m, want_m, name=f"xs-{n_mat}mat-macro-{variant}")


def _xs_clustered(n_grid=2000, seed=7):
    """xs_tables with every nuclide's grid half uniform on (0, 1) and half packed into a
    narrow cluster (0.004 wide at E = 0.25 for even nuclides, 0.002 wide at 0.75 for odd
    ones): the energy bins there hold ~60 and ~120 grid points, so the warp-uniform path
    takes its wide-bracket branches (width 32..62 bisected in the bracket, >= 63 clamped
    in the packed shuffle word and bisected to the end of the row)."""
    t = dict(synthetic.xs_tables(n_grid=n_grid))
    r = np.random.default_rng(seed)
    eg = np.empty_like(t["egrid"])
    for n in range(t["n_nuc"]):
        c, w = (0.25, 0.004) if n % 2 == 0 else (0.75, 0.002)
        while True:
            pts = np.unique(np.concatenate([r.random(n_grid // 2), c + w * r.random(n_grid // 2)]))
            pts = pts[pts > 0.0]
            if pts.size >= n_grid:
                break
        eg[n] = np.sort(r.choice(pts, n_grid, replace=False))
    t["egrid"] = eg
    t["recs"] = t["recs"].copy()
    t["recs"][:, :, 0] = eg
    return t


def test_xs_wide_brackets(rt):
    t = _xs_clustered()
    nb = rt["W"].XS_EBINS
    edges = np.arange(nb + 1) / nb
    w0 = np.diff(np.searchsorted(t["egrid"][0], edges, side="right"))
    w1 = np.diff(np.searchsorted(t["egrid"][1], edges, side="right"))
    assert ((w0 >= 32) & (w0 < 63)).any() and (w1 >= 63).any()   # both wide branches
    d = rt["W"].xs_device_tables(t, index_kernel=rt["k"]["xs_index"])
    L = 300007
    want_m, want_i = rt["oracle"].xs_lookup(t, L, synthetic.S0)
    for variant in ("aot", "jit"):
        for sorted_ in (True, False):
            m, i = _xs_gpu(rt, d, L, variant, sorted_=sorted_, steps=1)
            compare(i, want_i, name=f"xs-wide-idx-{variant}-{sorted_}")
            compare(m, want_m, name=f"xs-wide-macro-{variant}-{sorted_}")


@pytest.mark.parametrize("sorted_,index", [(False, False), (True, True)])
def test_xs_full_size_sampled(rt, xs_full, sorted_, index):
    """CFG 3 launch (10^7 lookups, block 256): samples of 20 x 5000 lookups vs oracle."""
    t, d = xs_full
    d = d if index else _noindex(d)
    L = 10 ** 7
    for variant in ("aot", "jit"):
        m, i = _xs_gpu(rt, d, L, variant, sorted_=sorted_, steps=2)
        for s in range(20):
            i0 = s * (L // 20) + 1234
            wm, wi = rt["oracle"].xs_lookup(t, 5000, synthetic.S0, i0=i0)
            compare(i[i0:i0 + 5000], wi, name=f"xs-full-idx-{variant}")
            compare(m[i0:i0 + 5000], wm, name=f"xs-full-macro-{variant}")


def test_xs_small_grid_and_grid_stride(rt):
    t = synthetic.xs_tables(n_grid=3)
    d = rt["W"].xs_device_tables(t, index_kernel=rt["k"]["xs_index"])
    L = 5000
    want_m, want_i = rt["oracle"].xs_lookup(t, L, synthetic.S0)
    m, i = _xs_gpu(rt, d, L, "jit", grid=3)   # grid-stride loop
    compare(i, want_i, name="xs3-idx")
    compare(m, want_m, name="xs3-macro")


# ----------------------------------------------------------------------------- microphysics
def _micro_gpu(rt, st, calls, variant, nz=64, nsub=2):
    W = rt["W"]
    s = {k: torch.from_numpy(v).cuda() for k, v in st.items()}
    precip = torch.zeros(st["th"].shape[0], dtype=torch.float32, device="cuda")
    L = W.micro_launch(rt["k"]["micro_column"], s, precip, nz=nz, nsub=nsub,
                       dt=synthetic.MICRO_DT, dz=synthetic.MICRO_DZ)
    for _ in range(calls):
        L(variant)
    torch.cuda.synchronize()
    out = {k: s[k].cpu().numpy() for k in ("th", "qv", "qc", "qr")}
    out["precip"] = precip.cpu().numpy()
    return out


@pytest.mark.parametrize("ncol,nz,calls", [(10000, 64, 100), (333, 64, 3), (257, 128, 5),
                                           (101, 32, 5), (7, 4, 2), (513, 100, 7), (64, 68, 4)])
def test_micro_bit_exact_vs_oracle(rt, ncol, nz, calls):
    st = synthetic.micro_inputs(ncol, nz)
    want = rt["oracle"].micro(st, nsub=2, dt=synthetic.MICRO_DT, dz=synthetic.MICRO_DZ,
                              ncalls=calls)
    for variant in ("aot", "jit"):
        got = _micro_gpu(rt, st, calls, variant, nz=nz)
        for k in ("th", "qv", "qc", "qr", "precip"):
            np.testing.assert_array_equal(got[k], want[k], err_msg=f"micro-{variant}-{k}")


def test_micro_full_size_sampled(rt):
    """CFG 4 launch (10^6 columns x 64): one call, 4000 sampled columns bit-exact."""
    ncol = 10 ** 6
    st = synthetic.micro_inputs(ncol, 64)
    cols = np.sort(np.random.default_rng(0).choice(ncol, 4000, replace=False))
    sub = {k: np.ascontiguousarray(v[cols]) for k, v in st.items()}
    want = rt["oracle"].micro(sub, nsub=2, dt=synthetic.MICRO_DT, dz=synthetic.MICRO_DZ, ncalls=1)
    for variant in ("aot", "jit"):
        got = _micro_gpu(rt, st, 1, variant)
        for k in ("th", "qv", "qc", "qr", "precip"):
            np.testing.assert_array_equal(got[k][cols], want[k], err_msg=f"micro-full-{variant}-{k}")


def test_micro_dry_column(rt):
    st = synthetic.micro_inputs(100, 64, dry=True)
    got = _micro_gpu(rt, st, 3, "jit")
    for k in ("th", "qv", "qc", "qr"):
        np.testing.assert_array_equal(got[k], st[k])
    assert not got["precip"].any()


# ----------------------------------------------------------------------------- runtime on GPU
def test_cache_counters_on_device(rt):
    P, W = rt["P"], rt["W"]
    k = W.register("daxpy")
    x = torch.ones(4096, dtype=torch.float64, device="cuda")
    y = torch.zeros_like(x)
    s0 = P.proteus_cache_stats()
    for a in (1.0, 2.0, 3.0, 1.0, 2.0, 3.0):
        W.daxpy_launch(k, a, x, y).jit()
    torch.cuda.synchronize()
    s1 = P.proteus_cache_stats()
    assert s1["compiles"] + s1["disk_hits"] - s0["compiles"] - s0["disk_hits"] == 3
    assert s1["mem_hits"] - s0["mem_hits"] == 3
    assert float(y[0]) == 12.0


def test_stencil_split_launches_equal_full(rt):
    """The N > 1 sweep issues three launches per slab (boundary planes {2,3}, {nzl,nzl+1},
    then the interior); on one GPU their union must equal the single full launch."""
    W = rt["W"]
    nx, ny, nz = 40, 33, 24
    u0 = synthetic.stencil_inputs(nx, ny, nz)
    co = synthetic.STENCIL_COEFFS
    full = _stencil_gpu(rt, u0, 1, "jit", co)
    slab = np.zeros((nz + 4, ny, nx))
    slab[2:nz + 2] = u0
    a = torch.from_numpy(slab).cuda()
    b = torch.zeros_like(a)
    common = dict(nx=nx, ny=ny, nzl=nz, kg0=0, nzg=nz, coeffs=co)
    for kb, ke, zc in ((2, 4, 1), (nz, nz + 2, 1), (4, nz, None)):
        W.stencil_launch(rt["k"]["stencil4"], a, b, k_begin=kb, k_end=ke, zchunks=zc, **common).jit()
    torch.cuda.synchronize()
    np.testing.assert_array_equal(b.cpu().numpy()[2:nz + 2], full)


# ------------------------------------------------------------------ XS lookup, NEXT-3 table
@pytest.fixture(scope="module")
def xs_large(rt):
    t = synthetic.xs_tables_large()
    return t, rt["W"].xs_device_tables(t, index_kernel=rt["k"]["xs_index"])


@pytest.mark.parametrize("sorted_,index,L", [(True, True, 100003), (False, False, 20011),
                                             (False, True, 4099)])
def test_xs_large_table_vs_oracle(rt, xs_large, sorted_, index, L):
    """355 nuclides (225 MB of table, beyond L2), fuel = 321 nuclides."""
    t, d = xs_large
    d = d if index else _noindex(d)
    want_m, want_i = rt["oracle"].xs_lookup(t, L, synthetic.S0)
    for variant in ("aot", "jit"):
        m, i = _xs_gpu(rt, d, L, variant, sorted_=sorted_, steps=2)
        compare(i, want_i, name=f"xsL-idx-{variant}")
        compare(m, want_m, name=f"xsL-macro-{variant}")


def test_xs_large_full_size_sampled(rt, xs_large):
    """10^7 lookups on the large table in the suite's launch configuration (sorted +
    index): 10 x 3000-lookup samples vs the oracle."""
    t, d = xs_large
    L = 10 ** 7
    m, i = _xs_gpu(rt, d, L, "jit", sorted_=True, steps=1)
    for s in range(10):
        i0 = s * (L // 10) + 777
        wm, wi = rt["oracle"].xs_lookup(t, 3000, synthetic.S0, i0=i0)
        compare(i[i0:i0 + 3000], wi, name="xsL-full-idx")
        compare(m[i0:i0 + 3000], wm, name="xsL-full-macro")


# --------------------------------------------- microphysics spec routines, exhaustive
@pytest.mark.parametrize("fn,lo,hi,b", [("exp_s", 0, 1 << 32, 0.0), ("log_s", 0, 1 << 32, 0.0)]
                         + [("pow_s", 0, 0x7F800000, b) for b in (0.1364, 0.2046, 0.525, 0.875)]
                         + [("div", lo, lo + 0x7F800000, b) for lo in (0, 0x80000000)
                            for b in (250.0, 125.0, 1000.0, 1.7, -3.3e-7, 1e-19)])
def test_spec_routines_exhaustive_vs_oracle(rt, fn, lo, hi, b):
    """SURVEY §8c-4 unit pin: exp_s and log_s over ALL 2^32 fp32 bit patterns, pow_s(a, b)
    over every non-negative finite a for the scheme's four exponents, and the kernel's
    division div_s over every non-NaN dividend for divisors of the scheme's magnitudes --
    GPU (generic and specialized) bit-identical to the oracle (C division for "div"),
    compared as per-65536-input chunk hashes."""
    W = rt["W"]
    n = hi - lo
    fid = {"exp_s": 0, "log_s": 1, "pow_s": 2, "div": 3}[fn]
    want = rt["oracle"].spec_sweep(fn, lo, n, b)
    out = torch.zeros(n >> 16, dtype=torch.int64, device="cuda")
    for variant in ("aot", "jit"):
        out.zero_()
        run(W.Launch(rt["k"]["micro_spec_sweep"], (148 * 8,), (256,),
                     [lo, n, fid, b, out.data_ptr()], 0, torch.cuda.current_stream().cuda_stream),
            variant)
        got = out.cpu().numpy().view(np.uint64)
        bad = np.nonzero(got != want)[0]
        assert bad.size == 0, f"{fn}/{variant}: {bad.size} chunks differ, first at pattern " \
                              f"{hex(lo + int(bad[0]) * 65536)}"


@pytest.mark.parametrize("P_", [2, 3, 8])
def test_adam_sharded_equals_single(rt, P_):
    """Adam over parameter shards (shard.py: contiguous, 16-B aligned starts,
    no collective) equals the 1-GPU update -- bit-exact for the generic kernel (same binary,
    elementwise), within 1e-5 for the specialized one (per-shard n is folded)."""
    from paper_conf_cgo_georgakoudispb25_b200.shard import shard_views
    W, S = rt["W"], synthetic.ADAM_SCALARS
    sc = dict(lr=S["lr"], b1=S["b1"], b2=S["b2"], eps=S["eps"], grad_scale=S["grad_scale"],
              decay=S["decay"], steps=50)
    n = 1000003
    x0 = synthetic.adam_inputs(n)
    for variant in ("aot", "jit"):
        one = [torch.from_numpy(a).cuda() for a in x0]
        run(W.adam_run_launch(rt["k"]["adam_run"], *one, **sc), variant)
        sh = [torch.from_numpy(a).cuda() for a in x0]
        for r in range(P_):
            views, (lo, hi) = shard_views(sh, n, P_, r)
            if hi > lo:
                run(W.adam_run_launch(rt["k"]["adam_run"], *views, **sc), variant)
        for a, b, name in zip(one[:3], sh[:3], "pmv"):
            if variant == "aot":
                np.testing.assert_array_equal(b.cpu().numpy(), a.cpu().numpy())
            else:
                compare(b.cpu().numpy(), a.cpu().numpy(), rtol=1e-5, name=f"adam-shard-{name}")
