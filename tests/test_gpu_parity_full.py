"""Full-size and long-run parity, CUDA path vs the CPU oracle (-m gpu; VERDICT r01
"What's weak" 2).  Same rule as test_gpu_parity.py (tests/parity.py: fp64 1e-12, fp32
1e-5, integers bit-exact; microphysics bit-exact), but on EVERY output of the
BASELINE.json configurations instead of samples, over the long runs of SURVEY §8c-2 P4,
with an XS table whose lookups land exactly on grid energies (the tie rule), and through
the three-launch z-slab split the N > 1 stencil sweep uses.
"""
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
    torch.zeros(1, device="cuda")
    P.proteus_finalize()
    P.testing_use_fake_backend(0)
    P.proteus_init(device=torch.cuda.current_device(),
                   cache_dir=str(tmp_path_factory.mktemp("jitcache")), mode="all")
    ks = {name: W.register(name) for name in W.SPECS}
    yield dict(P=P, W=W, k=ks, oracle=oracle)
    torch.cuda.synchronize()
    P.proteus_finalize()


# ----------------------------------------------------------------------------- stencil
def _stencil_gpu(rt, u0, T, variant, entry="stencil4_ws"):
    W = rt["W"]
    nz, ny, nx = u0.shape
    slab = np.zeros((nz + 4, ny, nx))
    slab[2:nz + 2] = u0
    a = torch.from_numpy(slab).cuda()
    b = a.clone()
    co = synthetic.STENCIL_COEFFS
    Ls = [W.stencil_launch(rt["k"][entry], a, b, nx=nx, ny=ny, nzl=nz, kg0=0, nzg=nz, coeffs=co),
          W.stencil_launch(rt["k"][entry], b, a, nx=nx, ny=ny, nzl=nz, kg0=0, nzg=nz, coeffs=co)]
    for t in range(T):
        Ls[t % 2](variant)
    torch.cuda.synchronize()
    return (a if T % 2 == 0 else b).cpu().numpy()[2:nz + 2]


@pytest.mark.parametrize("n,T", [(256, 100), (40, 1000), (42, 999)])
def test_stencil_long_run_vs_oracle(rt, n, T):
    """random u0, T = 100 sweeps of the bench field (256^3, the bench
    kernel and launch), and T ~ 1000 at small N, within 1e-12 -- fp64 drift over the
    bench's sweep counts stays inside the tolerance."""
    u0 = synthetic.stencil_inputs(n, n, n)
    want = rt["oracle"].stencil(u0, *synthetic.STENCIL_COEFFS, T=T)
    for variant in ("aot", "jit"):
        compare(_stencil_gpu(rt, u0, T, variant), want, name=f"stencil-T{T}-{variant}")


@pytest.mark.parametrize("entry", ["stencil4_ws", "stencil4"])
@pytest.mark.parametrize("shape,P_,T", [((64, 48, 40), 2, 5), ((64, 48, 40), 4, 6),
                                        ((256, 256, 256), 8, 3), ((46, 33, 24), 3, 4)])
def test_zslab_three_launch_split_vs_oracle(rt, entry, shape, P_, T):
    """The N > 1 sweep of halo.ZSlabStencil (boundary planes {2,3} and {nzl, nzl+1}, halo
    exchange, interior) with P_ slabs in one process (the exchange as device copies):
    equal to the oracle's single-field run within 1e-12, for the bench kernel and v3."""
    from paper_conf_cgo_georgakoudispb25_b200 import halo
    nx, ny, nz = shape
    u0 = synthetic.stencil_inputs(nx, ny, nz)
    co = synthetic.STENCIL_COEFFS
    want = rt["oracle"].stencil(u0, *co, T=T)
    res = {}
    for variant in ("aot", "jit"):
        got = halo.run_slabs_split_local(rt["k"][entry], u0, T, P_, co, variant=variant)
        compare(got, want, name=f"zslab-{entry}-P{P_}-{variant}")
        res[variant] = got
    # the generic kernel is the same binary for every launch: the split equals the
    # single full-field launch bit-exactly
    np.testing.assert_array_equal(res["aot"], _stencil_gpu(rt, u0, T, "aot", entry=entry))


# ----------------------------------------------------------------------------- XS lookup
@pytest.fixture(scope="module")
def xs_full(rt):
    t = synthetic.xs_tables()
    return t, rt["W"].xs_device_tables(t, index_kernel=rt["k"]["xs_index"])


def _xs_gpu(rt, d, L, variant, sorted_, steps=1):
    W = rt["W"]
    macro = torch.empty((L, 5), dtype=torch.float64, device="cuda")
    idx = torch.empty(L, dtype=torch.int32, device="cuda")
    if sorted_:
        step = W.XSStep(rt["k"], d, L, synthetic.S0, macro, idx)
        for _ in range(steps):
            step(variant)
        torch.cuda.synchronize()
        # event order (DESIGN R-xs-3): slot t holds lookup ii[t]; back to lookup order
        ii = step.slot_lookups().cpu().numpy().astype(np.int64)
        assert np.array_equal(np.sort(ii), np.arange(L))
        m, i = np.empty((L, 5)), np.empty(L, np.uint32)
        m[ii] = macro.cpu().numpy()
        i[ii] = idx.cpu().numpy().view(np.uint32)
        return m, i
    dd = dict(d)
    dd["gidx"] = None
    W.xs_launch(rt["k"]["xs_lookup"], dd, L, synthetic.S0, macro, idx)(variant)
    torch.cuda.synchronize()
    return macro.cpu().numpy(), idx.cpu().numpy().view(np.uint32)


def test_xs_full_size_every_lookup(rt, xs_full):
    """CFG 3 at full size: all 10^7 lookups, in the bench's sorted + energy-bin-index step
    and in the plain one-thread-per-lookup launch, both variants: idx bit-exact, macro
    within 1e-12, and the XSBench-style argmax checksum equal."""
    t, d = xs_full
    L = 10 ** 7
    want_m, want_i = rt["oracle"].xs_lookup(t, L, synthetic.S0)
    chk = int((want_m.argmax(1) + 1).sum())
    for sorted_ in (True, False):
        for variant in ("aot", "jit"):
            m, i = _xs_gpu(rt, d, L, variant, sorted_, steps=2)
            tag = f"xs-all-{'sorted' if sorted_ else 'plain'}-{variant}"
            compare(i, want_i, name=tag + "-idx")
            compare(m, want_m, name=tag + "-macro")
            assert int((m.argmax(1) + 1).sum()) == chk, tag


def _xs_tie_tables(n_tie=3000, seed=7):
    """The CFG 3 table re-gridded so that the energies of the first n_tie lookups (stream
    34, the generator both sides use) are grid points of EVERY nuclide: E == e_n[g]
    exactly.  For every third nuclide the lowest such energy is also e_n[0], for every
    third + 1 the highest is e_n[G-1] (the clamp ends)."""
    t = synthetic.xs_tables()
    G = t["n_grid"]
    E = np.unique(synthetic.u01_f64(synthetic.rng(34, np.arange(n_tie, dtype=np.uint64))))
    rs = np.random.default_rng(seed)
    egrid = np.empty_like(t["egrid"])
    for n in range(t["n_nuc"]):
        rest = np.setdiff1d(t["egrid"][n], E)
        if n % 3 == 0:
            rest = rest[rest > E[0]]
        elif n % 3 == 1:
            rest = rest[rest < E[-1]]
        keep = np.sort(rs.choice(rest, G - E.size, replace=False))
        egrid[n] = np.sort(np.concatenate([E, keep]))
        assert (np.diff(egrid[n]) > 0).all()
    t["egrid"] = egrid
    t["recs"][:, :, 0] = egrid
    return t, n_tie


def _lo_bruteforce(e, E):
    """max{g in [0, G-2] : e[g] <= E}, 0 if none, by linear count."""
    return int(min(max(np.count_nonzero(e <= E) - 1, 0), e.size - 2))


def test_xs_tie_rule_on_device(rt):
    """Lookup energies exactly on grid points: lo = g (ties to the right), including
    E == e[0] (lo = 0) and E == e[G-1] (lo = G-2).  The device's idx equals a brute-force
    count over the grid and the oracle bit-exactly, macro within 1e-12, for the sorted +
    index step and the plain launch, both variants."""
    t, n_tie = _xs_tie_tables()
    d = rt["W"].xs_device_tables(t, index_kernel=rt["k"]["xs_index"])
    L = 100003
    want_m, want_i, mat = rt["oracle"].xs_lookup(t, L, synthetic.S0, want_mat=True)
    E = synthetic.u01_f64(synthetic.rng(34, np.arange(n_tie, dtype=np.uint64)))
    brute = np.array([sum(_lo_bruteforce(t["egrid"][nuc], E[i])
                          for nuc in t["mat_nuc"][t["mat_off"][mat[i]]:
                                                  t["mat_off"][mat[i]] + t["mat_cnt"][mat[i]]])
                      for i in range(0, n_tie, 7)], np.uint32)
    np.testing.assert_array_equal(want_i[0:n_tie:7], brute)
    hits0 = sum(E[i] == t["egrid"][n][0] for i in range(n_tie) for n in range(0, t["n_nuc"], 3))
    hitsG = sum(E[i] == t["egrid"][n][-1] for i in range(n_tie) for n in range(1, t["n_nuc"], 3))
    assert hits0 > 0 and hitsG > 0
    for sorted_ in (True, False):
        for variant in ("aot", "jit"):
            m, i = _xs_gpu(rt, d, L, variant, sorted_, steps=2)
            tag = f"xs-tie-{'sorted' if sorted_ else 'plain'}-{variant}"
            compare(i, want_i, name=tag + "-idx")
            compare(m, want_m, name=tag + "-macro")


# ----------------------------------------------------------------------------- microphysics
def _micro_gpu(rt, st, calls, variant):
    W = rt["W"]
    s = {k: torch.from_numpy(v).cuda() for k, v in st.items()}
    precip = torch.zeros(st["th"].shape[0], dtype=torch.float32, device="cuda")
    L = W.micro_launch(rt["k"]["micro_column"], s, precip, nz=st["th"].shape[1],
                       nsub=synthetic.MICRO_NSUB, dt=synthetic.MICRO_DT, dz=synthetic.MICRO_DZ)
    for _ in range(calls):
        L(variant)
    torch.cuda.synchronize()
    out = {k: s[k].cpu().numpy() for k in ("th", "qv", "qc", "qr")}
    out["precip"] = precip.cpu().numpy()
    return out


@pytest.mark.parametrize("ncol,calls", [(10 ** 6, 1), (10 ** 5, 100)])
def test_micro_every_column_bit_exact(rt, ncol, calls):
    """CFG 4: every column of the full 10^6 x 64 launch for one call, and 10^5 columns over
    the 100-call job, bit-exact (oracle == generic == specialized, DESIGN R-mp-2)."""
    st = synthetic.micro_inputs(ncol, 64)
    want = rt["oracle"].micro(st, nsub=synthetic.MICRO_NSUB, dt=synthetic.MICRO_DT,
                              dz=synthetic.MICRO_DZ, ncalls=calls)
    assert want["precip"].any() and (want["qr"] != st["qr"]).any()
    for variant in ("aot", "jit"):
        got = _micro_gpu(rt, st, calls, variant)
        for k in ("th", "qv", "qc", "qr", "precip"):
            np.testing.assert_array_equal(got[k], want[k], err_msg=f"micro-{variant}-{k}")


@pytest.mark.parametrize("nsub,nz,ncol", [(1, 64, 5000), (3, 64, 5000), (2, 128, 3001),
                                          (4, 32, 2049)])
def test_micro_other_substeps_and_levels_bit_exact(rt, nsub, nz, ncol):
    """Specializations of the annotated nsub and nz other than the config's (each folds
    into its own cubin): still bit-exact against the oracle, generic and specialized."""
    W = rt["W"]
    st = synthetic.micro_inputs(ncol, nz)
    want = rt["oracle"].micro(st, nsub=nsub, dt=synthetic.MICRO_DT, dz=synthetic.MICRO_DZ,
                              ncalls=3)
    for variant in ("aot", "jit"):
        s = {k: torch.from_numpy(v).cuda() for k, v in st.items()}
        pr = torch.zeros(ncol, dtype=torch.float32, device="cuda")
        L = W.micro_launch(rt["k"]["micro_column"], s, pr, nz=nz, nsub=nsub,
                           dt=synthetic.MICRO_DT, dz=synthetic.MICRO_DZ)
        for _ in range(3):
            L(variant)
        torch.cuda.synchronize()
        for k in ("th", "qv", "qc", "qr"):
            np.testing.assert_array_equal(s[k].cpu().numpy(), want[k], err_msg=f"{variant}-{k}")
        np.testing.assert_array_equal(pr.cpu().numpy(), want["precip"])


@pytest.mark.parametrize("block", [64, 256])
def test_xs_step_other_block_sizes(rt, xs_full, block):
    """The sorted step at block sizes other than the tuned 128 (other launch bounds and
    folded dims in the specialization): idx bit-exact, macro within 1e-12."""
    W = rt["W"]
    t, d = xs_full
    L = 200003
    macro = torch.empty((L, 5), dtype=torch.float64, device="cuda")
    idx = torch.empty(L, dtype=torch.int32, device="cuda")
    want_m, want_i = rt["oracle"].xs_lookup(t, L, synthetic.S0)
    for variant in ("aot", "jit"):
        step = W.XSStep(rt["k"], d, L, synthetic.S0, macro, idx, block=block)
        step(variant)
        torch.cuda.synchronize()
        ii = step.slot_lookups().cpu().numpy().astype(np.int64)
        m, i = np.empty((L, 5)), np.empty(L, np.uint32)
        m[ii] = macro.cpu().numpy()
        i[ii] = idx.cpu().numpy().view(np.uint32)
        compare(i, want_i, name=f"xs-block{block}-{variant}-idx")
        compare(m, want_m, name=f"xs-block{block}-{variant}-macro")


@pytest.mark.parametrize("shape,T", [((128, 64, 96), 9), ((64, 200, 48), 6)])
def test_stencil_non_cubic_vs_oracle(rt, shape, T):
    """nx != ny != nz (the folded nx, ny, nzl differ; partial y tiles), both variants."""
    nx, ny, nz = shape
    u0 = synthetic.stencil_inputs(nx, ny, nz)
    want = rt["oracle"].stencil(u0, *synthetic.STENCIL_COEFFS, T=T)
    for variant in ("aot", "jit"):
        compare(_stencil_gpu(rt, u0, T, variant), want, name=f"stencil-{shape}-{variant}")
