"""NEXT-1: the IR-level specialization path (PROTEUS_F_IR, mode "ir") on the
B200 (-m gpu) -- kernel LTO-IR compiled once with the annotated values and grid dims as
extern device constants, per key a constants module + nvJitLink -lto -- against the
oracle with the same rule as the source path: fp64 1e-12, fp32 1e-5, integers and the
reproducible-fp32 microphysics bit-exact (so the link honours -fmad=false: -fma=0)."""
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
                   cache_dir=str(tmp_path_factory.mktemp("ircache")), mode="ir")
    ks = {name: W.register(name) for name in W.SPECS}
    yield dict(P=P, W=W, k=ks, oracle=oracle)
    torch.cuda.synchronize()
    P.proteus_finalize()


@pytest.mark.parametrize("shape,T", [((64, 48, 40), 5), ((256, 256, 256), 3)])
def test_ir_stencil_vs_oracle(rt, shape, T):
    W = rt["W"]
    nx, ny, nz = shape
    u0 = synthetic.stencil_inputs(nx, ny, nz)
    co = synthetic.STENCIL_COEFFS
    want = rt["oracle"].stencil(u0, *co, T=T)
    slab = np.zeros((nz + 4, ny, nx))
    slab[2:nz + 2] = u0
    a = torch.from_numpy(slab).cuda()
    b = a.clone()
    k = rt["k"]["stencil4_ws"]
    Ls = [W.stencil_launch(k, a, b, nx=nx, ny=ny, nzl=nz, kg0=0, nzg=nz, coeffs=co),
          W.stencil_launch(k, b, a, nx=nx, ny=ny, nzl=nz, kg0=0, nzg=nz, coeffs=co)]
    for t in range(T):
        Ls[t % 2]("jit")
    torch.cuda.synchronize()
    got = (a if T % 2 == 0 else b).cpu().numpy()[2:nz + 2]
    compare(got, want, name="ir-stencil")
    st = rt["P"].proteus_cache_stats()
    assert st["ir_compiles"] >= 1 and st["compile_failures"] == 0, st


def test_ir_micro_bit_exact(rt):
    W = rt["W"]
    st = synthetic.micro_inputs(2000, 64)
    want = rt["oracle"].micro(st, nsub=2, dt=synthetic.MICRO_DT, dz=synthetic.MICRO_DZ, ncalls=5)
    s = {k: torch.from_numpy(v).cuda() for k, v in st.items()}
    pr = torch.zeros(2000, dtype=torch.float32, device="cuda")
    L = W.micro_launch(rt["k"]["micro_column"], s, pr, nz=64, nsub=2, dt=synthetic.MICRO_DT,
                       dz=synthetic.MICRO_DZ)
    for _ in range(5):
        L("jit")
    torch.cuda.synchronize()
    for k_ in ("th", "qv", "qc", "qr"):
        np.testing.assert_array_equal(s[k_].cpu().numpy(), want[k_], err_msg=k_)
    np.testing.assert_array_equal(pr.cpu().numpy(), want["precip"])


def test_ir_xs_step_vs_oracle(rt):
    W = rt["W"]
    t = synthetic.xs_tables()
    d = W.xs_device_tables(t, index_kernel=rt["k"]["xs_index"])
    L = 100003
    macro = torch.empty((L, 5), dtype=torch.float64, device="cuda")
    idx = torch.empty(L, dtype=torch.int32, device="cuda")
    step = W.XSStep(rt["k"], d, L, synthetic.S0, macro, idx)
    step("jit")
    torch.cuda.synchronize()
    ii = step.slot_lookups().cpu().numpy().astype(np.int64)
    m, i = np.empty((L, 5)), np.empty(L, np.uint32)
    m[ii] = macro.cpu().numpy()
    i[ii] = idx.cpu().numpy().view(np.uint32)
    want_m, want_i = rt["oracle"].xs_lookup(t, L, synthetic.S0)
    compare(i, want_i, name="ir-xs-idx")
    compare(m, want_m, name="ir-xs-macro")


def test_ir_adam_run_vs_oracle(rt):
    W = rt["W"]
    S = synthetic.ADAM_SCALARS
    n = 1000003
    p0, m0, v0, g = synthetic.adam_inputs(n)
    tt = [torch.from_numpy(a).cuda() for a in (p0, m0, v0, g)]
    W.adam_run_launch(rt["k"]["adam_run"], *tt, lr=S["lr"], b1=S["b1"], b2=S["b2"], eps=S["eps"],
                      grad_scale=S["grad_scale"], decay=S["decay"], steps=100)("jit")
    torch.cuda.synchronize()
    f = lambda x: float(np.float32(x))
    want = rt["oracle"].adam(p0, m0, v0, g, lr=f(S["lr"]), b1=f(S["b1"]), b2=f(S["b2"]),
                             eps=f(S["eps"]), grad_scale=f(S["grad_scale"]), decay=f(S["decay"]),
                             steps=100)
    for name, x, r in zip("pmv", tt[:3], want):
        compare(x.cpu().numpy(), r, rtol=1e-5, name=f"ir-adam-{name}")
