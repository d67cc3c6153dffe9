"""Degenerate inputs through the C ABI (-m gpu): empty workloads launch cleanly in both
variants and write nothing.  Each output is an empty view into the middle of a larger
buffer filled with a sentinel pattern; the buffer must come back unchanged."""
import numpy as np
import pytest

import synthetic

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

SENT = 0x7FC0DEAD   # a NaN payload no kernel produces


@pytest.fixture(scope="module")
def rt(tmp_path_factory):
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_cgo_georgakoudispb25_b200 import proteus as P
    from paper_conf_cgo_georgakoudispb25_b200 import workloads as W
    torch.zeros(1, device="cuda")
    P.proteus_finalize()
    P.testing_use_fake_backend(0)
    P.proteus_init(device=torch.cuda.current_device(),
                   cache_dir=str(tmp_path_factory.mktemp("jitcache")), mode="all")
    ks = {name: W.register(name) for name in ("adam_step", "adam_run", "micro_column",
                                              "xs_lookup", "xs_index", "xs_bin", "xs_scan",
                                              "xs_scatter")}
    yield dict(P=P, W=W, k=ks)
    torch.cuda.synchronize()
    P.proteus_finalize()


def guarded(dtype, shape_tail=(), pad=64):
    """(buffer, empty view at offset pad): the view has 0 rows of shape_tail."""
    row = int(np.prod(shape_tail)) if shape_tail else 1
    buf = torch.empty(2 * pad * row, dtype=torch.int32 if dtype == torch.float32 else torch.int64,
                      device="cuda")
    buf.fill_(SENT if dtype == torch.float32 else (SENT << 32) | SENT)
    view = buf.view(dtype)[pad * row:pad * row].view((0,) + tuple(shape_tail))
    return buf, view


def untouched(buf, dtype):
    want = SENT if dtype == torch.float32 else (SENT << 32) | SENT
    return bool((buf == want).all())


@pytest.mark.parametrize("variant", ["aot", "jit"])
def test_adam_empty(rt, variant):
    W, S = rt["W"], synthetic.ADAM_SCALARS
    sc = dict(lr=S["lr"], b1=S["b1"], b2=S["b2"], eps=S["eps"], grad_scale=S["grad_scale"],
              decay=S["decay"])
    bufs = [guarded(torch.float32) for _ in range(4)]
    t = [v for _, v in bufs]
    L = W.adam_launch(rt["k"]["adam_step"], *t, **sc)
    W.adam_set_step(L, 1)
    L(variant)
    W.adam_run_launch(rt["k"]["adam_run"], *t, steps=10, **sc)(variant)
    torch.cuda.synchronize()
    assert all(untouched(b, torch.float32) for b, _ in bufs)


@pytest.mark.parametrize("variant", ["aot", "jit"])
def test_micro_empty(rt, variant):
    W = rt["W"]
    bufs = {n: guarded(torch.float32, (64,)) for n in ("th", "qv", "qc", "qr", "rho", "pk", "p")}
    pb, pr = guarded(torch.float32)
    s = {n: v for n, (_, v) in bufs.items()}
    W.micro_launch(rt["k"]["micro_column"], s, pr, nz=64, nsub=2, dt=20.0, dz=250.0)(variant)
    torch.cuda.synchronize()
    assert all(untouched(b, torch.float32) for b, _ in bufs.values())
    assert untouched(pb, torch.float32)


@pytest.mark.parametrize("variant", ["aot", "jit"])
@pytest.mark.parametrize("sorted_", [False, True])
def test_xs_empty(rt, variant, sorted_):
    W = rt["W"]
    t = synthetic.xs_tables(n_grid=50)
    d = W.xs_device_tables(t, index_kernel=rt["k"]["xs_index"])
    mb, macro = guarded(torch.float64, (5,))
    ib, idx = guarded(torch.float32)            # 4-B words; the kernel writes u32
    if sorted_:
        W.XSStep(rt["k"], d, 0, synthetic.S0, macro, idx.view(torch.int32))(variant)
    else:
        W.xs_launch(rt["k"]["xs_lookup"], d, 0, synthetic.S0, macro,
                    idx.view(torch.int32))(variant)
    torch.cuda.synchronize()
    assert untouched(mb, torch.float64) and untouched(ib, torch.float32)
