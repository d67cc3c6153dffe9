"""NEXT-2 on one B200: the stencil's z-slab halo exchange fused into the kernel's stores
over peer memory, ordered by stream flags (halo.P2PZSlabStencil, stencil4_p2p).

* in one process: P "ranks" with their own arenas and streams, wired with plain device
  pointers -> equals the single-slab sweep (generic: bit-exact; specialized: tolerance)
  and the oracle;
* across two processes sharing the GPU: the same protocol with CUDA IPC mappings
  (proteus_ipc_get_handle / proteus_ipc_open_handle) -> equals the oracle.
"""
import os
import subprocess
import sys

import numpy as np
import pytest

import synthetic
from parity import compare

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def rt(tmp_path_factory):
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import oracle
    oracle.build()
    from paper_conf_cgo_georgakoudispb25_b200 import halo
    from paper_conf_cgo_georgakoudispb25_b200 import proteus as P
    from paper_conf_cgo_georgakoudispb25_b200 import workloads as W
    torch.zeros(1, device="cuda")
    P.proteus_finalize()
    P.testing_use_fake_backend(0)
    P.proteus_init(device=torch.cuda.current_device(),
                   cache_dir=str(tmp_path_factory.mktemp("p2pcache")), mode="all")
    ks = {e: W.register(e) for e in ("stencil4_ws", "stencil4_p2p")}
    yield dict(P=P, W=W, halo=halo, k=ks, oracle=oracle)
    torch.cuda.synchronize()
    P.proteus_finalize()


def _single(rt, u0, T, variant):
    W = rt["W"]
    nz, ny, nx = u0.shape
    slab = np.zeros((nz + 4, ny, nx))
    slab[2:nz + 2] = u0
    a = torch.from_numpy(slab).cuda()
    b = a.clone()
    co = synthetic.STENCIL_COEFFS
    Ls = [W.stencil_launch(rt["k"]["stencil4_ws"], a, b, nx=nx, ny=ny, nzl=nz, kg0=0, nzg=nz,
                           coeffs=co),
          W.stencil_launch(rt["k"]["stencil4_ws"], b, a, nx=nx, ny=ny, nzl=nz, kg0=0, nzg=nz,
                           coeffs=co)]
    for t in range(T):
        Ls[t % 2](variant)
    torch.cuda.synchronize()
    return (a if T % 2 == 0 else b).cpu().numpy()[2:nz + 2]


@pytest.mark.parametrize("P_,shape,T", [(2, (40, 36, 32), 5), (4, (64, 38, 32), 6),
                                        (8, (130, 66, 64), 3), (2, (256, 256, 256), 2)])
def test_p2p_local_ranks_match_single_slab(rt, P_, shape, T):
    nx, ny, nz = shape
    u0 = synthetic.stencil_inputs(nx, ny, nz)
    co = synthetic.STENCIL_COEFFS
    want = rt["oracle"].stencil(u0, *co, T=T) if nx * ny * nz <= 10 ** 6 else None
    for variant in ("aot", "jit"):
        got, flags = rt["halo"].run_slabs_p2p_local(rt["k"]["stencil4_p2p"], u0, T, P_, co,
                                                    variant=variant)
        ref = _single(rt, u0, T, variant)
        if variant == "aot":
            np.testing.assert_array_equal(got, ref)
        else:
            compare(got, ref, name="p2p-jit-vs-single")
        if want is not None:
            compare(got, want, name=f"p2p-{variant}-vs-oracle")
        # every existing neighbour signalled each of the T sweeps
        for r, (fl, fr) in enumerate(flags):
            assert fl == (T if r > 0 else 0) and fr == (T if r < P_ - 1 else 0), flags


def test_p2p_polynomial_exact_across_ranks(rt):
    """Pin P1 through the fused exchange: 12*Laplacian of a quintic, bit-exact, P = 4."""
    nx, ny, nz = 46, 38, 32
    coefs = [(1, 5, 0, 0), (-2, 0, 3, 2), (3, 1, 1, 3), (7, 2, 0, 0), (1, 0, 0, 5)]
    u = synthetic.polynomial_field(nx, ny, nz, coefs).astype(np.float64)
    want = rt["oracle"].stencil(u, -90.0, 16.0, -1.0, T=1)
    for variant in ("aot", "jit"):
        got, _ = rt["halo"].run_slabs_p2p_local(rt["k"]["stencil4_p2p"], u, 1, 4,
                                                (-90.0, 16.0, -1.0), variant=variant)
        np.testing.assert_array_equal(got, want)


def test_p2p_two_processes_ipc_same_gpu(rt, tmp_path):
    """Two processes share the GPU, map each other's arenas with CUDA IPC and run the
    flag protocol; rank 0 checks the gathered field against the oracle."""
    script = os.path.join(ROOT, "tests", "p2p_worker.py")
    env = dict(os.environ, PYTHONPATH=ROOT + os.pathsep + os.path.join(ROOT, "tests"),
               P2P_OUT=str(tmp_path / "out.npy"))
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2",
           "--master-addr", "127.0.0.1", "--master-port", str(29500 + os.getpid() % 1000),
           script]
    r = subprocess.run(cmd, env=env, capture_output=True, text=True, timeout=240)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-3000:]
    got = np.load(tmp_path / "out.npy")
    nx, ny, nz, T = 48, 40, 32, 5
    u0 = synthetic.stencil_inputs(nx, ny, nz)
    want = rt["oracle"].stencil(u0, *synthetic.STENCIL_COEFFS, T=T)
    compare(got, want, name="p2p-ipc-vs-oracle")
