"""bench.py's N > 1 path on the one B200 this pool leases (-m gpu; VERDICT r01 "Next" 6).

Two ranks launched exactly as the driver's scaling run launches them (torch.distributed.run,
one process per rank) but sharing the GPU (BENCH_SHARE_GPU=1: the process group is gloo,
so the "nccl" halo option stages the exchanged planes through the host -- NCCL refuses two
ranks on one device).  For the fused P2P halo (CUDA-IPC peer stores + stream flags) and
for the process-group exchange with the three-launch split, the JSON line must come out
and the ranks' owned planes after a fixed number of sweeps must equal the oracle's
single-field run within 1e-12.
"""
import glob
import json
import os
import socket
import subprocess
import sys

import numpy as np
import pytest

import synthetic
from parity import compare

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


@pytest.mark.parametrize("halo,ranks", [("p2p", 2), ("nccl", 2), ("p2p", 4)])
def test_ranks_share_gpu_vs_oracle(tmp_path, halo, ranks):
    """2 ranks (edge ranks only) and 4 (two interior ranks: both neighbours' halos and
    flags) through the bench's own launch."""
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import oracle
    oracle.build()
    n, T = 64, 9
    dump = str(tmp_path / "slab")
    env = dict(os.environ, BENCH_SHARE_GPU="1")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", str(ranks),
           "--master-addr", "127.0.0.1", "--master-port", str(_free_port()),
           os.path.join(ROOT, "bench.py"), "--gpus", str(ranks), "--steps", "20", "--warmup", "3",
           "--field-n", str(n), "--no-e2e-jobs", "--e2e-processes", "0", "--halo", halo,
           "--dump-final", dump, "--dump-sweeps", str(T)]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=900, cwd=ROOT, env=env)
    assert r.returncode == 0, r.stderr[-4000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout
    d = json.loads(lines[0])
    assert d["n_gpus"] == ranks and d["value"] > 0
    assert f"world={ranks}" in r.stderr
    if halo == "p2p":
        assert d["config"]["halo"].startswith("p2p (validated bit-exact against the gloo"), d["config"]
    else:
        assert d["config"]["halo"].startswith("gloo"), d["config"]
    parts = sorted(glob.glob(dump + ".rank*.npy"))
    assert len(parts) == ranks
    got = np.concatenate([np.load(p) for p in parts])
    want = oracle.stencil(synthetic.stencil_inputs(n, n, n), *synthetic.STENCIL_COEFFS, T=T)
    compare(got, want, name=f"bench-{ranks}rank-{halo}")
