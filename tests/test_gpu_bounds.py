"""Device bounds checks in place of compute-sanitizer (which the GPU pool refuses since
r02at): every workload kernel's specialization compiled with -DPROTEUS_CHECK
(proteus_device.h: PROTEUS_CHECK_IDX traps on an out-of-bounds index at the kernels'
global index computations -- the XS sort's bucket keys and perm slots, the lookup's slot,
gidx, record and result indices, the microphysics column ranges, the stencil's slab
stores, Adam's float4 index) and run at small ragged sizes (scripts/sanitize_run.py); a
trap fails the launch and the process."""
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_every_kernel_in_bounds_with_device_checks():
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    env = dict(os.environ, PYTHONPATH=ROOT, BOUNDS="1")
    r = subprocess.run([sys.executable, os.path.join(ROOT, "scripts", "sanitize_run.py")],
                       env=env, capture_output=True, text=True, timeout=900)
    out = r.stdout + r.stderr
    assert r.returncode == 0 and "sanitize-run ok" in out, out[-4000:]


_PROBE = r"""
import sys, tempfile, torch
sys.path.insert(0, {root!r})
from paper_conf_cgo_georgakoudispb25_b200 import proteus as P
torch.zeros(1, device="cuda")
P.proteus_init(device=0, cache_dir=tempfile.mkdtemp(), mode="all")
src = '#include "proteus_device.h"\nextern "C" __global__ void chk(int i, int n) {{ PROTEUS_CHECK_IDX(i, n); }}\n'
k = P.proteus_register_kernel("chk", src, [P.I32, P.I32], [], None, "-DPROTEUS_CHECK")
P.proteus_launch(k, (1,), (32,), [{i}, 3])
torch.cuda.synchronize()
print("probe ok")
"""


@pytest.mark.parametrize("i,traps", [(2, False), (3, True), (-1, True)])
def test_the_check_traps_out_of_bounds(i, traps):
    """Negative control: PROTEUS_CHECK_IDX(i, 3) traps for i = 3 and i = -1 (the launch
    fails, the process reports an error), not for i = 2."""
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    code = _PROBE.format(root=ROOT, i=i)
    r = subprocess.run([sys.executable, "-c", code], capture_output=True, text=True,
                       timeout=300)
    ok = r.returncode == 0 and "probe ok" in r.stdout
    assert ok != traps, (r.returncode, r.stdout[-500:], r.stderr[-1500:])
