"""compute-sanitizer over every workload kernel, generic and specialized, at small
ragged sizes (memcheck, racecheck, synccheck; plus initcheck)."""
import os
import shutil
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SAN = shutil.which("compute-sanitizer") or "/usr/local/cuda/bin/compute-sanitizer"


@pytest.mark.parametrize("tool", ["memcheck", "racecheck", "synccheck", "initcheck"])
def test_compute_sanitizer_clean(tool):
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    if not os.path.exists(SAN):
        pytest.skip("compute-sanitizer not found")
    cmd = [SAN, "--tool", tool, "--error-exitcode", "17", "--print-limit", "20"]
    cmd += [sys.executable, os.path.join(ROOT, "scripts", "sanitize_run.py")]
    env = dict(os.environ, PYTHONPATH=ROOT, CUDA_CACHE_DISABLE="1")
    r = subprocess.run(cmd, env=env, capture_output=True, text=True, timeout=900)
    out = r.stdout + r.stderr
    if "compute-sanitizer is closed" in out:
        # the GPU pool refuses compute-sanitizer (its runs left GPUs needing a reset): the
        # wrapper exits 86 before any kernel runs, so there is nothing to judge
        pytest.skip(out.strip().splitlines()[-1][:200])
    assert r.returncode == 0 and "sanitize-run ok" in out, out[-4000:]
    clean = ("RACECHECK SUMMARY: 0 hazards displayed (0 errors, 0 warnings)" if tool == "racecheck"
             else "ERROR SUMMARY: 0 errors")
    assert clean in out, out[-4000:]
