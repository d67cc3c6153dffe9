"""libproteus under ThreadSanitizer and AddressSanitizer+UBSan (CPU, fake backend):
tests/native/stress.cpp drives 8 launcher threads, async workers, LRU eviction, the disk
cap, counter snapshots and concurrent cache clears; the sanitizer must report nothing."""
import os
import shutil
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
RT = os.path.join(ROOT, "paper_conf_cgo_georgakoudispb25_b200", "csrc", "proteus")
INC = os.path.join(ROOT, "include")


def _build(tmp_path, san):
    from paper_conf_cgo_georgakoudispb25_b200 import _build as B
    B.gen_device_header()
    srcs = [os.path.join(d, f) for d in (RT, RT + "_testing") for f in sorted(os.listdir(d))
            if f.endswith(".cpp")]
    exe = str(tmp_path / f"stress_{san.split(',')[0]}")
    cmd = ["g++", "-std=c++17", "-O1", "-g", f"-fsanitize={san}", "-fno-omit-frame-pointer",
           f"-I{INC}", f"-I{RT}", os.path.join(ROOT, "tests", "native", "stress.cpp"), *srcs,
           "-o", exe, "-ldl", "-lpthread"]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0 and "sanitize" in r.stderr and "cannot find" in r.stderr:
        pytest.skip(f"{san} runtime not available: {r.stderr[-300:]}")
    assert r.returncode == 0, r.stderr[-3000:]
    return exe


@pytest.mark.parametrize("san", ["thread", "address,undefined"])
def test_runtime_clean_under_sanitizer(tmp_path, san):
    if not shutil.which("g++"):
        pytest.skip("no g++")
    exe = _build(tmp_path, san)
    env = dict(os.environ, TSAN_OPTIONS="halt_on_error=1 second_deadlock_stack=1",
               ASAN_OPTIONS="detect_leaks=1 halt_on_error=1",
               UBSAN_OPTIONS="halt_on_error=1 print_stacktrace=1")
    r = subprocess.run([exe, str(tmp_path / "cache"), "1500"], capture_output=True, text=True,
                       env=env, timeout=600)
    out = r.stdout + r.stderr
    assert r.returncode == 0 and "stress ok" in out, out[-5000:]
    for bad in ("WARNING: ThreadSanitizer", "ERROR: AddressSanitizer", "runtime error:",
                "ERROR: LeakSanitizer"):
        assert bad not in out, out[-5000:]
