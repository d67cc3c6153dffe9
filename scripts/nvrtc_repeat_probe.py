#!/usr/bin/env python
"""Probe: NVRTC compile time of the same specialized source repeated in one process
(does anything cache?).  Dumps the specialized sources with the fake backend first.
  python scripts/nvrtc_repeat_probe.py"""
import os, sys, subprocess, tempfile
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OUT = tempfile.mkdtemp()
subprocess.run([sys.executable, "-c", f"""
import sys, tempfile; sys.path.insert(0, {ROOT!r}); sys.path.insert(0, {ROOT!r} + '/tests')
from paper_conf_cgo_georgakoudispb25_b200 import proteus as P
from paper_conf_cgo_georgakoudispb25_b200 import workloads as W
import test_nvrtc_specialize as T
P.testing_use_fake_backend(2)
P.proteus_init(device=0, cache_dir=tempfile.mkdtemp(), mode='all')
for e in ('stencil4_ws', 'micro_column', 'xs_lookup', 'adam_step'):
    g, b, args = T.CASES[e]
    k = W.register(e, with_generic=False)
    open({OUT!r} + '/' + e + '.cu', 'w').write(P.proteus_specialized_source(k, g, b, list(args)))
"""], check=True)
import ctypes, time, sys, glob
lib = ctypes.CDLL(sorted(glob.glob("/usr/local/cuda/lib64/libnvrtc.so*"))[0])
def comp(src, opts):
    prog = ctypes.c_void_p()
    assert lib.nvrtcCreateProgram(ctypes.byref(prog), src.encode(), b"k.cu", 0, None, None) == 0
    arr = (ctypes.c_char_p * len(opts))(*[o.encode() for o in opts])
    t0 = time.perf_counter()
    r = lib.nvrtcCompileProgram(prog, len(opts), arr)
    dt = (time.perf_counter() - t0) * 1e3
    if r != 0:
        n = ctypes.c_size_t(); lib.nvrtcGetProgramLogSize(prog, ctypes.byref(n)); b = ctypes.create_string_buffer(n.value); lib.nvrtcGetProgramLog(prog, b); print(b.value.decode()[:2000])
    lib.nvrtcDestroyProgram(ctypes.byref(prog))
    return dt
for f in [OUT + "/" + e + ".cu" for e in ("stencil4_ws", "micro_column", "xs_lookup", "adam_step")]:
    src = open(f).read()
    extra = ["-fmad=false"] if "micro" in f else []
    for arch, name in (("-arch=compute_100a", "ptx"), ("-arch=sm_100a", "cubin")):
        ts = [comp(src, [arch, "-std=c++17", "-minimal", f"-I{ROOT}/paper_conf_cgo_georgakoudispb25_b200/csrc/kernels"] + extra) for _ in range(6)]
        print(f, name, " ".join(f"{t:.0f}" for t in ts))
