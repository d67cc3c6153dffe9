#!/usr/bin/env python
"""NVRTC compile time per specialization (backend 2: real NVRTC, no GPU needed).
Prints ms per compile for each workload kernel at its config shape, cold (first in
process) and steady, plus adam_step across distinct lr values."""
import os
import sys
import tempfile
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
from paper_conf_cgo_georgakoudispb25_b200 import proteus as P  # noqa: E402
from paper_conf_cgo_georgakoudispb25_b200 import workloads as W  # noqa: E402
import test_nvrtc_specialize as T  # noqa: E402

P.proteus_finalize()
if os.environ.get("REAL"):
    import torch
    torch.zeros(1, device="cuda")
else:
    P.testing_use_fake_backend(2)
P.proteus_init(device=0, cache_dir=tempfile.mkdtemp(), mode=os.environ.get("MODE", "all"))
for rep in range(3):
    for e, (g, b, args) in T.CASES.items():
        k = W.register(e, with_generic=False)
        a = list(args)
        # perturb an annotated value so every compile is a distinct key
        t0 = time.perf_counter()
        try:
            a_mod = a
            P.proteus_cache_clear(memory=True, disk=True)
            P.proteus_get_specialization(k, g, b, a_mod)
        except Exception as ex:
            print(e, "failed", ex)
            continue
        print(f"rep {rep} {e:14s} {1e3*(time.perf_counter()-t0):8.1f} ms", flush=True)
k = W.register("adam_step", with_generic=False)
ts = []
for i in range(20):
    args = [0, 0, 0, 0, 65536, 1e-3 * (1 + i / 4096), 0.9, 0.999, 1e-8, 1024.0, 0.01, 1, 0.1, 0.001]
    t0 = time.perf_counter()
    P.proteus_get_specialization(k, (64,), (256,), args)
    ts.append(1e3 * (time.perf_counter() - t0))
print("adam distinct lr ms:", " ".join(f"{t:.1f}" for t in ts))
st = P.proteus_cache_stats()
print("stats: compiles", st["compiles"], "compile_ms_total", round(st["compile_ms_total"], 1))
P.proteus_finalize()
