#!/usr/bin/env python
"""NEXT-1 measurement: the IR-level path (mode "ir") against the source path (mode "all")
on one GPU -- per-key compile ms (first key of a kernel: kernel IR + constants + link;
further keys: constants + link only) for CFG 5's 10 adam_step keys and each workload's
kernel, and the kernel time of both builds (they should be the same code)."""
import json
import os
import statistics
import sys
import tempfile
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import synthetic  # noqa: E402
from paper_conf_cgo_georgakoudispb25_b200 import proteus as P  # noqa: E402
from paper_conf_cgo_georgakoudispb25_b200 import workloads as W  # noqa: E402

torch.zeros(1, device="cuda")
S = synthetic.ADAM_SCALARS
sc = dict(b1=S["b1"], b2=S["b2"], eps=S["eps"], grad_scale=S["grad_scale"], decay=S["decay"])
out = {}
for mode in ("all", "ir"):
    P.proteus_init(device=0, cache_dir=tempfile.mkdtemp(), mode=mode)
    k = W.register("daxpy")          # NVRTC's one-time initialisation outside the numbers
    P.proteus_get_specialization(k, (1,), (32,), [1.0, 32, 0, 0])
    k = W.register("adam_step")
    t = [torch.from_numpy(a).cuda() for a in synthetic.adam_inputs(1 << 16)]
    L = W.adam_launch(k, *t, lr=1e-3, **sc)
    per = []
    for i in range(10):
        L.set(5, float(np.float32(1e-3 * (1 + i / 4096))))
        t0 = time.perf_counter()
        L.jit()
        per.append((time.perf_counter() - t0) * 1e3)
    torch.cuda.synchronize()
    row = {"adam_step_key_ms": [round(x, 1) for x in per],
           "adam_step_later_keys_p50_ms": round(statistics.median(per[1:]), 1)}
    # stencil: first key and a second key (other a0), then kernel time
    n = 256
    slab = np.zeros((n + 4, n, n))
    slab[2:n + 2] = synthetic.stencil_inputs(n, n, n)
    a = torch.from_numpy(slab).cuda()
    b = a.clone()
    ks = W.register("stencil4_ws")
    times = []
    for a0 in (synthetic.STENCIL_COEFFS[0], 0.25):
        Ls = W.stencil_launch(ks, a, b, nx=n, ny=n, nzl=n, kg0=0, nzg=n,
                              coeffs=(a0,) + synthetic.STENCIL_COEFFS[1:])
        t0 = time.perf_counter()
        Ls.jit()
        torch.cuda.synchronize()
        times.append(round((time.perf_counter() - t0) * 1e3, 1))
    row["stencil_key_ms"] = times
    Ls2 = W.stencil_launch(ks, b, a, nx=n, ny=n, nzl=n, kg0=0, nzg=n, coeffs=(0.25,) + synthetic.STENCIL_COEFFS[1:])
    Ls2.jit()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for i in range(50):
        (Ls if i % 2 == 0 else Ls2).jit()
    e1.record()
    torch.cuda.synchronize()
    row["stencil_sweep_us"] = round(e0.elapsed_time(e1) / 50 * 1e3, 2)
    st = P.proteus_cache_stats()
    row["ir_compiles"] = st["ir_compiles"]
    row["ir_ms_total"] = round(st["ir_ms_total"], 1)
    out[mode] = row
    P.proteus_finalize()
print(json.dumps(out))
