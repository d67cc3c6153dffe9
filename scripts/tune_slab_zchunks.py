#!/usr/bin/env python
"""z-chunk count of stencil4_ws for the per-rank slabs of the N-GPU z-slab decomposition
(256^3 over P = 1, 2, 4, 8 ranks -> nzl = 256, 128, 64, 32 planes), measured on one B200
as a single interior rank's sweep (JIT, PDL, back-to-back launches; no halo exchange)."""
import os
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import synthetic  # noqa: E402
from paper_conf_cgo_georgakoudispb25_b200 import proteus as P  # noqa: E402
from paper_conf_cgo_georgakoudispb25_b200 import workloads as W  # noqa: E402

torch.zeros(1, device="cuda")
P.proteus_init(device=0, cache_dir=tempfile.mkdtemp(), mode="all")
k = W.register("stencil4_ws")
n = 256
co = synthetic.STENCIL_COEFFS
for nzl in (256, 128, 64, 32):
    a = torch.rand((nzl + 4, n, n), dtype=torch.float64, device="cuda") + 1.0
    b = a.clone()
    kg0 = 0 if nzl == n else n // 2 - nzl // 2      # an interior rank
    best = None
    for zc in (1, 2, 3, 4, 6, 8, 12, 16):
        if nzl // zc < 4:
            continue
        Ls = [W.stencil_launch(k, a, b, nx=n, ny=n, nzl=nzl, kg0=kg0, nzg=n, coeffs=co, zchunks=zc),
              W.stencil_launch(k, b, a, nx=n, ny=n, nzl=nzl, kg0=kg0, nzg=n, coeffs=co, zchunks=zc)]
        for i in range(6):
            Ls[i % 2]("jit")
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        reps = 400
        e0.record()
        for i in range(reps):
            Ls[i % 2]("jit")
        e1.record()
        torch.cuda.synchronize()
        us = e0.elapsed_time(e1) / reps * 1e3
        gbs = nzl * n * n * 16 / (us * 1e-6) / 1e9
        blocks = 4 * 32 * zc
        print(f"nzl={nzl:4d} zchunks={zc:3d} blocks={blocks:5d}: {us:8.2f} us/sweep {gbs:8.1f} GB/s",
              flush=True)
        best = min(best or (1e9, 0), (us, zc))
    print(f"nzl={nzl}: best zchunks={best[1]} ({best[0]:.2f} us)", flush=True)
