#!/usr/bin/env python
"""Sweep stencil4 (TMA) launch/compile parameters at 256^3 on one GPU (JIT variant):
ring slots ST_S, rows per thread ST_RY, thread tile, z-chunks.  Prints us/sweep, GB/s."""
import itertools
import os
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import synthetic  # noqa: E402
from paper_conf_cgo_georgakoudispb25_b200 import proteus as P  # noqa: E402
from paper_conf_cgo_georgakoudispb25_b200 import workloads as W  # noqa: E402

n = int(os.environ.get("N", "256"))
torch.zeros(1, device="cuda")
P.proteus_init(device=0, cache_dir=tempfile.mkdtemp(), mode=os.environ.get("MODE", "all"))
slab = np.zeros((n + 4, n, n))
slab[2:n + 2] = synthetic.stencil_inputs(n, n, n)
a = torch.from_numpy(slab).cuda()
b = a.clone()
co = synthetic.STENCIL_COEFFS
types, ann, _ = W.SPECS["stencil4"]
results = []
VARIANTS = os.environ.get("VARIANTS", "")   # e.g. "-DST_WSTORE=1;-DST_L2HINT=2"
CONFIGS = [(6, 2), (8, 2), (4, 4), (6, 4)] if VARIANTS else \
    [(4, 2), (6, 2), (8, 2), (4, 4), (6, 4), (8, 4), (5, 1), (6, 1)]
TILES = [(32, 4), (32, 2), (64, 2)] if VARIANTS else [(32, 4), (32, 2), (32, 8), (16, 8), (64, 2)]
ZCS = [2, 3, 4, 6] if VARIANTS else [2, 4, 6, 8, 12]
for extra, (S, RY) in itertools.product(VARIANTS.split(";"), CONFIGS):
    k = P.proteus_register_kernel("stencil4", W.kernel_source("stencil4"), types, ann, None,
                                  f"-DST_S={S} -DST_RY={RY} {extra}")
    for tile, zc in itertools.product(TILES, ZCS):
        if tile[0] * tile[1] > 1024:
            continue
        smem = S * (2 * tile[0] + 4) * (tile[1] * RY + 4) * 8
        if smem > 220 * 1024:
            continue
        try:
            Ls = [W.stencil_launch(k, a, b, nx=n, ny=n, nzl=n, kg0=0, nzg=n, coeffs=co, tile=tile,
                                   zchunks=zc, ry=RY, ring=S),
                  W.stencil_launch(k, b, a, nx=n, ny=n, nzl=n, kg0=0, nzg=n, coeffs=co, tile=tile,
                                   zchunks=zc, ry=RY, ring=S)]
            for i in range(6):
                Ls[i % 2].jit()
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            reps = 40
            e0.record()
            for i in range(reps):
                Ls[i % 2].jit()
            e1.record()
            torch.cuda.synchronize()
            us = e0.elapsed_time(e1) / reps * 1e3
            gbs = n ** 3 * 16 / (us * 1e-6) / 1e9
            results.append((us, S, RY, tile, zc, gbs, extra))
            print(f"{extra} S={S} RY={RY} tile={tile} zchunks={zc}: {us:8.2f} us  {gbs:7.1f} GB/s",
                  flush=True)
        except Exception as e:
            print(f"S={S} RY={RY} tile={tile} zchunks={zc}: FAILED {e}", flush=True)
results.sort()
print("BEST", results[:8])
