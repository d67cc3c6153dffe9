#!/usr/bin/env python
"""Sweep stencil4_ws (warp-specialized TMA ring) at 256^3 on one GPU (JIT variant):
consumer warps TY, rows per thread WS_RY, ring slots WS_S, z-chunks.  Prints us/sweep,
GB/s (16 B/point algorithmic).  Env: N (grid edge), CONFIGS="ty,ry,s;..", ZCS="2,4,..",
EXTRA (NVRTC options appended), MINB (launch-bounds minBlocks hint, default 4),
PROTEUS_PDL=0 (no programmatic dependent launch)."""
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
types, ann, _ = W.SPECS["stencil4_ws"]
CONFIGS = [tuple(int(v) for v in c.split(",")) for c in os.environ.get(
    "CONFIGS", "4,2,6;4,2,8;5,2,6").split(";")]
ZCS = [int(z) for z in os.environ.get("ZCS", "3,4,8").split(",")]
EXTRA = os.environ.get("EXTRA", "")
results = []
for ty, ry, S in CONFIGS:
    k = P.proteus_register_kernel("stencil4_ws", W.kernel_source("stencil4_ws"), types, ann, None,
                                  f"-DWS_S={S} -DWS_RY={ry} {EXTRA}")
    if int(os.environ.get("MINB", "4")):
        k.set_min_blocks(int(os.environ.get("MINB", "4")))
    if os.environ.get("PROTEUS_PDL", "1") != "0":
        k.set_launch_attrs(P.LAUNCH_PDL)
    for zc in ZCS:
        smem = S * (-(-68 * (ty * ry + 4) // 16) * 16) * 8
        if smem > 220 * 1024:
            continue
        try:
            Ls = [W.stencil_launch(k, a, b, nx=n, ny=n, nzl=n, kg0=0, nzg=n, coeffs=co,
                                   tile=(32, ty), zchunks=zc, ry=ry, ring=S),
                  W.stencil_launch(k, b, a, nx=n, ny=n, nzl=n, kg0=0, nzg=n, coeffs=co,
                                   tile=(32, ty), zchunks=zc, ry=ry, ring=S)]
            for i in range(6):
                Ls[i % 2].jit()
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            reps = 60
            e0.record()
            for i in range(reps):
                Ls[i % 2].jit()
            e1.record()
            torch.cuda.synchronize()
            us = e0.elapsed_time(e1) / reps * 1e3
            gbs = n ** 3 * 16 / (us * 1e-6) / 1e9
            blocks = Ls[0].dims[0] * Ls[0].dims[1] * Ls[0].dims[2]
            results.append((us, ty, ry, S, zc, gbs))
            print(f"TY={ty} RY={ry} S={S} zchunks={zc} blocks={blocks}: {us:8.2f} us  "
                  f"{gbs:7.1f} GB/s", flush=True)
        except Exception as e:
            print(f"TY={ty} RY={ry} S={S} zchunks={zc}: FAILED {e}", flush=True)
results.sort()
print("BEST", results[:8])
