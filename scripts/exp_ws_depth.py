#!/usr/bin/env python
"""Experiment: steady-state vs ramp/tail of stencil4_ws.  Same 256x256 planes and 512
blocks, z depth 256 vs 512 vs 1024 planes: if GB/s rises with depth, the per-launch ramp
(pipeline fill) and tail (last blocks) cost what the difference shows."""
import os, sys, tempfile
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np, torch
import synthetic
from paper_conf_cgo_georgakoudispb25_b200 import proteus as P, workloads as W

torch.zeros(1, device="cuda")
P.proteus_init(device=0, cache_dir=tempfile.mkdtemp(), mode="all")
k = W.register("stencil4_ws")
co = synthetic.STENCIL_COEFFS
for nz in (256, 512, 1024):
    for zc in (4, 8):
        slab = torch.ones((nz + 4, 256, 256), dtype=torch.float64, device="cuda")
        b = slab.clone()
        Ls = [W.stencil_launch(k, slab, b, nx=256, ny=256, nzl=nz, kg0=0, nzg=nz, coeffs=co, zchunks=zc),
              W.stencil_launch(k, b, slab, nx=256, ny=256, nzl=nz, kg0=0, nzg=nz, coeffs=co, zchunks=zc)]
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
        print(f"nz={nz:5d} zchunks={zc} blocks={512 * zc // 4}: {us:8.2f} us/sweep  "
              f"{256 * 256 * nz * 16 / us / 1e3:7.1f} GB/s", flush=True)
        del slab, b, Ls
        torch.cuda.empty_cache()
