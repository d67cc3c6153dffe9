#!/usr/bin/env python
"""A/B of stencil4_ws compile-time variants (JIT, PDL, CFG 2 256^3): env AB="opt1;opt2".
Times 400 back-to-back sweeps per variant (2 reps) and checks that the field after 20
sweeps is bit-identical across variants."""
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

torch.zeros(1, device="cuda")
P.proteus_init(device=0, cache_dir=tempfile.mkdtemp(), mode="all")
n = 256
slab = np.zeros((n + 4, n, n))
slab[2:n + 2] = synthetic.stencil_inputs(n, n, n)
types, ann, base = W.SPECS["stencil4_ws"]
co = synthetic.STENCIL_COEFFS
ref = None
for rep in range(2):
    for opt in os.environ.get("AB", "-DWS_ZDIR=0;-DWS_ZDIR=1").split(";"):
        src = W.kernel_source("stencil4_ws")
        if opt.startswith("file:"):            # another source file of the same kernel
            src = open(opt[5:]).read()
        k = P.proteus_register_kernel("stencil4_ws", src, types, ann, None,
                                      base if opt.startswith("file:") else (base + " " + opt).strip())
        k.set_min_blocks(W.MIN_BLOCKS["stencil4_ws"])
        k.set_launch_attrs(P.LAUNCH_PDL)
        a = torch.from_numpy(slab).cuda()
        b = a.clone()
        Ls = [W.stencil_launch(k, a, b, nx=n, ny=n, nzl=n, kg0=0, nzg=n, coeffs=co),
              W.stencil_launch(k, b, a, nx=n, ny=n, nzl=n, kg0=0, nzg=n, coeffs=co)]
        for i in range(20):
            Ls[i % 2]("jit")
        torch.cuda.synchronize()
        out = a.clone()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for i in range(400):
            Ls[i % 2]("jit")
        e1.record()
        torch.cuda.synchronize()
        same = ""
        if rep == 0:
            if ref is None:
                ref = out
            else:
                same = "bit-identical" if torch.equal(out.view(torch.int64), ref.view(torch.int64)) else "DIFFERS"
        us = e0.elapsed_time(e1) / 400 * 1e3
        print(f"{opt:22s} {us:7.2f} us/sweep {n**3*16/us/1e3:8.1f} GB/s {same}", flush=True)
