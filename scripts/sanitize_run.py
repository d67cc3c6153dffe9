#!/usr/bin/env python
"""Every workload kernel, generic (AOT) and specialized (JIT), once at a small size with
ragged tails -- the process compute-sanitizer (memcheck / racecheck / synccheck /
initcheck) runs over (tests/test_gpu_sanitizer.py).  Prints "sanitize-run ok"."""
import os
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import synthetic  # noqa: E402
from paper_conf_cgo_georgakoudispb25_b200 import halo  # noqa: E402
from paper_conf_cgo_georgakoudispb25_b200 import proteus as P  # noqa: E402
from paper_conf_cgo_georgakoudispb25_b200 import workloads as W  # noqa: E402

only = set(sys.argv[1:])
# BOUNDS=1: every specialization compiled with the device bounds checks (-DPROTEUS_CHECK,
# proteus_device.h) and only the JIT variant run -- an out-of-bounds index traps and the
# process fails (tests/test_gpu_bounds.py; the pool refuses compute-sanitizer)
BOUNDS = os.environ.get("BOUNDS") == "1"
if BOUNDS:
    _register = W.register
    W.register = lambda entry, **kw: _register(entry, options="-DPROTEUS_CHECK", **kw)
torch.zeros(1, device="cuda")
P.proteus_init(device=0, cache_dir=tempfile.mkdtemp(prefix="proteus-san-"), mode="all")


def want(name):
    return not only or name in only


for variant in (("jit",) if BOUNDS else ("aot", "jit")):
    if want("daxpy"):
        k = W.register("daxpy")
        x = torch.ones(1003, dtype=torch.float64, device="cuda")
        y = torch.zeros_like(x)
        W.daxpy_launch(k, 2.0, x, y)(variant)
    if want("adam"):
        k = W.register("adam_step")
        S = synthetic.ADAM_SCALARS
        t = [torch.from_numpy(a).cuda() for a in synthetic.adam_inputs(4099)]
        L = W.adam_launch(k, *t, lr=S["lr"], b1=S["b1"], b2=S["b2"], eps=S["eps"],
                          grad_scale=S["grad_scale"], decay=S["decay"])
        for s in (1, 2):
            W.adam_set_step(L, s)
            L(variant)
    if want("stencil"):
        for entry in ("stencil4_ws", "stencil4", "stencil4_smem"):
            k = W.register(entry)
            nx = 70 if entry != "stencil4_smem" else 45
            ny, nz = 37, 19
            slab = np.zeros((nz + 4, ny, nx))
            slab[2:nz + 2] = synthetic.stencil_inputs(nx, ny, nz)
            a = torch.from_numpy(slab).cuda()
            b = a.clone()
            for src, dst in ((a, b), (b, a)):
                W.stencil_launch(k, src, dst, nx=nx, ny=ny, nzl=nz, kg0=0, nzg=nz,
                                 coeffs=synthetic.STENCIL_COEFFS)(variant)
            torch.cuda.synchronize()
    if want("p2p"):
        k = W.register("stencil4_p2p")
        halo.run_slabs_p2p_local(k, synthetic.stencil_inputs(40, 36, 16), 3, 2,
                                 synthetic.STENCIL_COEFFS, variant=variant)
    if want("xs"):
        names = ("xs_index", "xs_bin", "xs_scan", "xs_scatter", "xs_lookup")
        ks = {e: W.register(e) for e in names}
        t = synthetic.xs_tables(n_nuc=68, n_grid=300)
        d = W.xs_device_tables(t, index_kernel=ks["xs_index"], variant=variant)
        L = 3001
        macro = torch.empty((L, 5), dtype=torch.float64, device="cuda")
        idx = torch.empty(L, dtype=torch.int32, device="cuda")
        W.XSStep(ks, d, L, synthetic.S0, macro, idx)(variant)
        W.xs_launch(ks["xs_lookup"], d, L, synthetic.S0, macro, idx)(variant)
    if want("micro"):
        k = W.register("micro_column")
        st = synthetic.micro_inputs(37, 64)
        s = {kk: torch.from_numpy(v).cuda() for kk, v in st.items()}
        pr = torch.zeros(37, device="cuda")
        W.micro_launch(k, s, pr, nz=64, nsub=2, dt=20.0, dz=250.0)(variant)
    torch.cuda.synchronize()
P.proteus_finalize()
print("sanitize-run ok")
