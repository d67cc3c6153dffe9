#!/usr/bin/env python
"""A/B of micro_column compile-time variants (JIT, CFG 4: 10^6 columns x 64 levels):
env AB="opt1;opt2;...".  Each variant runs from the same initial state; the outputs of
all variants must be bit-identical (the spec is evaluated exactly in every variant)."""
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
st0 = synthetic.micro_inputs(10 ** 6, 64)
types, ann, base = W.SPECS["micro_column"]
ref = None
for rep in range(2):
    for opt in os.environ.get("AB", "-DMICRO_GATE=0;-DMICRO_GATE=1").split(";"):
        k = P.proteus_register_kernel("micro_column", W.kernel_source("micro_column"), types, ann,
                                      None, (base + " " + opt).strip())
        k.set_min_blocks(int(os.environ.get("MINB", W.MIN_BLOCKS["micro_column"])))
        s = {kk: torch.from_numpy(v).cuda() for kk, v in st0.items()}
        pr = torch.zeros(10 ** 6, device="cuda")
        L = W.micro_launch(k, s, pr, nz=64, nsub=2, dt=20.0, dz=250.0,
                           block=int(os.environ.get("BLOCK", 128)))
        if "MICRO_LPL=2" in opt:          # a warp per column: twice the threads
            L = W.micro_launch(k, s, pr, nz=64, nsub=2, dt=20.0, dz=250.0, lanes=32)
        for _ in range(3):
            L("jit")
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(10):
            L("jit")
        e1.record()
        torch.cuda.synchronize()
        out = torch.cat([s[x].view(torch.int32).reshape(-1) for x in ("th", "qv", "qc", "qr")]
                        + [pr.view(torch.int32)])
        same = ""
        if ref is None:
            ref = out
        else:
            same = "bit-identical" if torch.equal(out, ref) else \
                f"DIFFERS in {(out != ref).sum().item()} words"
        print(f"{opt:22s} {e0.elapsed_time(e1) / 10:.4f} ms/call  {same}", flush=True)
