#!/usr/bin/env python
"""A/B of adam_run compile-time variants (JIT, CFG 1: 10^6 params, 100 steps in one launch):
env AB="opt1;opt2;...".  Checks each variant against the fp64 oracle (1e-5) too."""
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
P.proteus_init(device=0, cache_dir=tempfile.mkdtemp(), mode=os.environ.get("MODE", "all"))
S = synthetic.ADAM_SCALARS
n, steps = 10 ** 6, 100
x0 = synthetic.adam_inputs(n)
types, ann, _ = W.SPECS["adam_run"]
for rep in range(2):
    for opt in os.environ.get("AB", "-DADAM_RCP_NEWTON=0;-DADAM_RCP_NEWTON=1").split(";"):
        # "file:<path>" as an option: that source instead of the product's adam_step.cu
        src = W.kernel_source("adam_run")
        if opt.startswith("file:"):
            src = open(os.path.join(ROOT, opt[5:])).read()
        k = P.proteus_register_kernel("adam_run", src, types, ann, None,
                                      "" if opt.startswith("file:") else opt)
        if os.environ.get("MINB"):
            k.set_min_blocks(int(os.environ["MINB"]))
        t = [torch.from_numpy(a).cuda() for a in x0]
        L = W.adam_run_launch(k, *t, lr=S["lr"], b1=S["b1"], b2=S["b2"], eps=S["eps"],
                              grad_scale=S["grad_scale"], decay=S["decay"], steps=steps,
                              block=int(os.environ.get("BLOCK", 256)))
        L("jit")
        torch.cuda.synchronize()
        p1 = t[0].cpu().numpy()
        for _ in range(3):
            L("jit")
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(20):
            L("jit")
        e1.record()
        torch.cuda.synchronize()
        msg = ""
        if rep == 0:
            import oracle  # test infrastructure: the oracle checks each variant
            f = lambda v: float(np.float32(v))
            want = oracle.adam(*x0, lr=f(S["lr"]), b1=f(S["b1"]), b2=f(S["b2"]),
                                      eps=f(S["eps"]), grad_scale=f(S["grad_scale"]),
                                      decay=f(S["decay"]), mode=1, steps=steps)[0]
            msg = f"  max rel err p {np.max(np.abs(p1 - want) / np.abs(want)):.2e}"
        print(f"{opt:24s} {e0.elapsed_time(e1) / 20:.4f} ms / {steps} steps{msg}", flush=True)
