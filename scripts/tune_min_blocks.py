#!/usr/bin/env python
"""Launch-bounds minBlocks sweep per workload kernel (mode all vs rcf), one GPU."""
import os
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import bench_suite as B  # noqa: E402
from paper_conf_cgo_georgakoudispb25_b200 import proteus as P  # noqa: E402
from paper_conf_cgo_georgakoudispb25_b200 import workloads as W  # noqa: E402

torch.zeros(1, device="cuda")
tmp = tempfile.mkdtemp()
for name in sys.argv[1:] or ["micro", "xs", "stencil", "adam"]:
    wl = B.WORKLOADS[name]()
    for mode, mbs in (("rcf", [0]), ("all", [1, 2, 3, 4, 5, 6, 8])):
        for mb in mbs:
            P.proteus_init(device=0, cache_dir=os.path.join(tmp, f"{name}-{mode}-{mb}"), mode=mode)
            ks = {e: W.register(e, min_blocks=mb) for e in W.SPECS}
            step = wl.make(ks)
            ms = B.time_steps(step, "jit", 20)
            fn, _ = B.spec_fn(step)
            print(f"{name} mode={mode} minB={mb}: {ms*1e3:9.2f} us  regs={B.func_regs(fn)}", flush=True)
            P.proteus_finalize()
    del wl
    torch.cuda.empty_cache()
