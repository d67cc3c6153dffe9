#!/usr/bin/env python
"""xs_lookup block size x launch-bounds minBlocks at the shipped XS_EBINS (JIT, CFG 3 step
and large table); the lookup kernel alone is timed."""
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
L = 10 ** 7
for large in (False, True):
    tb = synthetic.xs_tables_large() if large else synthetic.xs_tables()
    ks = {e: W.register(e) for e in ("xs_index", "xs_bin", "xs_scan", "xs_scatter")}
    d = W.xs_device_tables(tb, index_kernel=ks["xs_index"])
    macro = torch.empty((L, 5), dtype=torch.float64, device="cuda")
    idx = torch.empty(L, dtype=torch.int32, device="cuda")
    for block in [int(x) for x in os.environ.get("BLOCKS", "128,256,512").split(",")]:
        if block <= 256:   # the generic AOT build (no launch bounds) at this block size
            st = W.XSStep(dict(ks, xs_lookup=W.register("xs_lookup")), d, L, synthetic.S0,
                          macro, idx, block=block)
            st("aot")
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            for _ in range(8):
                st.launches[3]("aot")
            e1.record()
            torch.cuda.synchronize()
            print(f"{'large' if large else 'small'} block={block} AOT generic: lookup "
                  f"{e0.elapsed_time(e1) / 8:.3f} ms", flush=True)
        for mb in [int(x) for x in os.environ.get("MINBS", "2,3,4,5,6,8").split(",")]:
            if block * mb > 2048:
                continue
            k = W.register("xs_lookup", min_blocks=mb)
            st = W.XSStep(dict(ks, xs_lookup=k), d, L, synthetic.S0, macro, idx, block=block)
            for _ in range(2):
                st("jit")
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            for _ in range(8):
                st.launches[3]("jit")
            e1.record()
            torch.cuda.synchronize()
            print(f"{'large' if large else 'small'} block={block} minB={mb}: lookup "
                  f"{e0.elapsed_time(e1) / 8:.3f} ms", flush=True)
    del d, macro, idx
    torch.cuda.empty_cache()
