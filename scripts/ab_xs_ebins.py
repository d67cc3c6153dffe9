#!/usr/bin/env python
"""A/B of the XS energy-bin count (search index + sort key), JIT, CFG 3 step and large
table: EBINS in env AB (default 1024,2048,4096).  Outputs must be bit-identical across
bin counts (the index only narrows the search; the arithmetic is the same)."""
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
BASE = dict(W.SPECS)
# every kernel of the step specialized here (the product runs xs_scan and xs_index as their
# generic builds, which exist only for the default bin count)
W.XSStep.JIT_ENTRIES = ("xs_bin", "xs_scan", "xs_scatter", "xs_lookup")
L = 10 ** 7
for large in (False, True):
    tb = synthetic.xs_tables_large() if large else synthetic.xs_tables()
    ref = None
    for rep in range(2):
        for E in [int(x) for x in os.environ.get("AB", "1024,2048,4096").split(",")]:
            W.XS_EBINS = E
            ks = {}
            for e in ("xs_index", "xs_bin", "xs_scan", "xs_scatter", "xs_lookup"):
                types, ann, opt = BASE[e]
                k = P.proteus_register_kernel(e, W.kernel_source(e), types, ann, None,
                                              (opt + f" -DXS_EBINS={E}").strip())
                if W.MIN_BLOCKS.get(e):
                    k.set_min_blocks(W.MIN_BLOCKS[e])
                ks[e] = k
            d = W.xs_device_tables(tb, index_kernel=ks["xs_index"], variant="jit")
            macro = torch.empty((L, 5), dtype=torch.float64, device="cuda")
            idx = torch.empty(L, dtype=torch.int32, device="cuda")
            st = W.XSStep(ks, d, L, synthetic.S0, macro, idx)
            for _ in range(3):
                st("jit")
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            for _ in range(10):
                st("jit")
            e1.record()
            torch.cuda.synchronize()
            f0, f1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            f0.record()
            for _ in range(10):
                st.launches[3]("jit")
            f1.record()
            torch.cuda.synchronize()
            # results in lookup order (slot t holds lookup slot_lookups()[t]; the order
            # within a bucket is not deterministic)
            sl = st.slot_lookups().long()
            om = torch.empty_like(macro)
            om[sl] = macro
            oi = torch.empty_like(idx)
            oi[sl] = idx
            out = (om.cpu(), oi.cpu())
            same = ""
            if ref is None:
                ref = out
            else:
                same = "bit-identical" if (torch.equal(out[0].view(torch.int64), ref[0].view(torch.int64))
                                           and torch.equal(out[1], ref[1])) else "DIFFERS"
            print(f"{'large' if large else 'small'} EBINS={E:5d} step {e0.elapsed_time(e1) / 10:.3f} ms "
                  f"lookup {f0.elapsed_time(f1) / 10:.3f} ms {same}", flush=True)
            del st, d, macro, idx
            torch.cuda.empty_cache()
