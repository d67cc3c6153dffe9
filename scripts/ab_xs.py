#!/usr/bin/env python
"""A/B of xs_lookup compile-time variants (JIT) on the CFG 3 step: env AB="opt1;opt2;..."
(default: the energy-bin count of the index and the sort key)."""
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
large = os.environ.get("LARGE") == "1"
tb = synthetic.xs_tables_large() if large else synthetic.xs_tables()
L = 10 ** 7
macro = torch.empty((L, 5), dtype=torch.float64, device="cuda")
idx = torch.empty(L, dtype=torch.int32, device="cuda")
ks = {e: W.register(e) for e in ("xs_index", "xs_bin", "xs_scan", "xs_scatter", "xs_lookup")}
d = W.xs_device_tables(tb, index_kernel=ks["xs_index"])
types, ann, _ = W.SPECS["xs_lookup"]
ref = {}   # per-lookup results of the first option: every other option must be bit-identical
for rep in range(2):
    for opt in os.environ.get("AB", "-DXS_EBINS=2048;-DXS_EBINS=4096").split(";"):
        # "opt@minBlocks" overrides the launch-bounds budget for one option
        opt, _, mb = opt.partition("@")
        k = P.proteus_register_kernel("xs_lookup", W.kernel_source("xs_lookup"), types, ann, None,
                                      opt)
        k.set_min_blocks(int(mb or os.environ.get("MINB", W.MIN_BLOCKS["xs_lookup"])))
        kk = dict(ks, xs_lookup=k)
        st = W.XSStep(kk, d, L, synthetic.S0, macro, idx)
        for _ in range(3):
            st("jit")
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(10):
            st("jit")
        e1.record()
        torch.cuda.synchronize()
        # results in lookup order (slot t holds lookup slot_lookups()[t])
        sl = st.slot_lookups().long()
        got_m = torch.empty_like(macro)
        got_m[sl] = macro
        got_i = torch.empty_like(idx)
        got_i[sl] = idx
        if not ref:
            ref.update(m=got_m.clone(), i=got_i.clone())
        same = torch.equal(got_m, ref["m"]) and torch.equal(got_i, ref["i"])
        # the lookup kernel alone
        for _ in range(2):
            st.launches[3]("jit")
        f0, f1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        f0.record()
        for _ in range(10):
            st.launches[3]("jit")
        f1.record()
        torch.cuda.synchronize()
        print(f"{'large' if large else 'small'} {opt + ('@' + mb if mb else ''):24s} step {e0.elapsed_time(e1) / 10:.3f} ms  "
              f"lookup {f0.elapsed_time(f1) / 10:.3f} ms  "
              f"{'bit-identical' if same else 'DIFFERS'} vs {os.environ.get('AB', '').split(';')[0]!r}",
              flush=True)
