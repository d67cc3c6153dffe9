#!/usr/bin/env python
"""Per-kernel CUDA-event times of the XS step (xs_bin, xs_scan, xs_scatter, xs_lookup), JIT."""
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
    ks = {e: W.register(e) for e in ("xs_index", "xs_bin", "xs_scan", "xs_scatter", "xs_lookup")}
    if os.environ.get("BIN_OPT"):     # a compile-time variant of xs_bin, e.g. -DXS_BIN_SMEM_MAX=0
        types, ann, base = W.SPECS["xs_bin"]
        ks["xs_bin"] = P.proteus_register_kernel("xs_bin", W.kernel_source("xs_bin"), types, ann,
                                                 None, (base + " " + os.environ["BIN_OPT"]).strip())
    d = W.xs_device_tables(tb, index_kernel=ks["xs_index"])
    macro = torch.empty((L, 5), dtype=torch.float64, device="cuda")
    idx = torch.empty(L, dtype=torch.int32, device="cuda")
    st = W.XSStep(ks, d, L, synthetic.S0, macro, idx)
    for _ in range(3):
        st("jit")
    torch.cuda.synchronize()
    names = ["xs_bin", "xs_scan", "xs_scatter", "xs_lookup"]
    for variant in ("jit", "aot"):
        for Lj in st.launches:     # every kernel in this variant compiled before timing
            Lj(variant)
        st(variant)
        tot = [0.0] * 4
        reps = 10
        for _ in range(reps):
            for j, Lj in enumerate(st.launches):
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                Lj(variant)
                e1.record()
                torch.cuda.synchronize()
                tot[j] += e0.elapsed_time(e1)
        print(("large " if large else "small ") + variant + " "
              + "  ".join(f"{n} {t / reps * 1e3:.1f} us" for n, t in zip(names, tot)), flush=True)
    del st, d, macro, idx
    torch.cuda.empty_cache()
