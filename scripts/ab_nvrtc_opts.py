#!/usr/bin/env python
"""A/B of extra NVRTC options on every workload kernel (B200): per option set, the JIT
compile ms of each specialization (cold in-memory and disk cache) and the kernel time
(median of CUDA-event times, back-to-back launches after warm-up).
  env AB="opt1;opt2;..."   (default: "", --Ofast-compile=min, --Ofast-compile=mid)"""
import os
os.environ.setdefault("CUDA_CACHE_DISABLE", "1")   # else the driver ComputeCache serves repeat NVRTC compiles
import statistics
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "scripts"))
import torch  # noqa: E402

from paper_conf_cgo_georgakoudispb25_b200 import proteus as P  # noqa: E402
from paper_conf_cgo_georgakoudispb25_b200 import workloads as W  # noqa: E402
import profile_workloads as PW  # noqa: E402

BASE = dict(W.SPECS)
torch.zeros(1, device="cuda")
os.environ.setdefault("STENCIL_ENTRY", "stencil4_ws")
opts = os.environ.get("AB", ";--Ofast-compile=min;--Ofast-compile=mid").split(";")
for rep in range(2):
    for opt in opts:
        for e, (types, ann, base) in BASE.items():
            W.SPECS[e] = (types, ann, (base + " " + opt).strip())
        for wl in ("stencil", "adam_run", "xs", "micro"):
            P.proteus_init(device=0, cache_dir=tempfile.mkdtemp(), mode="all")
            Ls, keep = PW.build(wl)
            s0 = P.proteus_cache_stats()
            for L in Ls:
                L("jit")
            torch.cuda.synchronize()
            s1 = P.proteus_cache_stats()
            comp = s1["compile_ms_total"] - s0["compile_ms_total"]
            ts = []
            for r in range(12):
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                Ls[r % len(Ls)]("jit")
                e1.record()
                torch.cuda.synchronize()
                ts.append(e0.elapsed_time(e1))
            print(f"rep {rep} {opt or '(default)':22s} {wl:9s} compile {comp:7.1f} ms "
                  f"({s1['compiles'] - s0['compiles']} keys)  kernel {statistics.median(ts[2:]):.4f} ms",
                  flush=True)
            del Ls, keep
            P.proteus_finalize()
