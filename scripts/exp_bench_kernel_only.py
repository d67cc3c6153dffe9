#!/usr/bin/env python
"""Why bench.py's kernel-only leg (50 sweeps after a sync) reads slower than the steady
loop and the suite: time the same ZSlabStencil with both protocols and several lengths."""
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

torch.zeros(1, device="cuda")
n = 256
slab = np.zeros((n + 4, n, n))
slab[2:n + 2] = synthetic.stencil_inputs(n, n, n)
P.proteus_init(device=0, cache_dir=tempfile.mkdtemp(), mode="all")
k = W.register("stencil4_ws")
st = halo.ZSlabStencil(k, torch.from_numpy(slab).cuda(), nx=n, ny=n, nzl=n, nzg=n, rank=0,
                       world=1, coeffs=synthetic.STENCIL_COEFFS)
stream = torch.cuda.current_stream()


def timed(variant, reps, warm=5, sync_first=True):
    st.variant = variant
    for _ in range(warm):
        st.sweep()
    if sync_first:
        torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(stream)
    for _ in range(reps):
        st.sweep()
    b.record(stream)
    torch.cuda.synchronize()
    return a.elapsed_time(b) / reps * 1e3


for reps in (50, 200, 1000, 3000):
    for v in ("jit", "aot"):
        print(f"{v} reps={reps}: {timed(v, reps):.2f} us/sweep", flush=True)
for v in ("jit", "aot"):
    print(f"{v} reps=50 no sync before: {timed(v, 50, sync_first=False):.2f} us/sweep")

# the bench's own sequence: NVML clock sampler around a 3000-sweep JIT loop, then the
# alternating kernel-only rounds
sys.argv = [sys.argv[0]]
import bench  # noqa: E402
with bench.ClockSampler(0):
    st.variant = "jit"
    for _ in range(3000):
        st.sweep()
    torch.cuda.synchronize()
for r in range(3):
    for v in ("aot", "jit"):
        print(f"after NVML sampler, round {r}: {v} {timed(v, 200):.2f} us/sweep", flush=True)
slab_pinned = torch.from_numpy(slab).pin_memory()
st2 = halo.ZSlabStencil(k, slab_pinned.to("cuda"), nx=n, ny=n, nzl=n, nzg=n, rank=0, world=1,
                        coeffs=synthetic.STENCIL_COEFFS)
st = st2
for v in ("aot", "jit"):
    print(f"new slab from pinned memory: {v} {timed(v, 200):.2f} us/sweep", flush=True)
