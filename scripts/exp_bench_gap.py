#!/usr/bin/env python
"""Why does bench.py's 3000-sweep loop run slower per sweep than the 60-rep tuning loop?
Times the same stencil4_ws launches: (a) 60 reps, (b) 3000 reps, (c) 3000 reps through
halo.ZSlabStencil, (d) = (c) with bench.ClockSampler running, (e) per-launch events."""
import os
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import bench  # noqa: E402
import synthetic  # noqa: E402
from paper_conf_cgo_georgakoudispb25_b200 import halo  # noqa: E402
from paper_conf_cgo_georgakoudispb25_b200 import proteus as P  # noqa: E402
from paper_conf_cgo_georgakoudispb25_b200 import workloads as W  # noqa: E402

n = 256
torch.zeros(1, device="cuda")
P.proteus_init(device=0, cache_dir=tempfile.mkdtemp(), mode="all")
k = W.register("stencil4_ws")
slab = np.zeros((n + 4, n, n))
slab[2:n + 2] = synthetic.stencil_inputs(n, n, n)
a = torch.from_numpy(slab).cuda()
co = synthetic.STENCIL_COEFFS
st = halo.ZSlabStencil(k, a, nx=n, ny=n, nzl=n, nzg=n, rank=0, world=1, coeffs=co)


def timed(fn, reps):
    for _ in range(5):
        fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        fn()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps * 1e3


L = st.launch
Ls = [L["uw"][0], L["wu"][0]]
cnt = [0]


def raw():
    Ls[cnt[0] % 2].jit()
    cnt[0] += 1


for reps in (60, 3000, 60, 3000):
    print(f"raw launches x{reps}: {timed(raw, reps):.2f} us/sweep", flush=True)
print(f"ZSlabStencil x3000: {timed(st.sweep, 3000):.2f} us/sweep", flush=True)
with bench.ClockSampler(0) as c:
    print(f"ZSlabStencil x3000 + ClockSampler: {timed(st.sweep, 3000):.2f} us/sweep", flush=True)
print(c.summary())
# per-launch events on a sample
ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
      for _ in range(400)]
for e in ev:
    e[0].record()
    raw()
    e[1].record()
torch.cuda.synchronize()
d = np.array([x.elapsed_time(y) * 1e3 for x, y in ev])
print(f"per-launch events: median {np.median(d):.2f} p10 {np.percentile(d, 10):.2f} "
      f"p90 {np.percentile(d, 90):.2f} max {d.max():.2f} us")
# gaps: start-to-start
s = np.array([ev[i][0].elapsed_time(ev[i + 1][0]) * 1e3 for i in range(len(ev) - 1)])
print(f"start-to-start: median {np.median(s):.2f} us")
P.proteus_finalize()
