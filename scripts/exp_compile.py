import os, sys, time, tempfile
sys.path.insert(0, os.getcwd())
import torch
import bench_suite as B
from paper_conf_cgo_georgakoudispb25_b200 import proteus as P, workloads as W
import synthetic
torch.zeros(1, device="cuda")
tmp = tempfile.mkdtemp()
# (1) the sweep's exact loop, timing compile via stats
for trial, n in enumerate([65536, 65536, 1000000]):
    P.proteus_init(device=0, cache_dir=os.path.join(tmp, f"t{trial}"), mode="all")
    k = W.register("adam_step")
    t = [torch.from_numpy(a).cuda() for a in synthetic.adam_inputs(n)]
    S = synthetic.ADAM_SCALARS
    L = W.adam_launch(k, *t, lr=1e-3, b1=S["b1"], b2=S["b2"], eps=S["eps"], grad_scale=S["grad_scale"], decay=S["decay"])
    per = []
    for i in range(10):
        L.set(5, 1e-3 * (1 + i / 4096))
        t0 = time.perf_counter(); L.jit(); per.append((time.perf_counter() - t0) * 1e3)
    st = P.proteus_cache_stats()
    print(f"trial {trial} n={n}: launch-miss ms", [round(x, 1) for x in per], "nvrtc mean", round(st["compile_ms_total"] / st["compiles"], 1), flush=True)
    P.proteus_finalize()
# (2) same but sleeping 0.3 s after init (warm thread done)
P.proteus_init(device=0, cache_dir=os.path.join(tmp, "t9"), mode="all")
time.sleep(0.5)
k = W.register("adam_step")
L = W.adam_launch(k, *t, lr=1e-3, b1=S["b1"], b2=S["b2"], eps=S["eps"], grad_scale=S["grad_scale"], decay=S["decay"])
per = []
for i in range(10):
    L.set(5, 2e-3 * (1 + i / 4096))
    t0 = time.perf_counter(); L.jit(); per.append((time.perf_counter() - t0) * 1e3)
st = P.proteus_cache_stats()
print("after sleep: launch-miss ms", [round(x, 1) for x in per], "nvrtc mean", round(st["compile_ms_total"] / st["compiles"], 1), flush=True)
P.proteus_finalize()
