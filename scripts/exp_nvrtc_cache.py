import os, sys, time, tempfile, random
sys.path.insert(0, os.getcwd())
from paper_conf_cgo_georgakoudispb25_b200 import proteus as P, workloads as W
P.testing_use_fake_backend(2)
P.proteus_init(device=0, cache_dir=tempfile.mkdtemp(), mode="all")
k = W.register("adam_step", with_generic=False)
seed = float(sys.argv[1])
ts = []
for i in range(5):
    args = [0, 0, 0, 0, 1000000, seed * (1 + i / 4096), 0.9, 0.999, 1e-8, 1024.0, 0.01, 1, 0.1, 0.001]
    t0 = time.perf_counter(); P.proteus_get_specialization(k, (977,), (256,), args); ts.append(1e3 * (time.perf_counter() - t0))
print("seed", seed, [round(t, 1) for t in ts], flush=True)
