"""Worker of tests/test_runtime_fake.py::test_processes_share_one_cache_dir: one process on
the fake backend launching K daxpy keys (in a rotated order) into a shared cache dir,
each compile slowed to widen the race window; prints its counters as JSON."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
from paper_conf_cgo_georgakoudispb25_b200 import proteus as P  # noqa: E402
from test_runtime_fake import reg_daxpy  # noqa: E402

cache_dir, K, rank = sys.argv[1], int(sys.argv[2]), int(sys.argv[3])
P.testing_use_fake_backend(True)
P.testing_fake_control(False, 2)
P.proteus_init(device=0, cache_dir=cache_dir)
k = reg_daxpy()
for j in range(K):
    i = (j + rank * 7) % K
    P.proteus_launch(k, (8,), (256,), [float(i), 2048, 0, 0])
s = P.proteus_cache_stats()
P.proteus_finalize()
print(json.dumps({kk: s[kk] for kk in ("compiles", "disk_hits", "disk_rejects", "misses")}))
