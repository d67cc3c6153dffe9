#!/bin/bash
# r02ao: does anything cache NVRTC compiles on the box? (repeat probe; proteus re-compile after clear)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 python scripts/nvrtc_repeat_probe.py 2>&1 | tee gpurun_out/nvrtc_repeat_r02ao.txt
timeout 600 python - <<'PY' 2>&1 | tee -a gpurun_out/nvrtc_repeat_r02ao.txt
import tempfile, torch, sys, os
sys.path.insert(0, os.getcwd()); sys.path.insert(0, os.getcwd() + "/scripts")
from paper_conf_cgo_georgakoudispb25_b200 import proteus as P
import profile_workloads as PW
torch.zeros(1, device="cuda")
os.environ["STENCIL_ENTRY"] = "stencil4_ws"
for rep in range(4):
    P.proteus_init(device=0, cache_dir=tempfile.mkdtemp(), mode="all")
    Ls, keep = PW.build("stencil")
    s0 = P.proteus_cache_stats()
    Ls[0]("jit"); torch.cuda.synchronize()
    s1 = P.proteus_cache_stats()
    print("proteus rep", rep, "compiles", s1["compiles"] - s0["compiles"], "disk_hits", s1["disk_hits"] - s0["disk_hits"],
          "compile ms", round(s1["compile_ms_total"] - s0["compile_ms_total"], 1), flush=True)
    del Ls, keep
    P.proteus_finalize()
PY
ls -la ~/.nv 2>/dev/null; ls ~/.cache 2>/dev/null | head; env | grep -i "cuda_cache\|nvrtc\|ptxas" 
