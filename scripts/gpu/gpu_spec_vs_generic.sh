#!/bin/bash
# ncu --set full of the specialized (JIT, mode all) and the generic (nvcc AOT) variant of
# every workload kernel at its BASELINE.json config (north_star: "every design choice is
# evidenced by ncu counters comparing the specialized and generic variants").
export PROTEUS_LINEINFO=1
mkdir -p gpurun_out
for w in stencil adam_run xs micro; do
  case $w in stencil) K=stencil4_ws;; adam_run) K=adam_run;; xs) K=xs_lookup;; micro) K=micro_column;; esac
  for v in jit aot; do
    STENCIL_ENTRY=stencil4_ws timeout 600 ncu --set full --clock-control none --import-source on -k regex:$K -s 2 -c 1 -f -o gpurun_out/sg_${w}_${v}_${TAG:-r01h} python scripts/profile_workloads.py --workload $w --variant $v --reps 3 > /dev/null 2>&1; echo ncu $w $v rc=$?
  done
done
