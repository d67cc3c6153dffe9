#!/bin/bash
# r02bl: XS_STREAM adopted: XS GPU tests, per-kernel step times, ncu --set full of
# xs_lookup JIT and AOT (L2 hit rate, DRAM bytes)
export PROTEUS_LINEINFO=1
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 1800 python -m pytest tests -m gpu -q -k "xs or XS" 2>&1 | tail -3 | tee gpurun_out/r02bl_xs_tests.txt
timeout 600 python scripts/xs_step_breakdown.py 2>&1 | tee gpurun_out/xs_step_breakdown_r02bl.txt
for v in jit aot; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:xs_lookup -s 2 -c 1 -f -o gpurun_out/xs_lookup_${v}_r02bl python scripts/profile_workloads.py --workload xs --variant $v --reps 3 > gpurun_out/prof_xs_${v}_r02bl.log 2>&1; echo ncu xs $v rc=$?
done
