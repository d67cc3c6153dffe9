#!/bin/bash
# r02c: XS event-order outputs -- parity, step breakdown, ncu of xs_lookup (both variants)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 1500 python -m pytest tests/test_gpu_parity_full.py tests/test_gpu_bench_multirank.py -q -x 2>&1 | tail -15 | tee gpurun_out/r02c_full.txt
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_edge.py -q -x -k "xs" 2>&1 | tail -5 | tee gpurun_out/r02c_xs.txt
timeout 300 python scripts/xs_step_breakdown.py 2>&1 | tail -3 | tee gpurun_out/r02c_xs_breakdown.txt
for v in jit aot; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:xs_lookup -s 1 -c 1 -f -o gpurun_out/xs_${v}_r02c python scripts/profile_workloads.py --workload xs --variant $v --reps 3 > gpurun_out/prof_xs_${v}_r02c.log 2>&1; echo ncu xs $v rc=$?
done
