#!/bin/bash
# r02bt: final validation after the final adam_run (L a factor, minBlocks 4): every GPU test, smoke, the default
# bench line and a --steps 20 line, ncu --set full of xs_lookup (JIT, AOT), XS e2e 2 s job
export PROTEUS_LINEINFO=1
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r02bt_build.log 2>&1; echo build rc=$?
timeout 2400 python -m pytest tests -m gpu -q 2>&1 | tail -4 | tee gpurun_out/r02bt_gpu_tests.txt
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1 | cut -c1-200 | tee gpurun_out/r02bt_smoke.txt
s=$(date +%s); timeout 1500 python bench.py > gpurun_out/bench_r02bt.json 2> gpurun_out/bench_r02bt.err; echo bench rc=$? wall=$(( $(date +%s) - s ))s
s=$(date +%s); timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/bench_r02bt_k20.json 2> gpurun_out/bench_r02bt_k20.err; echo bench k20 rc=$? wall=$(( $(date +%s) - s ))s
for v in jit aot; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:xs_lookup -s 2 -c 1 -f -o gpurun_out/xs_lookup_${v}_r02bt python scripts/profile_workloads.py --workload xs --variant $v --reps 3 > gpurun_out/prof_xs_${v}_r02bt.log 2>&1; echo ncu xs $v rc=$?
done
