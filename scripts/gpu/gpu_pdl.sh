#!/bin/bash
# programmatic dependent launch: GPU tests, A/B of stencil and adam with PDL on/off, bench
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
for PDL in 0 1; do
  echo "PROTEUS_PDL=$PDL"
  PROTEUS_PDL=$PDL timeout 600 python scripts/tune_stencil_ws.py 2>&1 | grep -v BEST
  for w in adam stencil; do for v in jit aot; do PROTEUS_PDL=$PDL timeout 300 python scripts/profile_workloads.py --workload $w --variant $v --reps 8 2>&1 | tail -1; done; done
done
timeout 900 python bench.py > gpurun_out/bench_pdl.json 2> gpurun_out/bench_pdl.err; echo bench rc=$?
tail -3 gpurun_out/bench_pdl.err; cat gpurun_out/bench_pdl.json
