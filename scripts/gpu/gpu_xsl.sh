#!/bin/bash
export PROTEUS_LINEINFO=1   # ncu --import-source maps JIT kernels to their source
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "xs_large" 2>&1 | tail -3
timeout 1200 python bench_suite.py --configs xs_large,stencil > gpurun_out/suite_xsl.jsonl 2> gpurun_out/suite_xsl.err; echo suite rc=$?
tail -3 gpurun_out/suite_xsl.err; cat gpurun_out/suite_xsl.jsonl
for v in jit aot; do
timeout 600 ncu --set full --clock-control none --import-source on -k regex:xs_lookup -s 1 -c 1 -f -o gpurun_out/xsl_${v} python scripts/profile_workloads.py --workload xs_large --variant $v --reps 2 > gpurun_out/prof_xsl_$v.log 2>&1; echo ncu $v rc=$?
done
