#!/bin/bash
# r02al: XS e2e at the paper's RSBench scale (NVIDIA AOT 2.67 s, Table 2 -> ~2200 steps of 10^7 lookups)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 1200 python bench_suite.py --configs e2e:xs@2200 --runs 5 > gpurun_out/e2e_rsbench_scale_xs_r02al.jsonl 2> gpurun_out/e2e_rsbench_scale_xs_r02al.err; echo e2e rc=$?
