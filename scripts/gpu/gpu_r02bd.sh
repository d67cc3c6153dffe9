#!/bin/bash
# r02bd: XS e2e incl. JIT after XS_PACK, fresh processes (the 2 s job: 1 500 steps; and the
# paper's RSBench AOT length, 2 200 steps)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 2400 python bench_suite.py --configs e2e:xs@1500 --runs 5 2>&1 | tail -1 | tee gpurun_out/e2e_2s_xs_r02bd.jsonl
timeout 2400 python bench_suite.py --configs e2e:xs@2200 --runs 5 2>&1 | tail -1 | tee gpurun_out/e2e_rsbench_scale_xs_r02bd.jsonl
