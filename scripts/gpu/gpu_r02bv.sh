#!/bin/bash
# r02bv: the 2 s fresh-process e2e jobs of the stencil and the microphysics on the final build
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 2400 python bench_suite.py --configs e2e:stencil@36000 --runs 5 2>&1 | tail -1 | tee gpurun_out/e2e_2s_stencil_r02bv.jsonl
timeout 2400 python bench_suite.py --configs e2e:micro@1000 --runs 5 2>&1 | tail -1 | tee gpurun_out/e2e_2s_micro_r02bv.jsonl
