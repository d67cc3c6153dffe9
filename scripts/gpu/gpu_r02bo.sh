#!/bin/bash
# r02bo: Adam e2e incl. JIT at the upper end of the paper's ADAM job lengths (Table 2: AOT
# 2.0-2.9 s): 55 000 adam_run launches (~2.7 s AOT), fresh processes, 5 rotated runs
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 2400 python bench_suite.py --configs e2e:adam_run@55000 --runs 5 2>&1 | tail -1 | tee gpurun_out/e2e_adam_run_55k_r02bo.jsonl
