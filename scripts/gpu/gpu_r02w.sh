#!/bin/bash
# r02w: proteus_prefetch on the GPU -- XS tests, XS e2e (~2 s, 5 runs), the suite's XS entry
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_parity_full.py tests/test_gpu_ir.py tests/test_gpu_runtime.py -q -x -k "xs or prefetch or runtime" 2>&1 | tail -2 | tee gpurun_out/r02w_tests.txt
timeout 1500 python bench_suite.py --configs e2e:xs@1500 --runs 5 > gpurun_out/e2e_2s_xs_r02w.jsonl 2>&1; echo rc=$?
