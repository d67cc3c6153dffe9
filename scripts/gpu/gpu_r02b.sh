#!/bin/bash
# r02: new parity tests (full-size, long-run, tie rule, z-slab split, 2-rank bench) + micro with R-mp-3
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 1500 python -m pytest tests/test_gpu_parity_full.py tests/test_gpu_bench_multirank.py -q -x -rA 2>&1 | tail -30 | tee gpurun_out/r02b_full.txt
timeout 900 python -m pytest tests/test_gpu_parity.py -q -k "micro or spec" 2>&1 | tail -5 | tee gpurun_out/r02b_micro.txt
