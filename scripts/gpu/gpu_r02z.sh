#!/bin/bash
# r02z: xs_lookup without the result staging -- XS parity + timing
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_parity_full.py tests/test_gpu_ir.py tests/test_gpu_edge.py tests/test_gpu_sanitizer.py -q -x -k "xs" 2>&1 | tail -2 | tee gpurun_out/r02z_tests.txt
timeout 300 python scripts/xs_step_breakdown.py 2>&1 | tail -4 | tee -a gpurun_out/r02z_tests.txt
