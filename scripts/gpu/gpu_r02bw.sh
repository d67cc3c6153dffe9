#!/bin/bash
# r02bw: device bounds checks (-DPROTEUS_CHECK) over every workload kernel's specialization
# at small ragged sizes, the negative control, and the GPU tests once more
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 1200 python -m pytest tests/test_gpu_bounds.py -q 2>&1 | tail -5 | tee gpurun_out/r02bw_bounds.txt
timeout 2400 python -m pytest tests -m gpu -q 2>&1 | tail -3 | tee gpurun_out/r02bw_gpu_tests.txt
