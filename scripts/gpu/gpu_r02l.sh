#!/bin/bash
# r02l: IR-level path on the GPU (parity + compile/kernel timing), full GPU suite
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_ir.py -q -x 2>&1 | tail -15 | tee gpurun_out/r02l_ir_tests.txt
timeout 600 python scripts/exp_ir_path.py 2>&1 | tail -3 | tee gpurun_out/r02l_ir_timing.json
timeout 2400 python -m pytest tests -m gpu -x -q 2>&1 | tail -6 | tee gpurun_out/r02l_gpu_tests.txt
