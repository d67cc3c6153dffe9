#!/bin/bash
# r02aa: new parity cases (micro nsub/nz, XS block sizes, non-cubic stencil)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 1200 python -m pytest tests/test_gpu_parity_full.py -q -x -k "other or non_cubic" 2>&1 | tail -5 | tee gpurun_out/r02aa_tests.txt
