#!/bin/bash
# r02by: micro_column PROD with the plain IEEE division instead of div_s (bit-identical by
# construction; only the zero-dividend slow path differs)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
AB="-DMICRO_PROD_PLAIN_DIV=0;-DMICRO_PROD_PLAIN_DIV=1" timeout 900 python scripts/ab_micro.py 2>&1 | tee gpurun_out/ab_micro_prod_r02by.txt
