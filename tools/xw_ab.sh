#!/bin/bash
# same-box A/B of the tcgen05 combination kernel's knobs (MPS_XW_PERSIST / _STAGED / _STAGES)
CFGS=${CFGS:-"MPS_XW_STAGED=1 MPS_XW_STAGED=0 MPS_XW_PERSIST=0"}
for cfg in $CFGS; do echo "$cfg"; env $cfg timeout 300 python tools/xw_bench.py 2>&1 | tail -5 | python -c "
import sys,json
for l in sys.stdin:
    d=json.loads(l); print('  ', d['case'], round(d['tcgen05_ms'],4), round(d['cublas_ms'],4), round(d['tcgen05_frac_hbm'],3))"; done
