#!/bin/bash
O=gpurun_out/r03s; mkdir -p $O
for rep in 1 2; do
for e in "MPS_X=0" "MPS_XW_SPLIT=2" "MPS_XW_SPLIT=4" "MPS_XW_STAGES=3" "MPS_XW_WSTREAM=1"; do
  env $e timeout 300 python tools/xw_bench.py 2>&1 | python -c "
import sys,json
for l in sys.stdin:
    try: d=json.loads(l)
    except Exception: continue
    if d['case'] in ('big-F','products'): print('$e', d['case'], round(d['tcgen05_ms'],4), round(d['cublas_ms'],4))"
done; done
