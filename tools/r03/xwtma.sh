#!/bin/bash
# TMA-store epilogue of the persistent X*W kernel: parity, then same-box A/B with xw_bench
O=gpurun_out/r03y; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_xw.py tests/test_gpu_xw_bcast.py tests/test_gpu_gcn_layer_sharded.py -x -q -p no:cacheprovider > $O/tests_xw.txt 2>&1; tail -n 2 $O/tests_xw.txt
for rep in 1 2; do
  MPS_XW_TMA_STORE=0 timeout 300 python tools/xw_bench.py > $O/xw_off_$rep.jsonl 2>&1
  MPS_XW_TMA_STORE=1 timeout 300 python tools/xw_bench.py > $O/xw_on_$rep.jsonl 2>&1
done
python - <<'PY'
import json,glob
for f in sorted(glob.glob("gpurun_out/r03y/xw_*.jsonl")):
    for l in open(f):
        try: d=json.loads(l)
        except Exception: continue
        print(f.split('/')[-1], d["case"], round(d["tcgen05_ms"],4), round(d["cublas_ms"],4), round(d["tcgen05_frac_hbm"],3), d["max_abs_diff_vs_cublas"])
PY
