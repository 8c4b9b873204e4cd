#!/bin/bash
# bf16 batch-shape sweep (same box): default / 4 slow-path parts / UL=4 at 6x4 warps /
# 8-B lanes; then fp32 bench lines with the same-depth gather replay
L=$PWD/paper_conf_ispass_shangndk23_b200
TAG=r03d ENVS="MPS_X=0;MPS_LIB=$L/libexpA.so;MPS_LIB=$L/libexpB.so;MPS_MAX_W=4" \
CFGS="rmat:64:bf16 reddit:64:bf16 products:64:bf16" bash tools/r02/abenv.sh
O=gpurun_out/r03d
for c in rmat:64 reddit:64 products:128; do
  timeout 900 python bench.py --workload ${c%%:*} --K ${c##*:} --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-cusparse --out $O/bench_depth.jsonl > $O/bench_depth.log 2>&1
done
python - <<'PY'
import json
for l in open("gpurun_out/r03d/bench_depth.jsonl"):
    d=json.loads(l); a=d["roofline"].get("attainable",{})
    print(d["config"]["workload"], round(d["segment_ms"],4), "replay", round(a.get("replay_ms",0),4), round(a.get("frac",0),3), "same_depth", a.get("same_depth"))
PY
