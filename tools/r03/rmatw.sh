#!/bin/bash
# R-MAT K=64 fp32: lane width (16-B NR=2 default vs 8-B NR=1) and segment cost, same box
O=gpurun_out/r03r; mkdir -p $O
run() { env $1 timeout 600 python bench.py --workload rmat --K 64 --steps 10 --warmup 3 --no-cpu-baseline --e2e-steps 0 --no-cusparse --no-l2-probe $2 --out $O/r.jsonl > $O/last.log 2>&1 || tail -n 3 $O/last.log
  python -c "import json;d=[json.loads(l) for l in open('$O/r.jsonl')][-1];print('$1','$2',round(d['segment_ms'],4),d['parity']['ok'],d['config']['num_parts'])"; }
for rep in 1 2; do
run MPS_X=0 ""
run MPS_MAX_W=2 ""
run MPS_X=0 "--items-per-part 256"
run MPS_X=0 "--items-per-part 1024"
run MPS_MAX_W=2 "--items-per-part 1024"
done
