#!/bin/bash
# with 512-non-zero chunks: segment cost and the deep-gather kernel, same box
O=gpurun_out/r03g; mkdir -p $O
run() { env $1 timeout 600 python bench.py --workload $2 --K $3 --dtype $4 --steps 10 --warmup 3 --no-cpu-baseline --e2e-steps 0 --no-cusparse --no-l2-probe $5 --out $O/r.jsonl > $O/last.log 2>&1 || tail -n 3 $O/last.log
  python -c "import json;d=[json.loads(l) for l in open('$O/r.jsonl')][-1];print('$1','$2','$3','$4','$5',round(d['segment_ms'],4),d['parity']['ok'],d['config']['num_parts'])"; }
for rep in 1 2; do
run MPS_X=0 rmat 64 f32 ""
run MPS_X=0 rmat 64 f32 "--items-per-part 1024"
run MPS_DEEP=1 rmat 64 f32 ""
run MPS_X=0 products 128 f32 ""
run MPS_X=0 products 128 f32 "--items-per-part 1024"
run MPS_DEEP=0 products 128 f32 ""
run MPS_X=0 reddit 64 f32 ""
run MPS_X=0 reddit 64 f32 "--items-per-part 4096"
run MPS_X=0 rmat 64 bf16 ""
run MPS_X=0 rmat 64 bf16 "--items-per-part 1024"
done
