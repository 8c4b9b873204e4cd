#!/bin/bash
# Bench sweep on the GPU box: every BASELINE workload/K, optional items_per_part list.
# Usage: TAG=x IPP="0 256 1024" FIX="atomic" ./sweep.sh
TAG=${TAG:-sweep}
IPP=${IPP:-0}
FIX=${FIX:-atomic}
CFGS=${CFGS:-"reddit:64 reddit:256 products:128 rmat:64 pubmed:64 cora:16"}
mkdir -p gpurun_out
python -c "import __graft_entry__ as e; e.build()"
if [ "${TESTS:-1}" = "1" ]; then
  timeout 900 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/tests_$TAG.txt 2>&1
  tail -3 gpurun_out/tests_$TAG.txt
fi
for c in $CFGS; do
  wl=${c%%:*}; k=${c##*:}
  for ipp in $IPP; do
    for fx in $FIX; do
      timeout 300 python bench.py --workload $wl --K $k --items-per-part $ipp --fixup $fx --steps 10 --warmup 3 \
        --e2e-steps 0 --no-cpu-baseline $EXTRA --out gpurun_out/sweep_$TAG.jsonl > /dev/null 2>gpurun_out/sweep_err_$TAG.txt || echo "FAIL $wl $k $ipp $fx"
    done
  done
done
python - <<'PY'
import json,os
tag=os.environ.get('TAG','sweep')
for l in open(f'gpurun_out/sweep_{tag}.jsonl'):
    d=json.loads(l); c=d['config']
    print(f"{c['workload']:14s} ipp={c['items_per_part']:5d} P={c['num_parts']:7d} {c['fixup']:6s} {c['b_dtype']} step={d['ms_per_step']:.3f}ms seg={d['segment_ms']:.3f}ms GF={d['value']:.0f} frac={d['roofline']['frac']:.2f}")
PY
