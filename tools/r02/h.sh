#!/bin/bash
O=gpurun_out/r02h; mkdir -p $O
python -c "import __graft_entry__ as e; e.build()" > $O/build.txt 2>&1
for c in reddit:64 rmat:64 products:128 reddit:256; do
  timeout 600 python bench.py --workload ${c%%:*} --K ${c##*:} --steps 10 --no-cpu-baseline --e2e-steps 0 --no-cusparse --out $O/roof.jsonl > $O/last.log 2>&1 || tail -5 $O/last.log
done
for c in reddit:64 products:128; do
  timeout 600 python bench.py --workload ${c%%:*} --K ${c##*:} --dtype bf16 --steps 10 --no-cpu-baseline --e2e-steps 0 --no-cusparse --out $O/roof.jsonl > $O/last.log 2>&1 || tail -5 $O/last.log
done
python - <<'PY'
import json
for l in open("gpurun_out/r02h/roof.jsonl"):
    d = json.loads(l); r = d["roofline"]
    print(d["config"]["workload"], d["config"]["b_dtype"], "seg %.4f" % d["segment_ms"], "bound", r["bound"], "frac %.3f" % r["frac"], "attainable", json.dumps(r.get("attainable")), "units", json.dumps(r.get("units_frac_against")), r.get("attainable_error"))
PY
