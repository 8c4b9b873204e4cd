#!/bin/bash
# Re-entry sanity check on a fresh box: build + smoke, default bench line, R-MAT and bf16 lines.
O=gpurun_out/r03a; mkdir -p $O
python -c "import __graft_entry__ as e; e.build(); e.smoke()" > $O/smoke.txt 2>&1; tail -1 $O/smoke.txt
timeout 600 python bench.py --out $O/bench_default.jsonl > $O/bench_default.log 2>&1; echo "bench rc=$?"
timeout 600 python bench.py --workload rmat --K 64 --e2e-steps 0 --no-cpu-baseline --out $O/bench_rmat.jsonl > $O/bench_rmat.log 2>&1; echo "rmat rc=$?"
timeout 600 python bench.py --workload reddit --K 64 --dtype bf16 --e2e-steps 0 --no-cpu-baseline --out $O/bench_bf16.jsonl > $O/bench_bf16.log 2>&1; echo "bf16 rc=$?"
python - <<'PY'
import json,glob
for f in sorted(glob.glob("gpurun_out/r03a/bench_*.jsonl")):
    for l in open(f):
        d=json.loads(l); print(f, d["config"]["workload"], d["config"]["b_dtype"], round(d["ms_per_step"],4), round(d["value"]), d["roofline"]["frac"], d.get("parity",{}).get("ok"))
PY
