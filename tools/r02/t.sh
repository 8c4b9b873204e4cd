#!/bin/bash
O=gpurun_out/r02t; mkdir -p $O
python -c "import __graft_entry__ as e; e.build(); e.smoke()" > $O/smoke.txt 2>&1; tail -1 $O/smoke.txt
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_small.py -q -p no:cacheprovider -k "gcn or small" > $O/tests.txt 2>&1; tail -2 $O/tests.txt
timeout 1200 python tools/gcn_bench.py > $O/gcn_bench.jsonl 2>&1; cat $O/gcn_bench.jsonl
for c in "reddit:64" "reddit:256" "products:128" "rmat:64" "pubmed:64" "pubmed:16" "cora:16"; do
  for dt in f32 bf16; do
    for fx in auto carry; do
      timeout 600 python bench.py --workload ${c%%:*} --K ${c##*:} --dtype $dt --fixup $fx --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-cusparse --out $O/sweep.jsonl > $O/last.log 2>&1 || echo "FAIL $c $dt $fx"
    done
  done
done
python - <<'PY'
import json
for l in open("gpurun_out/r02t/sweep.jsonl"):
    d=json.loads(l); c=d["config"]; r=d["roofline"]
    print(c["workload"], c["b_dtype"], c["fixup"], c["path"][:12], "ms %.4f" % d["ms_per_step"], "GF %.0f" % d["value"], "frac %.3f" % r["frac"], "parity", d["parity"]["ok"])
PY
