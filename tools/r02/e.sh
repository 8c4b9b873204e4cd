#!/bin/bash
O=gpurun_out/r02e; mkdir -p $O
python -c "import __graft_entry__ as e; e.build(); e.smoke()" > $O/smoke.txt 2>&1; tail -1 $O/smoke.txt
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_small.py tests/test_gpu_state.py -q -p no:cacheprovider > $O/tests.txt 2>&1; tail -2 $O/tests.txt
timeout 600 python tools/r02/floor.py > $O/floor.txt 2>&1; cat $O/floor.txt
B="--cuda-graph --steps 30 --warmup 5 --e2e-steps 0 --no-cpu-baseline --no-l2-probe"
for wl in cora:16 pubmed:16 pubmed:64; do
  for fx in auto atomic; do
    timeout 300 python bench.py --workload ${wl%%:*} --K ${wl##*:} --fixup $fx $B --out $O/tiny.jsonl > $O/last.log 2>&1 || tail -5 $O/last.log
  done
done
for wl in rmat:64 reddit:64; do
  timeout 300 python bench.py --workload ${wl%%:*} --K ${wl##*:} --steps 10 --e2e-steps 0 --no-cpu-baseline --no-cusparse --out $O/big.jsonl > $O/last.log 2>&1 || tail -5 $O/last.log
done
python - <<'PY'
import json
for f in ("tiny", "big"):
    for l in open("gpurun_out/r02e/%s.jsonl" % f):
        d=json.loads(l); c=d["config"]
        print(c["workload"], c["fixup"], c.get("path"), "ms %.4f" % d["ms_per_step"], "min/med", [round(x, 4) for x in d["step_ms_min_median"]], "part %.4f seg %.4f" % (d["partition_zero_ms"], d["segment_ms"]), "cusparse", (d.get("cusparse") or {}).get("ms"), "parity", d["parity"]["ok"])
PY
