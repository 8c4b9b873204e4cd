#!/bin/bash
# tiny graphs: small-graph fused path vs partition+segments, CUDA-graph replay, L2 flushed
O=gpurun_out/${TAG:-r02c}
mkdir -p $O
python -c "import __graft_entry__ as e; e.build(); e.smoke()" > $O/smoke.txt 2>&1; tail -1 $O/smoke.txt
timeout 900 python -m pytest tests/test_gpu_small.py tests/test_gpu_state.py tests/test_gpu_parity.py -q -p no:cacheprovider > $O/tests_small.txt 2>&1; tail -3 $O/tests_small.txt
B="--cuda-graph --steps 30 --warmup 5 --e2e-steps 0 --no-cpu-baseline --no-l2-probe"
for wl in cora:16 pubmed:16 pubmed:64; do
  for fx in auto atomic; do
    for ipp in ${IPPS:-0}; do
      timeout 300 python bench.py --workload ${wl%%:*} --K ${wl##*:} --fixup $fx --items-per-part $ipp $B --out $O/tiny.jsonl > $O/last.log 2>&1 || tail -5 $O/last.log
    done
  done
done
python - <<'PY'
import json,os
O=os.environ.get("TAG","r02c")
for l in open("gpurun_out/%s/tiny.jsonl"%O):
    d=json.loads(l); c=d["config"]
    print(c["workload"], c["fixup"], c.get("path"), "ipp", c["items_per_part"], "P", c["num_parts"], "ms %.4f"%d["ms_per_step"], "cusparse", (d.get("cusparse") or {}).get("ms"), "parity", d["parity"]["ok"])
PY
