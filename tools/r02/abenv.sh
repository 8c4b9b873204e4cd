#!/bin/bash
# same-box A/B of env settings on bench lines: ENVS="A=0;A=1" CFGS="rmat:64 reddit:64:bf16"
O=gpurun_out/${TAG:-abenv}
mkdir -p $O
IFS=';' read -ra EL <<< "$ENVS"
for rep in 1 2; do
for c in $CFGS; do
  IFS=':' read -ra P <<< "$c"; wl=${P[0]}; k=${P[1]}; dt=${P[2]:-f32}
  for i in "${!EL[@]}"; do
    env ${EL[$i]} timeout 600 python bench.py --workload $wl --K $k --dtype $dt --steps ${STEPS:-10} --warmup 3 --no-cpu-baseline --e2e-steps 0 --no-cusparse --no-l2-probe $EXTRA --out $O/env_$i.jsonl > $O/last.log 2>&1 || tail -3 $O/last.log
  done
done
done
python - <<'PY'
import json, glob, os, collections
O = os.environ.get("TAG", "abenv")
envs = os.environ["ENVS"].split(";")
res = collections.defaultdict(dict)
for i, e in enumerate(envs):
    f = "gpurun_out/%s/env_%d.jsonl" % (O, i)
    if not os.path.exists(f): continue
    for l in open(f):
        d = json.loads(l)
        key = d["config"]["workload"] + "-" + d["config"]["b_dtype"]
        res[key].setdefault(e, []).append((round(d["segment_ms"], 4), d["parity"]["ok"]))
for k, r in res.items():
    print(k, json.dumps(r))
PY
