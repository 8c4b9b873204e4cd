#!/bin/bash
# same-box A/B of library builds on bench lines: LIBS="a.so b.so" CFGS="rmat:64 reddit:64"
O=gpurun_out/${TAG:-ab}
mkdir -p $O
for rep in 1 2; do
for c in $CFGS; do
  for lib in $LIBS; do
    MPS_LIB=$PWD/paper_conf_ispass_shangndk23_b200/$lib timeout 600 python bench.py --workload ${c%%:*} --K ${c##*:} --steps ${STEPS:-10} --warmup 3 --no-cpu-baseline --e2e-steps 0 --no-cusparse --no-l2-probe $EXTRA --out $O/ab_${lib%.so}.jsonl > $O/last.log 2>&1 || tail -3 $O/last.log
  done
done
done
python - <<'PY'
import json, glob, os, collections
O = os.environ.get("TAG", "ab")
res = collections.defaultdict(dict)
for f in sorted(glob.glob("gpurun_out/%s/ab_*.jsonl" % O)):
    lib = os.path.basename(f)[3:-6]
    for l in open(f):
        d = json.loads(l)
        res[d["config"]["workload"]].setdefault(lib, []).append(round(d["segment_ms"], 4))
for wl, r in res.items():
    print(wl, json.dumps(r))
PY
