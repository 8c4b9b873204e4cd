#!/bin/bash
O=gpurun_out/r02f; mkdir -p $O
python -c "import __graft_entry__ as e; e.build()" > $O/build.txt 2>&1
B="--cuda-graph --steps 30 --warmup 5 --e2e-steps 0 --no-cpu-baseline --no-l2-probe"
for wl in cora:16 pubmed:16 pubmed:64; do
  timeout 300 python bench.py --workload ${wl%%:*} --K ${wl##*:} $B --out $O/tiny.jsonl > $O/last.log 2>&1 || tail -5 $O/last.log
  timeout 300 python bench.py --workload ${wl%%:*} --K ${wl##*:} --steps 30 --warmup 5 --e2e-steps 0 --no-cpu-baseline --no-l2-probe --out $O/tiny.jsonl > $O/last.log 2>&1 || tail -5 $O/last.log
done
python - <<'PY'
import json
for l in open("gpurun_out/r02f/tiny.jsonl"):
    d=json.loads(l); c=d["config"]
    print(c["workload"], "graph" if c["cuda_graph"] else "eager", c.get("path"), "ms %.4f" % d["ms_per_step"], "min/med", [round(x, 4) for x in d["step_ms_min_median"]], "cusparse", (d.get("cusparse") or {}).get("ms"), "parity", d["parity"]["ok"])
PY
TAG=r02f LIBS="lib_base.so lib_dyncap4.so lib_minb2.so" CFGS="rmat:64 reddit:64 products:128 reddit:256" bash tools/r02/ab.sh
MPS_LIB=$PWD/paper_conf_ispass_shangndk23_b200/lib_base.so tools/prof.sh r02f_rmat_k64 rmat 64
ncu -i /tmp/prof/r02f_rmat_k64.ncu-rep --page source --csv --print-source cuda,sass > $O/ncu_rmat_cuda_sass.csv 2>/dev/null
mv gpurun_out/ncu_r02f_rmat_k64* $O/ 2>/dev/null
