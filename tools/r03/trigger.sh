#!/bin/bash
# partition kernel triggers its dependents at its start (PDL) vs at exit; CUDA-graph
# replay of the online step (no inner events between the two kernels)
L=$PWD/paper_conf_ispass_shangndk23_b200
O=gpurun_out/r03v; mkdir -p $O
timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_state.py -x -q -p no:cacheprovider > $O/tests.txt 2>&1; tail -n 1 $O/tests.txt
for rep in 1 2; do
for c in rmat:64 reddit:64 products:128; do
  for e in "MPS_X=0" "MPS_LIB=$L/libexpPT0.so"; do
    env $e timeout 600 python bench.py --workload ${c%%:*} --K ${c##*:} --steps 20 --warmup 5 --cuda-graph --e2e-steps 0 --no-cpu-baseline --no-cusparse --no-l2-probe --out $O/g.jsonl > $O/last.log 2>&1 || tail -n 3 $O/last.log
    python -c "import json;d=[json.loads(l) for l in open('$O/g.jsonl')][-1];print('$c','${e:0:12}',round(d['ms_per_step'],4),d['parity']['ok'])"
  done
done; done
