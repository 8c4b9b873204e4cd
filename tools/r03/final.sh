#!/bin/bash
# Final evidence of the round (r03z): build + smoke, the whole GPU suite, bench lines of
# every BASELINE config (fp32, bf16, graph replay), the ncu launch list of the default
# bench command, ncu --set full of the segment kernel (4 fp32 workloads + bf16 products)
# and of the small-graph kernel, X*W bench, traffic.json, compute-sanitizer.
TAG=${TAG:-r03z}
O=gpurun_out/$TAG; mkdir -p $O
python -c "import __graft_entry__ as e; e.build(); e.smoke()" > $O/smoke.txt 2>&1; tail -n 1 $O/smoke.txt
if [ "${TESTS:-1}" = "1" ]; then
  timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider > $O/tests_gpu.txt 2>&1; tail -n 3 $O/tests_gpu.txt
fi
timeout 900 python bench.py --out $O/bench_default.jsonl > $O/bench_default.log 2>&1; echo "bench rc=$?"
for c in rmat:64 reddit:256 products:128 pubmed:64 pubmed:16 cora:16; do
  timeout 900 python bench.py --workload ${c%%:*} --K ${c##*:} --out $O/bench_cfgs.jsonl > $O/bench_${c%%:*}_${c##*:}.log 2>&1; echo "bench $c rc=$?"
done
for c in cora:16 pubmed:16 pubmed:64; do
  timeout 900 python bench.py --workload ${c%%:*} --K ${c##*:} --cuda-graph --e2e-steps 0 --out $O/bench_graph.jsonl > $O/bench_graph.log 2>&1
done
for c in reddit:64 products:128 rmat:64 reddit:256; do
  timeout 900 python bench.py --workload ${c%%:*} --K ${c##*:} --dtype bf16 --e2e-steps 0 --no-cpu-baseline --out $O/bench_bf16.jsonl > $O/bench_bf16_${c%%:*}.log 2>&1
done
timeout 300 python tools/xw_bench.py > $O/xw_bench.jsonl 2>&1
if [ "${NCU:-1}" = "1" ]; then
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
     --log-file $O/ncu_launches_bench_default.csv python bench.py --steps 3 --warmup 3 \
     --e2e-steps 0 --no-cpu-baseline --no-cusparse --no-l2-probe > $O/ncu_launch.log 2>&1
  for c in reddit:64 reddit:256 products:128 rmat:64; do
    tools/prof.sh ${TAG}_${c%%:*}_k${c##*:} ${c%%:*} ${c##*:}
  done
  tools/prof.sh ${TAG}_products_k128_bf16 products 128 --dtype bf16
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:small_online -s 1 -c 1 \
     -o /tmp/prof/${TAG}_small_cora -f python bench.py --workload cora --K 16 --steps 1 --warmup 1 \
     --e2e-steps 0 --no-cpu-baseline --no-cusparse --no-l2-probe > $O/ncu_small.log 2>&1
  ncu -i /tmp/prof/${TAG}_small_cora.ncu-rep --page raw --csv > $O/ncu_full_small_cora_raw.csv 2>/dev/null
  XW_SHAPE="1000000 256 256" bash tools/prof_xw.sh ${TAG}_xw_bigF
  mv gpurun_out/ncu_${TAG}_* $O/ 2>/dev/null
  python tools/make_traffic.py $TAG $O > $O/traffic.txt 2>&1
fi
if [ "${SANITIZE:-1}" = "1" ]; then
  bash tools/sanitize.sh > /dev/null 2>&1; mv gpurun_out/compute_sanitizer.txt $O/ 2>/dev/null
fi
ls $O | head -80
