#!/bin/bash
# One GPU-box session: smoke, parity tests, default bench line, ncu launch list of the
# same bench command, and --set full captures (CSV exports) of the segment kernel.
TAG=${TAG:-r01}
mkdir -p gpurun_out
python -c "import __graft_entry__ as e; e.build(); e.smoke()" > gpurun_out/smoke_$TAG.txt 2>&1
if [ "${TESTS:-1}" = "1" ]; then
  timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/tests_$TAG.txt 2>&1
  tail -3 gpurun_out/tests_$TAG.txt
fi
timeout 900 python bench.py $BENCH_ARGS --out gpurun_out/bench_$TAG.jsonl > gpurun_out/bench_$TAG.log 2>&1
tail -1 gpurun_out/bench_$TAG.log | cut -c1-300
if [ "${NCU:-1}" = "1" ]; then
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
     --log-file gpurun_out/launches_$TAG.csv python bench.py $BENCH_ARGS --steps 3 --warmup 3 \
     --e2e-steps 0 --no-cpu-baseline --no-cusparse --no-l2-probe > gpurun_out/ncu_launch_$TAG.log 2>&1
  for c in ${PROF_CFGS:-reddit:64 reddit:256 products:128 rmat:64}; do
    tools/prof.sh ${TAG}_${c%%:*}_k${c##*:} ${c%%:*} ${c##*:}
  done
fi
