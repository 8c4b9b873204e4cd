#!/bin/bash
# One GPU-box session: parity tests, bench, ncu launch list and a full capture of the
# dominant kernel.  Outputs under gpurun_out/ (scratch; summaries go to profiles/).
set -x
TAG=${TAG:-r01}
WL=${WL:-reddit}
mkdir -p gpurun_out
python -c "import __graft_entry__ as e; e.build(); e.smoke()" > gpurun_out/smoke_$TAG.txt 2>&1
if [ "${TESTS:-1}" = "1" ]; then
  timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/tests_$TAG.txt 2>&1
fi
timeout 600 python bench.py --workload $WL $BENCH_ARGS --out gpurun_out/bench_$TAG.jsonl > gpurun_out/bench_$TAG.log 2>&1
if [ "${NCU:-1}" = "1" ]; then
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
     --log-file gpurun_out/launches_$TAG.csv python bench.py --workload $WL $BENCH_ARGS --steps 2 --warmup 1 \
     --e2e-steps 0 --no-cpu-baseline > gpurun_out/ncu_launch_$TAG.log 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:segment_kernel -s 1 -c 1 \
     -o gpurun_out/prof_$TAG -f python bench.py --workload $WL $BENCH_ARGS --steps 1 --warmup 1 \
     --e2e-steps 0 --no-cpu-baseline > gpurun_out/ncu_full_$TAG.log 2>&1
fi
tail -5 gpurun_out/tests_$TAG.txt 2>/dev/null
cat gpurun_out/bench_$TAG.log | tail -3
