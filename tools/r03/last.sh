#!/bin/bash
# last capture of the round: NEXT-1 sweep (fp32 + bf16) with the bf16 cost rule, the whole
# GPU suite, smoke and the default bench line at the final build
O=gpurun_out/r03t; mkdir -p $O
python -c "import __graft_entry__ as e; e.build(); e.smoke()" > $O/smoke.txt 2>&1; tail -n 1 $O/smoke.txt
SENS_DTYPE=bf16 SENS_KS="16 64 128 256" timeout 1500 python tools/sensitivity.py --out $O/sens_bf16.jsonl > $O/sens_bf16.log 2>&1
timeout 2300 python tools/sensitivity.py --out $O/sens_f32.jsonl > $O/sens_f32.log 2>&1
python tools/sensitivity_summary.py $O/sens_f32.jsonl > $O/summary_f32.md 2>&1
python tools/sensitivity_summary.py $O/sens_bf16.jsonl > $O/summary_bf16.md 2>&1
head -n 12 $O/summary_bf16.md
timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider > $O/tests_gpu.txt 2>&1; tail -n 2 $O/tests_gpu.txt
timeout 900 python bench.py --out $O/bench_default.jsonl > $O/bench_default.log 2>&1; echo "bench rc=$?"
