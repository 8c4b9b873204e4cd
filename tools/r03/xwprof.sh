#!/bin/bash
# NEXT-3 big-F: xw_bench of all shapes + ncu --set full (source page) of the big-F kernel
mkdir -p gpurun_out/r03x
timeout 300 python tools/xw_bench.py > gpurun_out/r03x/xw_bench.jsonl 2>&1; cat gpurun_out/r03x/xw_bench.jsonl | cut -c1-200
XW_SHAPE="1000000 256 256" bash tools/prof_xw.sh r03x_bigF
mv gpurun_out/ncu_r03x_bigF* gpurun_out/r03x/ 2>/dev/null
python tools/ncu_source.py gpurun_out/r03x/ncu_r03x_bigF_sass.csv 40 > gpurun_out/r03x/bigF_stalls.txt 2>&1; head -60 gpurun_out/r03x/bigF_stalls.txt
