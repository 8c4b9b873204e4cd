#!/bin/bash
# ncu --set full of the segment kernel for one workload; keeps the .ncu-rep on the box
# (/tmp) and exports the raw + source pages as CSV into gpurun_out/ (small).
# Usage: ./prof.sh TAG WORKLOAD K [extra bench args]
TAG=$1; WL=$2; K=$3; shift 3
mkdir -p gpurun_out /tmp/prof
timeout 900 ncu --set full --clock-control none --cache-control ${CACHE_CONTROL:-all} --import-source on -k regex:segment_kernel -s 1 -c 1 \
  -o /tmp/prof/$TAG -f python bench.py --workload $WL --K $K --steps 1 --warmup 1 --e2e-steps 0 \
  --no-cpu-baseline "$@" > gpurun_out/ncu_$TAG.log 2>&1
ncu -i /tmp/prof/$TAG.ncu-rep --page raw --csv > gpurun_out/ncu_${TAG}_raw.csv 2>/dev/null
ncu -i /tmp/prof/$TAG.ncu-rep --page details --csv > gpurun_out/ncu_${TAG}_details.csv 2>/dev/null
ncu -i /tmp/prof/$TAG.ncu-rep --page source --csv --print-source sass > gpurun_out/ncu_${TAG}_sass.csv 2>/dev/null
if [ "${KEEP_REP:-0}" = "1" ]; then cp /tmp/prof/$TAG.ncu-rep gpurun_out/; fi
