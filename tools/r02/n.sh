#!/bin/bash
# NEXT-1 sensitivity study additions (K=256 fp32 and bf16; kernel-side Fig. 5 counters at
# K=16) and one ncu capture of the big-F X*W GEMM
O=gpurun_out/r02n; mkdir -p $O
python -c "import __graft_entry__ as e; e.build()" > $O/build.txt 2>&1
SENS_KS="16" timeout 1800 python tools/sensitivity.py --out $O/sens_k16_counts.jsonl > $O/sens16.log 2>&1; tail -2 $O/sens16.log
SENS_KS="256" SENS_STATS_K=256 timeout 1800 python tools/sensitivity.py --out $O/sens_k256_f32.jsonl > $O/sens256.log 2>&1; tail -2 $O/sens256.log
SENS_DTYPE=bf16 SENS_KS="256" SENS_STATS_K=0 timeout 1800 python tools/sensitivity.py --out $O/sens_k256_bf16.jsonl > $O/sens256b.log 2>&1; tail -2 $O/sens256b.log
XW_SHAPE="1000000 256 256" tools/prof_xw.sh r02n_xw_bigF
mv gpurun_out/ncu_r02n_xw_bigF* $O/ 2>/dev/null
