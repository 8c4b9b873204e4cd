#!/bin/bash
# 128-thread CTAs at 96 registers also for the two-rows-per-instruction bf16 kernels
# (256-B bf16 rows: products K=128, Reddit K=256), slow path in two parts
L=$PWD/paper_conf_ispass_shangndk23_b200
mkdir -p gpurun_out/r03j
MPS_LIB=$L/libexpNR2.so timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -x -q -p no:cacheprovider -k "bf16 or prefetch" > gpurun_out/r03j/tests_exp.txt 2>&1; tail -n 2 gpurun_out/r03j/tests_exp.txt
TAG=r03j ENVS="MPS_X=0;MPS_LIB=$L/libexpNR2.so" \
CFGS="products:128:bf16 reddit:256:bf16 rmat:128:bf16" bash tools/r02/abenv.sh
