#!/bin/bash
# 128-thread CTAs at 96 registers for the 4/8-rows-per-instruction bf16 kernels (slow-path
# values re-read from shared memory: no spills) vs the default 256-thread CTAs at 128
L=$PWD/paper_conf_ispass_shangndk23_b200
mkdir -p gpurun_out/r03c
MPS_LIB=$L/libexp_b128.so timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -x -q -p no:cacheprovider -k "bf16 or prefetch or dynamic" > gpurun_out/r03c/tests_exp.txt 2>&1; tail -n 2 gpurun_out/r03c/tests_exp.txt
TAG=r03c ENVS="MPS_X=0;MPS_LIB=$L/libexp_b128.so" \
CFGS="${CFGS:-reddit:64:bf16 rmat:64:bf16 products:64:bf16}" bash tools/r02/abenv.sh
