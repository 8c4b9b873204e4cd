#!/bin/bash
# bf16 prefetch parity (new test + full-size bf16), then same-box A/B: 256-thread CTAs at
# 128 registers (default) vs 128-thread CTAs at 96 registers (5 CTAs = 20 warps/SM)
L=$PWD/paper_conf_ispass_shangndk23_b200
mkdir -p gpurun_out/r03b
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -x -q -p no:cacheprovider -k "prefetch or bf16" > gpurun_out/r03b/tests.txt 2>&1; tail -2 gpurun_out/r03b/tests.txt
MPS_LIB=$L/libexp_b128m5.so timeout 900 python -m pytest tests/test_gpu_fullsize.py -x -q -p no:cacheprovider -k "bf16" > gpurun_out/r03b/tests_exp.txt 2>&1; tail -2 gpurun_out/r03b/tests_exp.txt
TAG=r03b ENVS="MPS_X=0;MPS_LIB=$L/libexp_b128m5.so" \
CFGS="${CFGS:-reddit:64:bf16 products:128:bf16 rmat:64:bf16 reddit:256:bf16}" bash tools/r02/abenv.sh
