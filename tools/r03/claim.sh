#!/bin/bash
# dynamic claims two ahead (no atomic round trip at a segment start) vs one ahead
L=$PWD/paper_conf_ispass_shangndk23_b200
mkdir -p gpurun_out/r03i
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py tests/test_gpu_state.py tests/test_gpu_int64.py -x -q -p no:cacheprovider > gpurun_out/r03i/tests.txt 2>&1; tail -n 2 gpurun_out/r03i/tests.txt
TAG=r03i ENVS="MPS_X=0;MPS_LIB=$L/libexpCA0.so" \
CFGS="rmat:64 reddit:64 products:128 rmat:64:bf16 reddit:64:bf16" bash tools/r02/abenv.sh
