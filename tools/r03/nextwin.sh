#!/bin/bash
# next segment's first coordinate + row_ptr window into L1 during the current segment
L=$PWD/paper_conf_ispass_shangndk23_b200
mkdir -p gpurun_out/r03n
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py tests/test_gpu_int64.py -x -q -p no:cacheprovider -k "dynamic or full_matrix or integer or deep or prefetch or int64" > gpurun_out/r03n/tests.txt 2>&1; tail -n 2 gpurun_out/r03n/tests.txt
TAG=r03n ENVS="MPS_X=0;MPS_LIB=$L/libexpNW0.so" \
CFGS="rmat:64 reddit:64 products:128 rmat:64:bf16" bash tools/r02/abenv.sh
