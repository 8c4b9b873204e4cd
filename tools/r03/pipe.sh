#!/bin/bash
# parity of the pipelined kernel at full size, then same-box A/B vs the round-2 head build
L=$PWD/paper_conf_ispass_shangndk23_b200
mkdir -p gpurun_out/r03pipe
MPS_PIPE=1 timeout 900 python -m pytest tests/test_gpu_fullsize.py -x -q -p no:cacheprovider -k "full_matrix_f32 or integer_exact" > gpurun_out/r03pipe/tests_pipe.txt 2>&1; tail -2 gpurun_out/r03pipe/tests_pipe.txt
TAG=r03pipe ENVS="MPS_LIB=$L/libmps_head.so;MPS_PIPE=0;MPS_PIPE=1" \
CFGS="${CFGS:-rmat:64 reddit:64 rmat:64:bf16 products:128:bf16}" bash tools/r02/abenv.sh
