#!/bin/bash
# fp32 dynamic two-rows kernel with 10 gathers per lane (U = 20, slow-path values from
# shared memory, 320-non-zero chunks) vs the default 8 (512 chunks) and a 320-chunk control
L=$PWD/paper_conf_ispass_shangndk23_b200
mkdir -p gpurun_out/r03k
MPS_LIB=$L/libexpUL10.so timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -x -q -p no:cacheprovider -k "dynamic or f32 or integer or deep" > gpurun_out/r03k/tests_exp.txt 2>&1; tail -n 2 gpurun_out/r03k/tests_exp.txt
TAG=r03k ENVS="MPS_X=0;MPS_LIB=$L/libexpUL10.so;MPS_LIB=$L/libexpC320.so" \
CFGS="rmat:64 reddit:64 reddit:256" bash tools/r02/abenv.sh
