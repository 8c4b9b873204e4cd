#!/bin/bash
# blocked batch-entry mapping (each lane's entries contiguous: 16-B LDS of col/val) for
# the one-part fp32 kernels vs the interleaved default
L=$PWD/paper_conf_ispass_shangndk23_b200
mkdir -p gpurun_out/r03x2
MPS_LIB=$L/libexpBLK.so timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py tests/test_gpu_small.py -x -q -p no:cacheprovider -k "not bf16" > gpurun_out/r03x2/tests_exp.txt 2>&1; tail -n 1 gpurun_out/r03x2/tests_exp.txt
TAG=r03x2 ENVS="MPS_X=0;MPS_LIB=$L/libexpBLK.so" CFGS="rmat:64 reddit:64 reddit:256" bash tools/r02/abenv.sh
