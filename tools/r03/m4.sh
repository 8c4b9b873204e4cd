#!/bin/bash
# fp32 at 4 x 8 warps per SM (64 registers, slow-path values from shared memory, some
# spills; 384-non-zero chunks to fit 32 warps' staging) vs the default 3 x 8 at 80
L=$PWD/paper_conf_ispass_shangndk23_b200
TAG=r03h ENVS="MPS_X=0;MPS_LIB=$L/libexpM4.so;MPS_LIB=$L/libexpC384.so" \
CFGS="rmat:64 reddit:64 reddit:256" bash tools/r02/abenv.sh
