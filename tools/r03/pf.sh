#!/bin/bash
# A/B of the next-batch L2 prefetch (MPS_PF) against the round-2 head build, one box
L=$PWD/paper_conf_ispass_shangndk23_b200
TAG=r03pf ENVS="MPS_LIB=$L/libmps_head.so;MPS_PF=0;MPS_PF=1;MPS_PF=2" \
CFGS="${CFGS:-rmat:64 rmat:64:bf16 products:128 products:128:bf16 reddit:64}" bash tools/r02/abenv.sh
