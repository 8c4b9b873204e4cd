#!/bin/bash
# col/val staging chunk size (non-zeros per warp per TMA chunk): 256 (default) vs 128 / 512
L=$PWD/paper_conf_ispass_shangndk23_b200
TAG=r03e ENVS="MPS_X=0;MPS_LIB=$L/libexpC128.so;MPS_LIB=$L/libexpC512.so" \
CFGS="rmat:64 reddit:64 products:128 rmat:64:bf16" bash tools/r02/abenv.sh
