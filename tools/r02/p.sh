#!/bin/bash
O=gpurun_out/r02p; mkdir -p $O
python -c "import __graft_entry__ as e; e.build()" > $O/build.txt 2>&1
TAG=r02p LIBS="lib_base.so lib_bf16a.so" CFGS="reddit:64 products:128 rmat:64" EXTRA="--dtype bf16" bash tools/r02/ab.sh
TAG=r02p2 ENVS="MPS_MAX_W=8;MPS_MAX_W=4" CFGS="reddit:64:bf16 products:128:bf16 rmat:64:bf16" bash tools/r02/abenv.sh
