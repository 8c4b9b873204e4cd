#!/bin/bash
O=gpurun_out/r02r; mkdir -p $O
python -c "import __graft_entry__ as e; e.build()" > $O/build.txt 2>&1
MPS_L2PF=1 timeout 900 python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -x -k "integer_exact" > $O/tests_pf.txt 2>&1; tail -2 $O/tests_pf.txt
TAG=r02r ENVS="MPS_L2PF=0;MPS_L2PF=1" CFGS="rmat:64 products:128 reddit:256 reddit:64 rmat:64:bf16 products:128:bf16" bash tools/r02/abenv.sh
