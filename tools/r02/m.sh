#!/bin/bash
O=gpurun_out/r02m; mkdir -p $O
python -c "import __graft_entry__ as e; e.build()" > $O/build.txt 2>&1
MPS_ASYNC=1 timeout 900 python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -x -k "integer_exact" > $O/tests_async.txt 2>&1; tail -2 $O/tests_async.txt
TAG=r02m ENVS="MPS_ASYNC=0;MPS_ASYNC=1" CFGS="reddit:64 rmat:64 reddit:64:bf16 rmat:64:bf16" bash tools/r02/abenv.sh
