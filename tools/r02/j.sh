#!/bin/bash
O=gpurun_out/r02j; mkdir -p $O
python -c "import __graft_entry__ as e; e.build()" > $O/build.txt 2>&1
MPS_ASYNC=1 timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_state.py -q -p no:cacheprovider -x > $O/tests_async.txt 2>&1; tail -2 $O/tests_async.txt
MPS_ASYNC=1 timeout 900 python -m pytest tests/test_gpu_fullsize.py -q -p no:cacheprovider -x -k "f32 or bf16" > $O/tests_async_full.txt 2>&1; tail -2 $O/tests_async_full.txt
TAG=r02j ENVS="MPS_ASYNC=0;MPS_ASYNC=1" CFGS="rmat:64 reddit:64 products:128 reddit:256 reddit:64:bf16 products:128:bf16 rmat:64:bf16 pubmed:64" bash tools/r02/abenv.sh
