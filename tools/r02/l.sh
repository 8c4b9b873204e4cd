#!/bin/bash
O=gpurun_out/r02l; mkdir -p $O
python -c "import __graft_entry__ as e; e.build()" > $O/build.txt 2>&1
MPS_ASYNC=1 timeout 600 compute-sanitizer --tool memcheck python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -x -k "bf16_integer_exact and 256 and atomic" > $O/sanit_async.txt 2>&1; grep -E "Invalid|Error|passed|failed|at 0x|by thread" $O/sanit_async.txt | head -20
TAG=r02l ENVS="MPS_ASYNC=0;MPS_ASYNC=1" CFGS="reddit:64 rmat:64 products:128 reddit:64:bf16 rmat:64:bf16" bash tools/r02/abenv.sh
python tools/xw_bench.py > $O/xw_bench.txt 2>&1; tail -5 $O/xw_bench.txt
