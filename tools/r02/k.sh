#!/bin/bash
O=gpurun_out/r02k; mkdir -p $O
python -c "import __graft_entry__ as e; e.build()" > $O/build.txt 2>&1
MPS_ASYNC=1 timeout 900 python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -x -k "integer_exact" > $O/tests_async.txt 2>&1; tail -2 $O/tests_async.txt
timeout 900 python -m pytest tests/test_gpu_xw.py -q -p no:cacheprovider > $O/tests_xw.txt 2>&1; tail -2 $O/tests_xw.txt
TAG=r02k ENVS="MPS_ASYNC=0;MPS_ASYNC=1" CFGS="reddit:64 rmat:64 reddit:64:bf16 rmat:64:bf16" bash tools/r02/abenv.sh
MPS_ASYNC=1 tools/prof.sh r02k_async_reddit reddit 64
mv gpurun_out/ncu_r02k_async_reddit* $O/ 2>/dev/null
python tools/xw_bench.py > $O/xw_bench.txt 2>&1; tail -8 $O/xw_bench.txt
MPS_XW_WSTREAM=1 python tools/xw_bench.py > $O/xw_bench_wstream.txt 2>&1; tail -8 $O/xw_bench_wstream.txt
