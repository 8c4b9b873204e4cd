#!/bin/bash
O=gpurun_out/r02q; mkdir -p $O
python -c "import __graft_entry__ as e; e.build()" > $O/build.txt 2>&1
timeout 1200 python -m pytest tests/test_gpu_bench_dist.py tests/test_gpu_parity.py -q -p no:cacheprovider -k "all_legs or strided or two_ranks" > $O/tests_new.txt 2>&1; tail -3 $O/tests_new.txt
TAG=r02q TESTS=0 NCU=0 SANITIZE=0 bash tools/r02/final.sh
