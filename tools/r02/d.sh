#!/bin/bash
O=gpurun_out/r02d; mkdir -p $O
python -c "import __graft_entry__ as e; e.build()" > $O/build.txt 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_small.py tests/test_gpu_state.py -q -p no:cacheprovider > $O/tests.txt 2>&1; tail -2 $O/tests.txt
timeout 600 python tools/r02/floor.py > $O/floor.txt 2>&1; cat $O/floor.txt
TAG=r02d LIBS="lib_pass.so lib_steps.so" CFGS="rmat:64 reddit:64 products:128 reddit:256" bash tools/r02/ab.sh
TAG=r02d LIBS="lib_pass.so lib_steps.so" CFGS="pubmed:64 pubmed:16" EXTRA="--fixup atomic" bash tools/r02/ab.sh
tools/prof.sh r02d_rmat_k64 rmat 64
ncu -i /tmp/prof/r02d_rmat_k64.ncu-rep --page source --csv --print-source cuda,sass > $O/ncu_rmat_cuda_sass.csv 2>/dev/null
mv gpurun_out/ncu_r02d_rmat_k64* $O/ 2>/dev/null
