#!/bin/bash
O=gpurun_out/r02s; mkdir -p $O
python -c "import __graft_entry__ as e; e.build()" > $O/build.txt 2>&1
MPS_LIB=$PWD/paper_conf_ispass_shangndk23_b200/lib_skip.so timeout 900 python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -x -k "integer_exact" > $O/tests_skip.txt 2>&1; tail -2 $O/tests_skip.txt
TAG=r02s LIBS="lib_base.so lib_skip.so" CFGS="rmat:64 reddit:64 products:128 reddit:256" bash tools/r02/ab.sh
TAG=r02s LIBS="lib_base.so lib_skip.so" CFGS="reddit:64 rmat:64" EXTRA="--dtype bf16" bash tools/r02/ab.sh
TAG=r02s2 LIBS="lib_base.so lib_skip.so" CFGS="pubmed:64 pubmed:16" EXTRA="--fixup atomic" bash tools/r02/ab.sh
