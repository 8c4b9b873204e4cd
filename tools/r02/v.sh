#!/bin/bash
O=gpurun_out/r02v; mkdir -p $O
python -c "import __graft_entry__ as e; e.build()" > $O/build.txt 2>&1
MPS_LIB=$PWD/paper_conf_ispass_shangndk23_b200/lib_er.so timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_small.py -q -p no:cacheprovider -x > $O/tests_er.txt 2>&1; tail -1 $O/tests_er.txt
MPS_LIB=$PWD/paper_conf_ispass_shangndk23_b200/lib_er.so timeout 900 python -m pytest tests/test_gpu_fullsize.py -q -p no:cacheprovider -x -k "rmat and (integer or f32)" > $O/tests_er_full.txt 2>&1; tail -1 $O/tests_er_full.txt
TAG=r02v LIBS="lib_base.so lib_er.so" CFGS="rmat:64 reddit:64 products:128" bash tools/r02/ab.sh
TAG=r02v2 LIBS="lib_base.so lib_er.so" CFGS="rmat:64 reddit:64" EXTRA="--dtype bf16" bash tools/r02/ab.sh
TAG=r02v3 LIBS="lib_base.so lib_er.so" CFGS="pubmed:64 cora:16" EXTRA="--fixup atomic" bash tools/r02/ab.sh
