#!/bin/bash
O=gpurun_out/r02u; mkdir -p $O
python -c "import __graft_entry__ as e; e.build()" > $O/build.txt 2>&1
for l in lib_sp2.so lib_sp4.so; do
MPS_LIB=$PWD/paper_conf_ispass_shangndk23_b200/$l timeout 900 python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -x -k "integer_exact" > $O/tests_$l.txt 2>&1; tail -1 $O/tests_$l.txt
done
TAG=r02u LIBS="lib_base.so lib_sp2.so lib_sp4.so" CFGS="rmat:64 reddit:64 products:128" bash tools/r02/ab.sh
TAG=r02u2 LIBS="lib_base.so lib_sp2.so lib_sp4.so" CFGS="rmat:64 reddit:64" EXTRA="--dtype bf16" bash tools/r02/ab.sh
TAG=r02u3 LIBS="lib_base.so lib_sp2.so lib_sp4.so" CFGS="pubmed:64 pubmed:16" EXTRA="--fixup atomic" bash tools/r02/ab.sh
