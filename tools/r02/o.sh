#!/bin/bash
O=gpurun_out/r02o; mkdir -p $O
python -c "import __graft_entry__ as e; e.build()" > $O/build.txt 2>&1
TAG=r02o LIBS="lib_base.so lib_bc1.so" CFGS="rmat:64 reddit:64 products:128 reddit:256" bash tools/r02/ab.sh
TAG=r02o LIBS="lib_base.so lib_bc1.so" CFGS="pubmed:64 pubmed:16" EXTRA="--fixup atomic" bash tools/r02/ab.sh
tools/prof.sh r02o_rmat_k64 rmat 64
mv gpurun_out/ncu_r02o_rmat_k64* $O/ 2>/dev/null
python tools/ncu_summary.py $O/ncu_r02o_rmat_k64_raw.csv | grep -E "time_dur|inst_executed.sum|issue_active"
