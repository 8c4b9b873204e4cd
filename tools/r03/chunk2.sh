#!/bin/bash
# staging buffers in dynamic shared memory: parity of the default build, then 256 vs 512
# non-zeros per chunk (512 needs > 48 KB per CTA)
L=$PWD/paper_conf_ispass_shangndk23_b200
mkdir -p gpurun_out/r03f
python -c "import __graft_entry__ as e; e.smoke()" > gpurun_out/r03f/smoke.txt 2>&1; tail -n 1 gpurun_out/r03f/smoke.txt
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_small.py tests/test_gpu_state.py -x -q -p no:cacheprovider > gpurun_out/r03f/tests.txt 2>&1; tail -n 2 gpurun_out/r03f/tests.txt
MPS_LIB=$L/libexpC512.so timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -x -q -p no:cacheprovider -k "dynamic or deep or prefetch or full_matrix_f32 or integer" > gpurun_out/r03f/tests_512.txt 2>&1; tail -n 2 gpurun_out/r03f/tests_512.txt
TAG=r03f ENVS="MPS_X=0;MPS_LIB=$L/libexpC512.so" \
CFGS="rmat:64 reddit:64 products:128 rmat:64:bf16 reddit:64:bf16" bash tools/r02/abenv.sh
