#!/bin/bash
# ncu --set full of the tcgen05 combination kernel (products shape: n=2.45M, F=100, N=128)
TAG=${1:-xw}
mkdir -p gpurun_out /tmp/prof
cat > /tmp/prof/xw_once.py <<'PY'
import sys, os
sys.path.insert(0, os.getcwd())
import torch, paper_conf_ispass_shangndk23_b200 as M
n, F, N = 2449029, 100, 128
X = torch.randn(n, 104, device="cuda").to(torch.bfloat16)[:, :F]
Wt = torch.randn(N, 104, device="cuda").to(torch.bfloat16)[:, :F]
for _ in range(2):
    B = M.xw_bf16(X, Wt)
torch.cuda.synchronize()
PY
timeout 600 ncu --set full --clock-control none --import-source on -k regex:xw_ -s 1 -c 1 \
  -o /tmp/prof/$TAG -f python /tmp/prof/xw_once.py > gpurun_out/ncu_$TAG.log 2>&1
ncu -i /tmp/prof/$TAG.ncu-rep --page raw --csv > gpurun_out/ncu_${TAG}_raw.csv 2>/dev/null
ncu -i /tmp/prof/$TAG.ncu-rep --page details --csv > gpurun_out/ncu_${TAG}_details.csv 2>/dev/null
