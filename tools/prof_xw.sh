#!/bin/bash
# ncu --set full of the tcgen05 combination kernel (default products shape: n=2.45M,
# F=100, N=128; XW_SHAPE="n F N" overrides)
TAG=${1:-xw}
read XN XF XNN <<< "${XW_SHAPE:-2449029 100 128}"
mkdir -p gpurun_out /tmp/prof
cat > /tmp/prof/xw_once.py <<'PY'
import sys, os
sys.path.insert(0, os.getcwd())
import torch, paper_conf_ispass_shangndk23_b200 as M
n, F, N = [int(v) for v in sys.argv[1:4]]
ld = (F + 7) // 8 * 8
X = torch.randn(n, ld, device="cuda").to(torch.bfloat16)[:, :F]
Wt = torch.randn(N, ld, device="cuda").to(torch.bfloat16)[:, :F]
for _ in range(2):
    B = M.xw_bf16(X, Wt)
torch.cuda.synchronize()
PY
timeout 600 ncu --set full --clock-control none --import-source on -k regex:xw_ -s 1 -c 1 \
  -o /tmp/prof/$TAG -f python /tmp/prof/xw_once.py $XN $XF $XNN > gpurun_out/ncu_$TAG.log 2>&1
ncu -i /tmp/prof/$TAG.ncu-rep --page raw --csv > gpurun_out/ncu_${TAG}_raw.csv 2>/dev/null
ncu -i /tmp/prof/$TAG.ncu-rep --page details --csv > gpurun_out/ncu_${TAG}_details.csv 2>/dev/null
ncu -i /tmp/prof/$TAG.ncu-rep --page source --csv --print-source sass > gpurun_out/ncu_${TAG}_sass.csv 2>/dev/null
