#!/bin/bash
# Same-box A/B of library builds / env settings through bench.py (segment_ms, ms_per_step).
# Usage: VARIANTS="libold.so: libmpspmm.so:MPS_DYN=0 libmpspmm.so:MPS_DYN=1" tools/ab_bench.sh "wl:K ..."
for c in $1; do IFS=: read wl k dt <<< "$c"; dt=${dt:-f32}
  for v in $VARIANTS; do lib=${v%%:*}; envs=${v#*:}
    r=$(env $envs MPS_LIB=$PWD/paper_conf_ispass_shangndk23_b200/$lib timeout 600 python bench.py --workload $wl --K $k --dtype $dt --steps ${STEPS:-20} --warmup 5 --e2e-steps 0 --no-cpu-baseline --no-cusparse --no-l2-probe 2>/dev/null | tail -1 | python -c "import json,sys; l=json.loads(sys.stdin.read()); print('%.4f %.4f' % (l['ms_per_step'], l['segment_ms']))")
    echo "$wl:$k:$dt $v $r"
  done
done
