#!/bin/bash
# items_per_part sweep through bench.py (ms_per_step, segment_ms, P) on one box.
for c in $1; do IFS=: read wl k <<< "$c"
  for cost in 0 ${COSTS:-256 512 1024 2048 4096 8192}; do
    r=$(timeout 600 python bench.py --workload $wl --K $k --items-per-part $cost --steps ${STEPS:-15} --warmup 4 --e2e-steps 0 --no-cpu-baseline --no-cusparse --no-l2-probe 2>/dev/null | tail -1 | python -c "import json,sys; l=json.loads(sys.stdin.read()); print('%.4f %.4f P=%d L=%d' % (l['ms_per_step'], l['segment_ms'], l['config']['num_parts'], l['config']['items_per_part']))")
    echo "$wl:$k cost=$cost $r"
  done
done
