#!/bin/bash
# Same-box A/B of library builds: ./ab.sh "lib1 lib2 ..." "wl:K wl:K ..."
LIBS=$1; CFGS=$2
for c in $CFGS; do IFS=: read wl k dt <<< "$c"; dt=${dt:-f32}
  for l in $LIBS; do
    r=$(env $ENVS MPS_LIB=$PWD/paper_conf_ispass_shangndk23_b200/$l python tools/microbench.py $wl $k $dt 2>&1 | tail -1)
    echo "$wl:$k:$dt $l $r" | cut -c1-150
  done
done
