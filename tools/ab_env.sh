#!/bin/bash
# Same-box A/B over env settings: ./ab_env.sh LIB "ENV1;ENV2;..." "wl:K ..."
LIB=$1; IFS=';' read -ra ENVL <<< "$2"; CFGS=$3
for c in $CFGS; do wl=${c%%:*}; k=${c##*:}
  for e in "${ENVL[@]}"; do
    r=$(env $e MPS_LIB=$PWD/paper_conf_ispass_shangndk23_b200/$LIB python tools/microbench.py $wl $k 2>&1 | tail -1)
    echo "$wl:$k $LIB [$e] $r" | sed 's/"after_zero.*//' | cut -c1-150
  done
done
