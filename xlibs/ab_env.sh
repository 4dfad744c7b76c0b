#!/bin/bash
# usage: xlibs/ab_env.sh reps "ENV=..." ... ; back-to-back and cold ms per config ("-" = no env)
reps=$1; shift
for r in $(seq $reps); do for e in "$@"; do for c in 2 3 4 5; do
  if [ "$e" = "-" ]; then ev=""; else ev="$e"; fi
  env $ev timeout 200 python bench.py --config $c --no-all-configs --cpu-seconds 0.2 --steps 30 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('$e C$c', d['ms_per_step'], d['single_layer_cold']['ms_per_step'], d['unfused']['ms_per_step'])"
done; done; done
