#!/bin/bash
# usage: xlibs/ab.sh reps lib... ; prints back-to-back and cold ms per config
reps=$1; shift
for r in $(seq $reps); do for lib in "$@"; do for c in 2 3 4 5; do
  if [ $lib = default ]; then unset SR_MHA_LIB; else export SR_MHA_LIB=$PWD/$lib; fi
  timeout 200 python bench.py --config $c --no-all-configs --cpu-seconds 0.2 --steps 30 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('$lib C$c', d['ms_per_step'], d['single_layer_cold']['ms_per_step'])"
done; done; done
