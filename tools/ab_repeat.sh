#!/bin/bash
# Interleaved repeated A/B of bench.py under env selections.  Usage: ab_repeat.sh TAG REPS name=ENV ...
TAG=$1; REPS=$2; shift 2
mkdir -p gpurun_out
for r in $(seq 1 $REPS); do
  for kv in "$@"; do
    name=${kv%%=*}; envs=${kv#*=}
    env $envs timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/${TAG}_${name}_$r.json 2>/dev/null
    python -c "
import json
d=json.load(open('gpurun_out/${TAG}_${name}_$r.json')); print('$name rep $r ms/step %.3f route %.3f' % (d['ms_per_step'], d['route_ms']))"
  done
done
