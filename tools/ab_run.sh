#!/bin/bash
# GPU tests, then the bench under several kernel selections (A/B).  Usage: ab_run.sh TAG [name=ENV ...]
TAG=${1:-ab}; shift
mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
VARS=("$@")
[ ${#VARS[@]} -eq 0 ] && VARS=("new=" "oldlarge=FGR_LARGE_KERNEL=old")
for kv in "${VARS[@]}"; do
  name=${kv%%=*}; envs=${kv#*=}
  env $envs timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/${TAG}_$name.json 2>gpurun_out/${TAG}_$name.err
  python -c "
import json,sys
try:
    d=json.load(open('gpurun_out/${TAG}_$name.json')); print('$name', 'ms/step %.2f route %.2f' % (d['ms_per_step'], d['route_ms']), {k: round(v, 2) for k, v in d['kernels_ms_per_step'].items()})
except Exception as e: print('$name failed', e, open('gpurun_out/${TAG}_$name.err').read()[-1500:])"
done
