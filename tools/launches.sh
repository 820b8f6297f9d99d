#!/bin/bash
# ncu launch lists (serialised, cold-cache per-kernel times) of one bench step, per kernel selection
TAG=${1:-r01}; shift
mkdir -p gpurun_out
for kv in "$@"; do
  name=${kv%%=*}; envs=${kv#*=}
  env $envs ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_${name}_launches.csv \
      python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > /dev/null 2>&1
  python tools/launch_batches.py gpurun_out/${TAG}_${name}_launches.csv | head -3
done
