#!/bin/bash
# Usage (on the GPU box): bash tools/profile_round.sh <tag>
# Writes gpurun_out/<tag>_launches.csv (every launch's device time, cold-cache,
# serialised), gpurun_out/<tag>_full_*.ncu-rep (ncu --set full of the main kernels)
# and gpurun_out/<tag>_bench.json (a clean bench line).
set -u
TAG=${1:-r01}
mkdir -p gpurun_out
python bench.py --steps 10 --warmup 3 > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches.csv \
    python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > /dev/null 2>&1
ncu --set full --import-source on --clock-control none -k regex:k_dp_large -s 60 -c 1 \
    -o gpurun_out/${TAG}_full_dp_large python tools/prof_step.py t9 > /dev/null 2>&1
ncu --set full --import-source on --clock-control none -k regex:k_dp_two -s 0 -c 1 \
    -o gpurun_out/${TAG}_full_dp_two python tools/prof_step.py t9 > /dev/null 2>&1
ncu --set full --import-source on --clock-control none -k regex:k_refresh -s 0 -c 2 \
    -o gpurun_out/${TAG}_full_refresh python tools/prof_step.py t9 > /dev/null 2>&1
ncu --set full --import-source on --clock-control none -k regex:k_color -s 0 -c 1 \
    -o gpurun_out/${TAG}_full_color python tools/prof_step.py t9 > /dev/null 2>&1
ls -la gpurun_out/
# per-launch DRAM traffic of the DP kernels and the refresh over one whole step (for roofline.traffic)
ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none --csv \
    -k regex:"k_dp_large|k_dp_group|k_dp_two|k_refresh|k_color" --log-file gpurun_out/${TAG}_traffic.csv \
    python tools/prof_step.py t9 > /dev/null 2>&1
