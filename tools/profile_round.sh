#!/bin/bash
# Usage (on the GPU box): bash tools/profile_round.sh <tag>
# gpurun_out/<tag>_bench.json      a clean bench line (default run, with the CPU oracle baseline)
# gpurun_out/<tag>_launches.csv    every launch's device time (ncu, cold-cache, serialised)
# gpurun_out/<tag>_summary.md      ncu --set full of the main kernels + per-launch DRAM traffic, summarised
# gpurun_out/<tag>_traffic.json    per-launch DRAM bytes per kernel class (bench.py roofline.traffic)
set -u
TAG=${1:-r01}
mkdir -p gpurun_out /tmp/ncu_$TAG
python bench.py --steps 10 --warmup 3 > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches.csv \
    python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > /dev/null 2>&1
cp gpurun_out/${TAG}_launches.csv /tmp/ncu_$TAG/
full() {  # name regex skip
  ncu --set full --import-source on --clock-control none -k regex:$2 -s $3 -c 1 \
      -o /tmp/ncu_$TAG/${TAG}_full_$1 python tools/prof_step.py t9 > /dev/null 2>&1
}
full walk_early 'k_dp_walk' 5
full walk_tail 'k_dp_walk' 150
full two 'k_dp_two' 3
full flow 'k_dp_flow' 40
full large 'k_dp_large' 60
full refresh 'k_refresh' 2
ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none --csv \
    -k regex:"k_dp_large|k_dp_walk|k_dp_flow|k_dp_two|k_refresh|k_color" --log-file /tmp/ncu_$TAG/${TAG}_traffic.csv \
    python tools/prof_step.py t9 > /dev/null 2>&1
python tools/summarize_profiles.py $TAG /tmp/ncu_$TAG
cp profiles/${TAG}_summary.md profiles/${TAG}_traffic.json gpurun_out/ 2>/dev/null
for r in walk_tail flow; do
  python tools/ncu_lines.py /tmp/ncu_$TAG/${TAG}_full_$r.ncu-rep 25 > gpurun_out/${TAG}_lines_$r.txt 2>&1
done
ls -la gpurun_out
