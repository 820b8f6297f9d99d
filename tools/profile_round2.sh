#!/bin/bash
# Round-2 profile set (on the GPU box): bash tools/profile_round2.sh <tag>
#   <tag>_bench.json        clean bench line (profiler off for the headline, CPU oracle baseline)
#   <tag>_launches.csv      ncu launch list of one bench step (cold-cache, serialised)
#   <tag>_full_*.ncu-rep    ncu --set full of the main kernels (tree: a tail launch of the 384-thread variant;
#                           walk/two captured twice: cold cache and --cache-control none = warm L2)
#   <tag>_traffic.csv/json  per-launch DRAM bytes per kernel class
set -u
TAG=${1:-r02}
mkdir -p gpurun_out /tmp/ncu_$TAG
python bench.py --steps 10 --warmup 3 > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches.csv \
    python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > /dev/null 2>&1
cp gpurun_out/${TAG}_launches.csv /tmp/ncu_$TAG/
python tools/launch_batches.py gpurun_out/${TAG}_launches.csv > gpurun_out/${TAG}_batches.txt 2>&1
full() {  # name regex skip [extra ncu args]
  ncu --set full --import-source on --clock-control none --kernel-name-base mangled -k regex:"$2" -s $3 -c 1 ${4:-} \
      -o /tmp/ncu_$TAG/${TAG}_full_$1 python tools/prof_step.py t9 > /dev/null 2>&1
}
full tree384 'k_dp_treeILi9ELi384' 30
full tree256 'k_dp_treeILi9ELi256' 40
full refresh 'k_refresh' 2
full walk_tail 'k_dp_walk' 150
full walk_warm 'k_dp_walk' 150 '--cache-control none'
full two 'k_dp_two' 3
full two_warm 'k_dp_two' 3 '--cache-control none'
ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none --csv \
    -k regex:"k_dp_tree|k_dp_walk|k_dp_two|k_refresh|k_color|k_commit_nets" --log-file /tmp/ncu_$TAG/${TAG}_traffic.csv \
    python tools/prof_step.py t9 > /dev/null 2>&1
cp /tmp/ncu_$TAG/${TAG}_traffic.csv gpurun_out/
python tools/summarize_profiles.py $TAG /tmp/ncu_$TAG > /dev/null 2>&1
cp profiles/${TAG}_summary.md profiles/${TAG}_traffic.json gpurun_out/ 2>/dev/null
cp /tmp/ncu_$TAG/${TAG}_full_tree384.ncu-rep /tmp/ncu_$TAG/${TAG}_full_refresh.ncu-rep gpurun_out/ 2>/dev/null
for r in tree384 walk_tail; do
  python tools/ncu_lines.py /tmp/ncu_$TAG/${TAG}_full_$r.ncu-rep 30 > gpurun_out/${TAG}_lines_$r.txt 2>&1
done
ls -la gpurun_out | tail -30
