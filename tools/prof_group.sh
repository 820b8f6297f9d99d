#!/bin/bash
# ncu --set full captures of the DP kernels (early wide batch / tail batch), summarised on the box
# (the .ncu-rep files are too large to bring back together).
TAG=${1:-r01e}
mkdir -p gpurun_out /tmp/ncu
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,launch__registers_per_thread,sm__warps_active.avg.pct_of_peak_sustained_active,launch__occupancy_limit_registers,launch__occupancy_limit_shared_mem,launch__grid_size,smsp__issue_active.avg.pct_of_peak_sustained_active,smsp__inst_executed.sum,lts__t_sector_hit_rate.pct
run() {  # name regex skip
  ncu --set full --import-source on --clock-control none -k regex:$2 -s $3 -c 1 -o /tmp/ncu/$1 python tools/prof_step.py t9 > /dev/null 2>&1
  { echo "== $1 ($2, skip $3)"; ncu -i /tmp/ncu/$1.ncu-rep --page raw --csv --metrics $M | tail -n +1;
    python tools/ncu_hot.py /tmp/ncu/$1.ncu-rep 40; python tools/ncu_inst.py /tmp/ncu/$1.ncu-rep 100; } > gpurun_out/${TAG}_$1.txt 2>&1
}
run group_early k_dp_group 7
run group_tail k_dp_group 170
run large_tail k_dp_large 80
cp /tmp/ncu/group_tail.ncu-rep gpurun_out/${TAG}_group_tail.ncu-rep
ls -la gpurun_out
