#!/bin/bash
# Quick GPU loop for the large-net kernel: parity on the large-net designs, t9 bench, per-phase timing.
TAG=${1:-r02x}
mkdir -p gpurun_out
timeout 600 python tools/hld_check.py bignets,chains,t5,huge,t1 > gpurun_out/${TAG}_check.txt 2>&1
echo "check rc=$?" >> gpurun_out/${TAG}_check.txt
grep -c OK gpurun_out/${TAG}_check.txt; grep -v OK gpurun_out/${TAG}_check.txt | head -8
timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err
python -c "import json;d=json.load(open('gpurun_out/${TAG}_bench.json'));print('bench', d['ms_per_step'], d['route_ms'], d['plan_ms'], d.get('kernels_ms_per_step'))"
FGR_LIB_PATH=build_t/libfastgr_tt.so timeout 300 python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-e2e > gpurun_out/${TAG}_timing.txt 2>&1
grep "TREE" gpurun_out/${TAG}_timing.txt | sort -t= -k2 -n -r | head -4
grep "ROOT" gpurun_out/${TAG}_timing.txt | head -4
