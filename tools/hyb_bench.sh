#!/bin/bash
# On the GPU box: L-only and hybrid bench lines plus the per-batch profile.
mkdir -p gpurun_out
python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/${1}_bench_L.json 2>gpurun_out/${1}_bench_L.err
python bench.py --steps 10 --warmup 3 --hybrid 10,500 > gpurun_out/${1}_bench_H.json 2>gpurun_out/${1}_bench_H.err
python tools/batch_profile.py t9 > gpurun_out/${1}_batches.txt 2>&1
