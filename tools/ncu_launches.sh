#!/bin/bash
# Launch list (per-launch device time, cold, serialised) of the default bench
# command, restricted to this repo's kernels.
mkdir -p gpurun_out/r1
ncu --metrics gpu__time_duration.sum --clock-control none -k regex:kami_ -c 200 --csv \
    --log-file gpurun_out/r1/launches_bench_${1:-f16-64}.csv \
    python bench.py --workload ${1:-f16-64} --steps 5 --warmup 3 --no-cpu-baseline --no-e2e \
    > gpurun_out/r1/bench_under_ncu_${1:-f16-64}.log 2>&1
