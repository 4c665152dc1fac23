#!/bin/bash
# per-variant timings for the planner calibration / CA comparison
mkdir -p gpurun_out/vs
for w in f64-16 f64-32 f64-64; do
  for a in 1d 2d 3d nonca; do
    timeout 300 python bench.py --workload $w --algo $a --steps 20 --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 > gpurun_out/vs/${w}_$a.json
  done
done
for w in f16-32 f16-64; do
  P=2; [ $w = f16-64 ] && P=4
  timeout 300 python bench.py --workload $w --algo 1d --p $P --steps 20 --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 > gpurun_out/vs/${w}_w1d.json
  for a in 2d 3d nonca; do
    timeout 300 python bench.py --workload $w --algo $a --steps 20 --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 > gpurun_out/vs/${w}_$a.json
  done
done
python tools/summarize.py gpurun_out/vs/*.json
