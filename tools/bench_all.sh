#!/bin/bash
# Every bench workload once (sustained timing, clocks sampled), one JSON line each.
mkdir -p gpurun_out/r1
python bench.py --steps 30 --warmup 5 > gpurun_out/r1/bench_default.json 2> gpurun_out/r1/bench_default.err
python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/r1/bench_reference.json 2>&1
for w in ${WORKLOADS:-f16-16 f16-32 f16-128 f64-16 f64-32 f64-64 lr-8 lr-16 lr-32 tf32-64 e4m3-64 e5m2-64 f16upd-64}; do
  python bench.py --workload $w --steps 30 --warmup 5 --no-cpu-baseline --no-e2e 2>&1 | tail -1 > gpurun_out/r1/bench_$w.json
done
