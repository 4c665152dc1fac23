#!/bin/bash
# ncu captures for profiles/r1 (run through gpurun on one B200).
#   launch list of the bench command (per-launch device time, cold, serialised)
#   + one `--set full` launch per workload for traffic / smem / tensor-pipe numbers.
mkdir -p gpurun_out/r1
ncu --metrics gpu__time_duration.sum --clock-control none -k regex:kami_ -c 200 --csv \
    --log-file gpurun_out/r1/launches_bench_f16-64.csv \
    python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/r1/bench_under_ncu.log 2>&1
for w in ${WORKLOADS:-f16-64 tf32-64 e4m3-64 f16upd-64}; do
  ncu --set full --clock-control none --import-source on -k regex:kami_ -s 2 -c 1 -f \
      -o gpurun_out/r1/full_$w python tools/prof_one.py --workload $w --iters 3 > gpurun_out/r1/full_$w.log 2>&1
done
ls -la gpurun_out/r1
