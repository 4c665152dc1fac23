#!/bin/bash
# Every bench workload once (graph timing, clocks sampled), one JSON line each, plus the default
# line (with e2e and cpu_baseline), the reference arm, and the ncu launch list of the default command.
OUT=${OUT:-gpurun_out/r1}
mkdir -p $OUT
python bench.py --steps 50 --warmup 5 > $OUT/bench_default.json 2> $OUT/bench_default.err
python bench.py --impl reference --steps 3 --warmup 3 > $OUT/bench_reference.json 2>&1
for w in ${WORKLOADS:-f16-16 f16-32 f16-128 f64-16 f64-32 f64-64 lr-8 lr-16 lr-32 tf32-64 e4m3-64 e5m2-64 f16upd-64}; do
  python bench.py --workload $w --steps 50 --warmup 5 --no-cpu-baseline --no-e2e 2>&1 | tail -1 > $OUT/bench_$w.json
done
ncu --metrics gpu__time_duration.sum --clock-control none -k regex:kami_ -c 200 --csv \
    --log-file $OUT/launches_bench_f16-64.csv \
    python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/bench_under_ncu.log 2>&1
python tools/summarize.py $OUT/bench_*.json
