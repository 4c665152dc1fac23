#!/bin/bash
# round 2 ncu evidence (one GPU): the bench command's launch list, one
# `--set full` capture per bench workload / TS variant / worst sweep points,
# summarised on the box (reports are too big to ship back), plus the SASS
# source page of the f16 64^3 kernels (per-instruction shared wavefronts).
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
O=gpurun_out/r2/ncu
mkdir -p $O
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:kami_ -c 200 --csv \
    --log-file $O/launches_bench_f16-64.csv \
    python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > $O/bench_under_ncu.log 2>&1
WL=(f16-64 f16-64 f16-64 f16-32 f16-128 lr-16 lr-8 f64-64 f64-32 f64-16 bf16-16x128x16:125000 bf16-16x192x16:125000 bf16-192x16x16:125000 f64-128x128x128:8192 f16-16 tf32-64 e4m3-64)
AL=(auto 1d_tmem 3d_tmem auto auto auto auto auto auto auto auto auto auto auto auto auto auto)
TG=(f16-64 f16-64-ts1d f16-64-ts3d f16-32 f16-128 lr-16 lr-8 f64-64 f64-32 f64-16 bf16-16x128x16 bf16-16x192x16 bf16-192x16x16 f64-128 f16-16 tf32-64 e4m3-64)
ARGS=""
for i in "${!WL[@]}"; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:kami_ -s 2 -c 1 -f \
      -o $O/full_${TG[$i]} python tools/prof_one.py --workload ${WL[$i]} --algo ${AL[$i]} --iters 3 > $O/full_${TG[$i]}.log 2>&1
  ARGS="$ARGS --rep $O/full_${TG[$i]}.ncu-rep:${TG[$i]}"
done
python tools/ncu_summary.py --round r2 $ARGS --launches $O/launches_bench_f16-64.csv:bench_f16-64 > /dev/null
cp profiles/r2/ncu_summary.json $O/
for t in f16-64 f16-64-ts1d; do
  ncu -i $O/full_$t.ncu-rep --page source --csv --print-source sass > $O/src_$t.csv 2>/dev/null
  ncu -i $O/full_$t.ncu-rep --page details --csv > $O/details_$t.csv 2>/dev/null
done
ls -la $O | head -50
rm -f $O/*.ncu-rep
