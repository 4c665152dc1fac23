#!/bin/bash
# round 2 final ncu evidence: the bench command's launch list and one --set full
# capture per changed path (headline, thin-m XT head / pair tiles, FP64 32^3 /
# 64^3, mixed sizes, SpMM), summarised into profiles/r2/ncu_summary.json
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
O=gpurun_out/r2e; mkdir -p $O
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:kami_ -c 200 --csv \
    --log-file $O/launches_bench_f16-64.csv \
    python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > $O/bench_under_ncu.log 2>&1
ARGS=""
WL=(f16-64 bf16-16x128x16:125000 bf16-16x192x16:125000 bf16-16x64x16:125000 f64-32 f64-64)
TG=(f16-64 bf16-16x128x16-xt bf16-16x192x16-xt bf16-16x64x16-xt f64-32 f64-64)
for i in "${!WL[@]}"; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:kami_ -s 2 -c 1 -f \
      -o $O/full_${TG[$i]} python tools/prof_one.py --workload ${WL[$i]} --iters 3 > $O/full_${TG[$i]}.log 2>&1
  ARGS="$ARGS --rep $O/full_${TG[$i]}.ncu-rep:${TG[$i]}"
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:kami_tc16_vb -s 3 -c 1 -f -o $O/full_vbmix \
    python tools/vb_bench.py --mode vb --batch 40000 --reps 1 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:kami_tc16_vb -s 3 -c 1 -f -o $O/full_spmm256 \
    python tools/vb_bench.py --mode spmm --shape 256x256x256 --batch 8000 --reps 1 > /dev/null 2>&1
ARGS="$ARGS --rep $O/full_vbmix.ncu-rep:vb-mix-40000 --rep $O/full_spmm256.ncu-rep:spmm-256-8000"
python tools/ncu_summary.py --round r2 $ARGS --launches $O/launches_bench_f16-64.csv:bench_f16-64_final > /dev/null
cp profiles/r2/ncu_summary.json $O/
for t in bf16-16x128x16-xt vbmix; do
  ncu -i $O/full_$t.ncu-rep --page source --csv --print-source sass > $O/src_$t.csv 2>/dev/null
done
python tools/ncu_stalls.py $O/src_bf16-16x128x16-xt.csv 15
rm -f $O/*.ncu-rep
ls $O
