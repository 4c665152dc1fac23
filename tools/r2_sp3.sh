#!/bin/bash
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
for sh in 256x256x256:8000 256x128x128:20000 224x96x160:20000 128x128x128:40000 64x64x64:65536; do
  IFS=: read shape batch <<< "$sh"
  timeout 60 python tools/vb_bench.py --mode spmm --shape $shape --batch $batch --reps 10 | cut -c1-150
  timeout 60 python tools/vb_bench.py --mode zmorton --shape $shape --batch $batch --reps 10 | cut -c1-150
done
for o in 16 32 64 128 256; do
  b=$(( 65536 * 64 * 64 / (o * o) )); [ $b -gt 262144 ] && b=262144; [ $b -lt 4000 ] && b=4000
  timeout 60 python tools/vb_bench.py --mode vb --orders $o --batch $b --reps 10 | cut -c1-150 | sed "s/^/order=$o /"
done
