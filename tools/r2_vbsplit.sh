#!/bin/bash
# mixed-size batch: per-order throughput of the sorted vbatched kernel (all
# entries one order, through the variable-size API) and the full mix; ncu stall
# profile of the mix
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
for o in 16 32 64 128 192 256; do
  b=$(( 65536 * 64 * 64 / (o * o) )); [ $b -gt 262144 ] && b=262144; [ $b -lt 4000 ] && b=4000
  timeout 300 python tools/vb_bench.py --mode vb --orders $o --batch $b --reps 10 | sed "s/^/order=$o /"
done
timeout 300 python tools/vb_bench.py --mode vb --orders 64,128,192,256 --batch 40000 --reps 10 | sed "s/^/big /"
timeout 300 python tools/vb_bench.py --mode vb --orders 16,32 --batch 200000 --reps 10 | sed "s/^/small /"
timeout 300 python tools/vb_bench.py --mode vb --batch 65536 --reps 10 | sed "s/^/mix /"
O=gpurun_out/r2v; mkdir -p $O
timeout 300 ncu --set full --import-source on --clock-control none -k regex:kami_tc16_vb -s 3 -c 1 -f -o $O/vbmix python tools/vb_bench.py --mode vb --batch 40000 --reps 1 > /dev/null 2>&1
ncu -i $O/vbmix.ncu-rep --page source --csv --print-source sass > $O/src_vbmix.csv 2>/dev/null
ncu -i $O/vbmix.ncu-rep --page details --csv > $O/det_vbmix.csv 2>/dev/null
rm -f $O/vbmix.ncu-rep
python tools/ncu_stalls.py $O/src_vbmix.csv 25
for spec in "spmm 64x64x64 65536 sp64" "spmm 256x256x256 8000 sp256"; do
  set -- $spec
  timeout 300 ncu --set full --import-source on --clock-control none -k regex:kami_tc16_vb -s 3 -c 1 -f -o $O/$4 python tools/vb_bench.py --mode $1 --shape $2 --batch $3 --reps 1 > /dev/null 2>&1
  ncu -i $O/$4.ncu-rep --page source --csv --print-source sass > $O/src_$4.csv 2>/dev/null
  ncu -i $O/$4.ncu-rep --page details --csv > $O/det_$4.csv 2>/dev/null
  rm -f $O/$4.ncu-rep
  python tools/ncu_stalls.py $O/src_$4.csv 25
done
