#!/bin/bash
# ncu source-level stall profile of the vbatched kernel: order-16 batch, the mix, SpMM 64^3
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
O=gpurun_out/r2v2; mkdir -p $O
for spec in "vb 16 262144 vb16" "vb 16,32,64,128,192,256 40000 vbmix" "spmm 64 65536 sp64"; do
  set -- $spec
  if [ $1 = vb ]; then args="--mode vb --orders $2 --batch $3"; else args="--mode spmm --shape 64x64x64 --batch $3"; fi
  timeout 300 ncu --set full --import-source on --clock-control none -k regex:kami_tc16_vb -s 3 -c 1 -f -o $O/$4 python tools/vb_bench.py $args --reps 1 > /dev/null 2>&1
  ncu -i $O/$4.ncu-rep --page source --csv --print-source sass > $O/src_$4.csv 2>/dev/null
  ncu -i $O/$4.ncu-rep --page details --csv > $O/det_$4.csv 2>/dev/null
  rm -f $O/$4.ncu-rep
  echo "== $4"; python tools/ncu_stalls.py $O/src_$4.csv 12
done
