#!/bin/bash
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
O=gpurun_out/r2v; mkdir -p $O
python tools/vb_bench.py --mode vb --batch 40000 --reps 10
python tools/vb_bench.py --mode spmm --shape 256x256x256 --batch 8000 --reps 10
python tools/vb_bench.py --mode spmm --shape 128x128x128 --batch 40000 --reps 10
for spec in "vb 64x64x64 40000 vbmix" "spmm 256x256x256 8000 spmm256"; do
  set -- $spec
  timeout 300 ncu --set full --import-source on --clock-control none -k regex:kami_tc16_vb -s 3 -c 1 -f -o $O/$4 python tools/vb_bench.py --mode $1 --shape $2 --batch $3 --reps 1 > /dev/null 2>&1
  ncu -i $O/$4.ncu-rep --page source --csv --print-source sass > $O/src_$4.csv 2>/dev/null
  ncu -i $O/$4.ncu-rep --page details --csv > $O/det_$4.csv 2>/dev/null
  rm -f $O/$4.ncu-rep
done
