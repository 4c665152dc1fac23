#!/bin/bash
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
O=gpurun_out/r2k; mkdir -p $O
timeout 300 ncu --set full --import-source on --clock-control none -k regex:kami_tc16_vb -s 3 -c 1 -f -o $O/vbk python tools/vb_bench.py --mode vb ${VBARGS:---korders 16,32} --batch 40000 --reps 1 > /dev/null 2>&1
ncu -i $O/vbk.ncu-rep --page source --csv --print-source sass > $O/src_vbk.csv 2>/dev/null
ncu -i $O/vbk.ncu-rep --page details --csv > $O/det_vbk.csv 2>/dev/null
rm -f $O/vbk.ncu-rep
python tools/ncu_stalls.py $O/src_vbk.csv 25
