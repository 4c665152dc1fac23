#!/bin/bash
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
mkdir -p gpurun_out/vbp
for srt in 0 1; do KAMI_VB_SORT=$srt timeout 300 python tools/vb_bench.py --mode vb --batch 65536 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('sort=$srt mix', round(d['tflops'],1), round(d['frac_hbm'],3), d['kernel'])"; done
KAMI_VB_SORT=1 timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv python tools/vb_bench.py --mode vb --batch 65536 --reps 1 2>/dev/null | grep -v "^==" | python -c "
import csv,sys
r=list(csv.reader(sys.stdin))
for x in r[1:]: print(x[4][:50], x[-1])
" | tail -4
KAMI_VB_SORT=1 timeout 600 ncu --set full --import-source on --clock-control none -k regex:kami_tc16_vb -s 3 -c 1 -o gpurun_out/vbp/mix_sorted python tools/vb_bench.py --mode vb --batch 16384 --reps 1 > gpurun_out/vbp/ncu2.log 2>&1
tail -1 gpurun_out/vbp/ncu2.log
