#!/bin/bash
# order-16 vbatched: per-kernel launch times (pre-pass + main) and one full ncu capture
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
O=gpurun_out/r2v16; mkdir -p $O
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches.csv python tools/vb_bench.py --mode vb --orders 16 --batch 262144 --reps 1 > /dev/null 2>&1
python - <<'PY'
import csv
rows=[r for r in csv.reader(open('gpurun_out/r2v16/launches.csv')) if len(r)>10]
hdr=rows[0]; ik=hdr.index('Kernel Name'); iv=hdr.index('Metric Value'); iu=hdr.index('Metric Unit')
for r in rows[1:][-8:]: print(r[ik][:60], r[iv], r[iu])
PY
timeout 300 ncu --set full --import-source on --clock-control none -k regex:kami_tc16_vb -s 3 -c 1 -f -o $O/vb16 python tools/vb_bench.py --mode vb --orders 16 --batch 262144 --reps 1 > /dev/null 2>&1
ncu -i $O/vb16.ncu-rep --page source --csv --print-source sass > $O/src_vb16.csv 2>/dev/null
ncu -i $O/vb16.ncu-rep --page details --csv > $O/det_vb16.csv 2>/dev/null
rm -f $O/vb16.ncu-rep
python tools/ncu_stalls.py $O/src_vb16.csv 30
