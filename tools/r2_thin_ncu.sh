#!/bin/bash
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
O=gpurun_out/r2t; mkdir -p $O
timeout 1200 python -m pytest tests/test_gpu_f64_general.py tests/test_gpu_ts.py -q --timeout 600 -p no:cacheprovider 2>&1 | tail -4
for spec in "bf16-16x128x16:125000 1d ss128" "bf16-16x192x16:125000 1d ss192" "bf16-16x64x16:125000 1d ss64"; do
  set -- $spec
  timeout 300 ncu --set full --import-source on --clock-control none -k regex:kami_ -s 2 -c 1 -f -o $O/$3 python tools/prof_one.py --workload $1 --algo $2 --iters 3 > /dev/null 2>&1
  ncu -i $O/$3.ncu-rep --page source --csv --print-source sass > $O/src_$3.csv 2>/dev/null
  ncu -i $O/$3.ncu-rep --page details --csv > $O/det_$3.csv 2>/dev/null
  rm -f $O/$3.ncu-rep
done
line() { python -c "import json,sys; d=json.loads(open('$1').read().strip().splitlines()[-1]); print('$2', round(d['value'],2), d['roofline']['kernel'], d['roofline']['bound'], round(d['roofline']['frac'],3), d['clocks']['sm_mhz'])" 2>/dev/null || echo "$2 FAILED"; }
for wl in f64-128x128x128:16384 f64-256x256x256:2048 f64-96x40x72:32768 f64-48x48x48 f16-32; do
  for algo in auto; do
  timeout 300 python bench.py --workload $wl --algo $algo --steps 20 --warmup 5 --no-cpu-baseline --no-e2e > $O/t.json 2>/dev/null
  line $O/t.json "$wl $algo"
  done
done
timeout 300 python bench.py --workload f16-32 --algo 1d_tmem --steps 20 --warmup 5 --no-cpu-baseline --no-e2e > $O/t.json 2>/dev/null; line $O/t.json "f16-32 1d_tmem"
timeout 300 python bench.py --workload f16-64 --algo 1d_tmem --steps 20 --warmup 5 --no-cpu-baseline --no-e2e > $O/t.json 2>/dev/null; line $O/t.json "f16-64 1d_tmem"
timeout 300 python bench.py --workload f16-64 --steps 20 --warmup 5 --no-cpu-baseline --no-e2e > $O/t.json 2>/dev/null; line $O/t.json "f16-64 auto"
