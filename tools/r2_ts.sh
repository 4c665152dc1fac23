#!/bin/bash
# round 2: TS-form (A in TMEM) vs SS-form tcgen05, FP64 general sizes; bench lines
set -x
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
mkdir -p gpurun_out/r2
timeout 900 python -m pytest tests/test_gpu_ts.py tests/test_gpu_f64_general.py -q -x --timeout 600 -p no:cacheprovider 2>&1 | tail -30
for wl in f16-64 f16-32 f16-128; do
  for algo in 1d 1d_tmem 3d_tmem; do
    timeout 300 python bench.py --workload $wl --algo $algo --steps 20 --warmup 5 --no-cpu-baseline --no-e2e > gpurun_out/r2/ts_${wl}_${algo}.json 2> gpurun_out/r2/ts_${wl}_${algo}.err
    python -c "import json,sys; d=json.loads(open('gpurun_out/r2/ts_${wl}_${algo}.json').read().strip().splitlines()[-1]); print('$wl $algo', round(d['value'],2), d['roofline']['kernel'], round(d['roofline']['frac'],3), d['clocks']['sm_mhz'])" || tail -3 gpurun_out/r2/ts_${wl}_${algo}.err
  done
done
for wl in f64-128x128x128:16384 f64-256x256x256:2048 f64-96x40x72:32768 f64-64x64x64 f64-48x48x48; do
  timeout 300 python bench.py --workload $wl --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/r2/g.json 2> gpurun_out/r2/g.err
  python -c "import json; d=json.loads(open('gpurun_out/r2/g.json').read().strip().splitlines()[-1]); print('$wl', round(d['value'],2), d['roofline']['kernel'], d['roofline']['bound'], round(d['roofline']['frac'],3), d['roofline'].get('peak'))" || tail -3 gpurun_out/r2/g.err
done
for pct in 100 75 50 25 0; do
  KAMI_F64_RESIDENT_PCT=$pct timeout 300 python bench.py --workload f64-128x128x128:16384 --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/r2/g.json 2>/dev/null
  python -c "import json; d=json.loads(open('gpurun_out/r2/g.json').read().strip().splitlines()[-1]); print('res $pct f64-128', round(d['value'],2))"
done
