#!/bin/bash
# bench lines for every workload of BASELINE.json configs (+ f4 and round-2 kernels), one box
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
O=gpurun_out/r2l; mkdir -p $O
for wl in f16-64 f16-32 f16-128 f16-16 f64-16 f64-32 f64-64 lr-8 lr-16 lr-32 tf32-64 e4m3-64 e5m2-64 f16upd-64 f64-128x128x128:16384 bf16-256x256x256:8000 bf16-192x192x192:20000 bf16-16x128x16:125000 bf16-16x192x16:125000 bf16-16x64x16:125000; do
  tag=$(echo $wl | tr ':' '_')
  timeout 600 python bench.py --workload $wl --steps 20 --warmup 5 --no-cpu-baseline > $O/$tag.json 2> $O/$tag.err
  python -c "import json; d=json.loads(open('$O/$tag.json').read().strip().splitlines()[-1]); print('$wl', round(d['value'],2), d['roofline']['kernel'], d['roofline']['bound'], round(d['roofline']['frac'],3), d['clocks']['sm_mhz'], d['clocks']['reasons'])" || tail -2 $O/$tag.err
done
for algo in 1d_tmem 3d_tmem; do
  timeout 600 python bench.py --workload f16-64 --algo $algo --steps 20 --warmup 5 --no-cpu-baseline > $O/f16-64_$algo.json 2>/dev/null
  python -c "import json; d=json.loads(open('$O/f16-64_$algo.json').read().strip().splitlines()[-1]); print('f16-64 $algo', round(d['value'],2), d['roofline']['kernel'], round(d['roofline']['frac'],3))"
done
timeout 600 python bench.py --workload bf16-240x256x192:10000 --algo 2d_pair --steps 20 --warmup 5 --no-cpu-baseline --no-e2e > $O/pair_240.json 2>/dev/null
python -c "import json; d=json.loads(open('$O/pair_240.json').read().strip().splitlines()[-1]); print('bf16-240x256x192 2d_pair', round(d['value'],2), d['roofline']['kernel'], round(d['roofline']['frac'],3))"
