#!/bin/bash
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
mkdir -p gpurun_out/r2p
timeout 900 python -m pytest tests/test_gpu_pair.py -q --timeout 300 -p no:cacheprovider 2>&1 | tail -5
line() { python -c "import json,sys; d=json.loads(open('$1').read().strip().splitlines()[-1]); print('$2', round(d['value'],2), d['roofline']['kernel'], round(d['roofline']['frac'],3), d['clocks']['sm_mhz'])" 2>/dev/null || echo "$2 FAILED"; }
for wl in bf16-256x256x256:8000 bf16-256x256x128:16000 bf16-256x256x64:30000 bf16-224x224x224:10000 bf16-256x128x256:16000 bf16-240x256x192:10000 bf16-208x208x208:12000 lr-8 lr-16 lr-32 bf16-256x64x64:60000 bf16-256x256x16:60000; do
  for algo in auto 2d_pair; do
    timeout 300 python bench.py --workload $wl --algo $algo --steps 20 --warmup 5 --no-cpu-baseline --no-e2e > gpurun_out/r2p/t.json 2>gpurun_out/r2p/t.err
    line gpurun_out/r2p/t.json "$wl $algo"
  done
done
