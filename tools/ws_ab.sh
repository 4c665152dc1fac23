#!/bin/bash
# per-warp C stores (KAMI_TC_TUNE ws = 1) vs default, graph-timed bench lines
for i in 1 2; do for w in ${WORKLOADS:-lr-16 lr-32 lr-8 f16-128 bf16-256x256x256 bf16-16x192x16 bf16-16x256x16 bf16-128x256x32 bf16-192x192x192}; do for t in 0 1; do
  echo -n "$w ws=$t: "; KAMI_TC_TUNE=0,0,0,-1,0,0,0,0,0,$t timeout 120 python bench.py --workload $w --steps 30 --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],2), round(d['roofline']['frac'],3), d['clocks']['sm_mhz'], d['roofline']['kernel'])"
done; done; done
