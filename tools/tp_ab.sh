#!/bin/bash
# tail packing for 128 < m <= 192 on (default) / off (KAMI_TC_TUNE tp = -1), graph-timed bench lines
for i in 1 2; do for w in ${WORKLOADS:-bf16-192x16x16 bf16-192x32x16 bf16-192x64x16 bf16-192x128x16 bf16-192x16x128 bf16-192x64x64 bf16-192x128x128 bf16-192x128x256 bf16-160x64x32}; do for t in 0 -1; do
  echo -n "$w tp=$t: "; KAMI_TC_TUNE=0,0,0,-1,0,0,0,0,$t timeout 120 python bench.py --workload $w --steps 30 --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],2), round(d['roofline']['frac'],3), d['clocks']['sm_mhz'], d['roofline']['kernel'])"
done; done; done
