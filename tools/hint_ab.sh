#!/bin/bash
# L2 eviction hints: none / C stores evict_first / C + A loads evict_first (KAMI_TC_TUNE hint field)
for i in 1 2; do for w in ${WORKLOADS:-lr-16 lr-32 f16-64 f16-128 bf16-256x256x256}; do for h in 0 1 2; do
  echo -n "$w hint=$h: "; KAMI_TC_TUNE=0,0,0,-1,0,0,0,$h timeout 120 python bench.py --workload $w --steps 30 --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],2), round(d['roofline']['frac'],3), d['clocks']['sm_mhz'])"
done; done; done
