#!/bin/bash
# stage-count sweep (KAMI_TC_TUNE stages) for the large-tile bf16 shapes, graph-timed bench lines
for i in 1 2; do for w in ${WORKLOADS:-bf16-192x192x192 bf16-256x256x256 bf16-192x256x192}; do for st in ${STAGES:-0 2 3 4}; do
  echo -n "$w stages=$st: "
  KAMI_TC_TUNE=$st,0,0,-1,0,0 timeout 120 python bench.py --workload $w --steps 30 --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],2), round(d['roofline']['frac'],3), d['clocks']['sm_mhz'])"
done; done; done
