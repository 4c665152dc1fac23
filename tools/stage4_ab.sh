#!/bin/bash
# small-stage shapes: planner default vs a 4-stage cap (KAMI_TC_TUNE stages=4), graph-timed bench lines
for i in 1 2; do for w in ${WORKLOADS:-e5m2-64 lr-8 lr-16 bf16-16x64x16 bf16-32x32x16 bf16-64x64x16 bf16-16x16x64 bf16-32x64x32 bf16-64x32x16 f16-16 f16upd-64}; do for st in 0 4; do
  echo -n "$w stages=$st: "
  KAMI_TC_TUNE=$st,0,0,-1,0,0 timeout 120 python bench.py --workload $w --steps 30 --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],2), round(d['roofline']['frac'],3), d['clocks']['sm_mhz'], d['roofline']['kernel'])"
done; done; done
