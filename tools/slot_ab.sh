#!/bin/bash
# thin-m 32-lane slots on / off (KAMI_TC_TUNE slot = -1), graph-timed bench lines
for i in 1 2; do for w in ${WORKLOADS:-bf16-16x64x16 bf16-16x128x16 bf16-16x128x32 bf16-16x64x32 bf16-16x64x64 bf16-16x128x64 bf16-16x64x256}; do for t in "0,0,0,-1,0,0,0" "0,0,0,-1,0,0,-1"; do
  echo -n "$w $t: "; KAMI_TC_TUNE=$t timeout 120 python bench.py --workload $w --steps 30 --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],2), round(d['roofline']['frac'],3), d['clocks']['sm_mhz'])"
done; done; done
