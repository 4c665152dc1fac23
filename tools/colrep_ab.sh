#!/bin/bash
# thin-m A replication / slots on (default) vs off (KAMI_TC_TUNE slot = -1), graph-timed bench lines
for i in 1 2; do for w in ${WORKLOADS:-bf16-16x192x16 bf16-16x256x16 bf16-16x192x32 bf16-16x256x32 bf16-32x192x16 bf16-32x256x16 bf16-32x256x32 bf16-16x256x64 bf16-32x256x128}; do for t in "0,0,0,-1,0,0,0" "0,0,0,-1,0,0,-1"; do
  echo -n "$w $t: "; KAMI_TC_TUNE=$t timeout 120 python bench.py --workload $w --steps 30 --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],2), round(d['roofline']['frac'],3), d['clocks']['sm_mhz'])"
done; done; done
