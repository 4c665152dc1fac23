#!/bin/bash
# A/B: old build (libkami_old.so) vs current, and split on/off, graph-timed bench lines
L=paper_conf_sc_wangdltsl25_b200
run() { # lib tune workload
  echo -n "$3 lib=$1 tune=$2: "
  KAMI_LIB=$L/$1 KAMI_TC_TUNE=$2 timeout 120 python bench.py --workload $3 --steps 30 --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],2), round(d['roofline']['frac'],3), d['clocks']['sm_mhz'], d['roofline']['kernel'])"
}
for i in 1 2; do
for w in ${WORKLOADS:-lr-16 lr-32 bf16-256x256x256 bf16-192x192x192 bf16-128x256x32 bf16-16x192x16}; do
  run libkami_old.so 0,0,0,-1,0,0 $w
  run libkami.so 0,0,0,-1,0,0 $w
  run libkami.so 0,0,0,-1,0,1 $w
  run libkami.so 0,0,0,-1,0,-1 $w
done; done
