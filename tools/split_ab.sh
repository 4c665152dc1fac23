#!/bin/bash
# per-atom C stores (split instantiation, default where it applies) vs one store per unit
# (KAMI_TC_TUNE split = -1); same box, interleaved
mkdir -p gpurun_out/sp4
timeout 600 python -m pytest -q -x tests/test_gpu_parity.py -k tc16 2>&1 | tail -1
for rep in a b; do for w in ${WL:-lr-8 lr-16 lr-32 f16-128 bf16-192x192x192 bf16-256x256x256 bf16-16x192x16 bf16-32x256x64 bf16-128x256x32}; do
  t=$(echo $w | tr ':x' '__')
  for md in 0 -1; do
  KAMI_TC_TUNE=0,0,0,-1,0,$md timeout 300 python bench.py --workload $w --steps 30 --warmup 5 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 > gpurun_out/sp4/${t}_m${md}_$rep.json
  done
done; done
python tools/summarize.py gpurun_out/sp4/*.json
