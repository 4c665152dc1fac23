#!/bin/bash
# source-level ncu captures of the worst bf16 sweep shapes + FP64 64^3 team-shape A/B
mkdir -p gpurun_out/r1c
for w in bf16-16x192x16:125000 bf16-192x16x16:125000; do
  t=$(echo $w | tr ':x' '__')
  ncu --set full --clock-control none --import-source on -k regex:kami_ -s 2 -c 1 -f \
      -o gpurun_out/r1c/full_$t python tools/prof_one.py --workload $w --iters 3 > gpurun_out/r1c/full_$t.log 2>&1
done
for rep in a b; do for cfg in 0 5 6; do
  KAMI_DMMA_TMA_CFG=$cfg timeout 300 python bench.py --workload f64-64 --steps 30 --warmup 5 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 > gpurun_out/r1c/f64-64_c${cfg}_$rep.json
done; done
KAMI_DMMA_TMA_CFG=5 timeout 300 python -m pytest -q -x tests/test_gpu_parity.py -k "f64" 2>&1 | tail -1
python tools/summarize.py gpurun_out/r1c/*.json
