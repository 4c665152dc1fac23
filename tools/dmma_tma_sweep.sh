#!/bin/bash
mkdir -p gpurun_out/dt
for cfg in 0 1 2; do for w in f64-16 f64-32 f64-64; do
  KAMI_DMMA_TMA_CFG=$cfg timeout 300 python bench.py --workload $w --algo 1d_tma --steps 20 --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 > gpurun_out/dt/${w}_c$cfg.json
done; done
python tools/summarize.py gpurun_out/dt/*.json
