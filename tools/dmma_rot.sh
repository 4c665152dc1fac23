#!/bin/bash
# A/B of the FP64 TMA-broadcast kernel: cfg 0 (B loaded at entry start) vs cfg 3 (B rotated half an entry ahead)
mkdir -p gpurun_out/dt
KAMI_DMMA_TMA_CFG=3 timeout 300 python -m pytest -q -x tests/test_gpu_parity.py -k "f64" 2>&1 | tail -2
for rep in a b; do for cfg in 0 3; do for w in f64-16 f64-32 f64-64; do
  KAMI_DMMA_TMA_CFG=$cfg timeout 300 python bench.py --workload $w --algo 1d_tma --steps 30 --warmup 5 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 > gpurun_out/dt/${w}_c${cfg}_$rep.json
done; done; done
python tools/summarize.py gpurun_out/dt/*_c[03]_*.json
