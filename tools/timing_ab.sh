#!/bin/bash
# same-box A/B of the three timing modes, interleaved
mkdir -p gpurun_out/tm
for rep in a b; do for w in ${WL:-f16-64 lr-16 f16-32 f64-64}; do for t in events b2b graph; do
  timeout 300 python bench.py --workload $w --timing $t --steps 50 --warmup 5 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 > gpurun_out/tm/${w}_${t}_$rep.json
done; done; done
python tools/summarize.py gpurun_out/tm/*.json
