#!/bin/bash
# usage: tools/quick_bench.sh w1 w2 ...  -> gpurun_out/qb_<w>.json (one bench line each, no e2e/cpu)
for w in "$@"; do
  timeout 300 python bench.py --workload $w --steps 20 --warmup 3 --no-cpu-baseline --no-e2e 2>gpurun_out/qb_$w.err | tail -1 > gpurun_out/qb_$w.json
done
python tools/summarize.py gpurun_out/qb_*.json
