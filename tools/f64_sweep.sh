#!/bin/bash
# FP64 schedule x DMMA shape x L2-prefetch sweep
mkdir -p gpurun_out/f64
for atom in 16 8; do for pf in 1 0; do
  for w in f64-16 f64-32 f64-64; do
    for a in 1d 2d 3d nonca; do
      KAMI_F64_ATOM=$atom KAMI_L2_PREFETCH=$pf timeout 300 python bench.py --workload $w --algo $a --steps 20 --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 > gpurun_out/f64/${w}_${a}_m${atom}_pf${pf}.json
    done
  done
done; done
python tools/summarize.py gpurun_out/f64/*.json
