#!/bin/bash
# timing-mode A/B: CUDA-graph replay (default) vs back-to-back launches
mkdir -p gpurun_out/ga
for w in ${WL:-f16-16 f16-32 f16-64 f16-128 f64-16 f64-32 f64-64 lr-8 lr-16 lr-32}; do
  timeout 300 python bench.py --workload $w --steps 50 --warmup 5 --no-cpu-baseline --no-e2e 2>gpurun_out/ga/$w.err | tail -1 > gpurun_out/ga/${w}_graph.json
done
for w in f16-16 f16-32 f16-64; do
  timeout 300 python bench.py --workload $w --steps 50 --warmup 5 --no-cpu-baseline --no-e2e --no-graph 2>/dev/null | tail -1 > gpurun_out/ga/${w}_nograph.json
done
python tools/summarize.py gpurun_out/ga/*.json
