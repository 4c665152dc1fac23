#!/bin/bash
# configs[0] (f16 16^3 x 1024): tcgen05 path vs the warp-level HMMA 1D (p = 1), graph timing
mkdir -p gpurun_out/s16
timeout 300 python -m pytest -q -x tests/test_gpu_parity.py -k "16" 2>&1 | tail -2
for rep in a b; do
python bench.py --workload f16-16 --steps 50 --warmup 5 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 > gpurun_out/s16/auto_$rep.json
python bench.py --workload f16-16 --algo 1d --p 1 --steps 50 --warmup 5 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 > gpurun_out/s16/warp1d_$rep.json
for b in 4096 16384 65536; do
python bench.py --workload bf16-16x16x16:$b --steps 50 --warmup 5 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 > gpurun_out/s16/b16_${b}_auto_$rep.json
python bench.py --workload bf16-16x16x16:$b --algo 1d --p 1 --steps 50 --warmup 5 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 > gpurun_out/s16/b16_${b}_warp_$rep.json
done; done
python tools/summarize.py gpurun_out/s16/*.json
