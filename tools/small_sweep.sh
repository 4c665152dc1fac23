#!/bin/bash
# f16 32^3 overhead study: batch scaling, unit size and ring depth; f16 16^3 x 1024 per-algo latency
mkdir -p gpurun_out/ss
for b in 16384 65536 262144 1048576; do
  python bench.py --workload bf16-32x32x32:$b --steps 20 --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 > gpurun_out/ss/b32_$b.json
done
python tools/summarize.py gpurun_out/ss/b32_*.json
python tools/tc_tune.py --workload f16-32 --tunes "0,0,0,-1,0" "0,0,0,-1,1" "0,0,0,-1,4" "2,0,0,-1,0" "4,0,0,-1,0" "6,0,0,-1,0" "0,1,0,-1,0" "0,0,0,0,0" "0,0,0,2,0"
for a in auto 1d 2d nonca; do
  python bench.py --workload f16-16 --algo $a --steps 50 --warmup 5 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 > gpurun_out/ss/f16-16_$a.json
done
python tools/summarize.py gpurun_out/ss/f16-16_*.json
