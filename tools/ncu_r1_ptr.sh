#!/bin/bash
# ncu --set full captures of the pointer-array paths (tc16 kPtr f16 64^3, dmma_tma kPtr f64 64^3)
mkdir -p gpurun_out/r1
ncu --set full --clock-control none --import-source on -k regex:kami_ -s 2 -c 1 -f -o gpurun_out/r1/full_ptr-f16-64 \
    python tools/vb_bench.py --mode ptr --dtype f16 --shape 64x64x64 --batch 65536 --reps 1 > gpurun_out/r1/full_ptr-f16-64.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:kami_ -s 2 -c 1 -f -o gpurun_out/r1/full_ptr-f64-64 \
    python tools/vb_bench.py --mode ptr --dtype f64 --shape 64x64x64 --batch 32768 --reps 1 > gpurun_out/r1/full_ptr-f64-64.log 2>&1
