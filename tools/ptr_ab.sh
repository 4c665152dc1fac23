#!/bin/bash
# pointer-array 16-bit: tc16_vb (default) vs warp-level family (KAMI_PTR16_WARP=1)
for s in 16x16x16 32x32x32 64x64x64 128x128x128; do for w in 0 1; do
  echo -n "ptr $s warp=$w: "; KAMI_PTR16_WARP=$w timeout 120 python tools/vb_bench.py --mode ptr --shape $s --batch 65536 2>&1 | tail -1
done; done
