#!/bin/bash
# pointer-array 16-bit: TMA over address-space views (tma) vs LDG-fed tc16_vb (vb) vs warp-level HMMA (warp)
for d in ${DTYPES:-f16}; do for s in ${SHAPES:-16x16x16 32x32x32 64x64x64 128x128x128 256x256x16 256x256x256}; do for r in tma vb warp; do
  echo -n "ptr $d $s route=$r: "; KAMI_PTR_ROUTE=$r timeout 120 python tools/vb_bench.py --mode ptr --dtype $d --shape $s --batch ${BATCH:-65536} 2>&1 | tail -1
done; done; done
