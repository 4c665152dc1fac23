#!/bin/bash
# small classes: TMA views (default) vs the cp.async copy path (KAMI_VB_VIEWS=2: views only for multiples of 64)
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
for v in 1 2; do
  for o in 16 32 16,32; do
    KAMI_VB_VIEWS=$v timeout 60 python tools/vb_bench.py --mode vb --orders $o --batch 262144 --reps 10 | sed "s/^/views=$v o=$o /"
  done
  KAMI_VB_VIEWS=$v timeout 60 python tools/vb_bench.py --mode vb --batch 65536 --reps 10 | sed "s/^/views=$v mix /"
done
