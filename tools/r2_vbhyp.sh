#!/bin/bash
# is the 16^3 class stage-bound?  3 stages (max_n 256) vs 4 (max_n 16)
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
for nm in 256 16; do
  timeout 60 python tools/vb_bench.py --mode vb --orders 16 --batch 262144 --reps 10 --nmax $nm | sed "s/^/nmax=$nm /"
  timeout 60 python tools/vb_bench.py --mode vb --orders 32 --batch 262144 --reps 10 --nmax $(( nm < 32 ? 32 : nm )) | sed "s/^/o32 nmax=$nm /"
done
timeout 60 python tools/vb_bench.py --mode ptr --shape 200x128x128 --batch 16384
timeout 60 python tools/vb_bench.py --mode ptr --shape 200x128x128 --batch 16384
