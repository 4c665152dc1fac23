#!/bin/bash
# vbatched / SpMM quick check: parity of the tc16_vb paths, per-order and mix throughput
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
timeout 600 python -m pytest tests/test_gpu_vbatched.py tests/test_gpu_grid8.py tests/test_gpu_steady.py tests/test_gpu_spmm.py -x -q -m gpu -p no:cacheprovider --timeout 120 2>&1 | tail -3
for o in 16 32 64 128 256; do
  b=$(( 65536 * 64 * 64 / (o * o) )); [ $b -gt 262144 ] && b=262144; [ $b -lt 4000 ] && b=4000
  timeout 60 python tools/vb_bench.py --mode vb --orders $o --batch $b --reps 10 | sed "s/^/order=$o /"
done
timeout 60 python tools/vb_bench.py --mode vb --orders 16,32 --batch 200000 --reps 10 | sed "s/^/small /"
timeout 60 python tools/vb_bench.py --mode vb --batch 65536 --reps 10 | sed "s/^/mix /"
timeout 60 python tools/vb_bench.py --mode vb --batch 65536 --reps 10 --dtype bf16 | sed "s/^/mix /"
for sh in 256x256x256:8000 128x128x128:40000 64x64x64:65536 224x96x160:20000; do
  IFS=: read shape batch <<< "$sh"
  timeout 60 python tools/vb_bench.py --mode spmm --shape $shape --batch $batch --reps 10
done
timeout 60 python tools/vb_bench.py --mode ptr --shape 200x128x128 --batch 16384
