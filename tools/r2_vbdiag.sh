#!/bin/bash
for L in paper_conf_sc_wangdltsl25_b200/libkami.so paper_conf_sc_wangdltsl25_b200/libkami_lb.so; do
 echo "== $L"
 KAMI_LIB=$L timeout 300 python -m pytest tests/test_gpu_vbatched.py -x -q -m gpu -p no:cacheprovider 2>&1 | grep -v "^$" | tail -4
 KAMI_LIB=$L timeout 300 python tools/vb_bench.py --mode vb --orders 16 --batch 262144 --reps 10 2>&1 | tail -1
 KAMI_LIB=$L timeout 300 python tools/vb_bench.py --mode vb --batch 65536 --reps 10 2>&1 | tail -1
 KAMI_LIB=$L timeout 300 python tools/vb_bench.py --mode spmm --shape 64x64x64 --batch 65536 --reps 10 2>&1 | tail -1
done
