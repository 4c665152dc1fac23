#!/bin/bash
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
timeout 900 python -m pytest tests/test_gpu_vbatched.py tests/test_gpu_grid8.py tests/test_gpu_steady.py tests/test_gpu_spmm.py -x -q -m gpu -p no:cacheprovider --timeout 120 2>&1 | tail -12
bash tools/r2_vbmap.sh 2>/dev/null | tail -12
timeout 60 python tools/vb_bench.py --mode ptr --shape 200x128x128 --batch 16384 | cut -c1-150
timeout 60 python tools/vb_bench.py --mode vb --batch 65536 --dtype bf16 --reps 10 | cut -c1-150
