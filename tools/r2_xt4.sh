#!/bin/bash
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
timeout 900 python -m pytest tests/test_gpu_xt.py -x -q -m gpu -p no:cacheprovider --timeout 120 2>&1 | tail -2
timeout 600 python tools/xt_ab.py
for s in "" "--sortalloc"; do timeout 60 python tools/vb_bench.py --mode vb --batch 65536 --reps 10 $s | cut -c1-170 | sed "s/^/mix$s /"; done
