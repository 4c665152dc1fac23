#!/bin/bash
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
timeout 900 python -m pytest tests/test_gpu_vbatched.py tests/test_gpu_parity.py tests/test_gpu_steady.py -k "f64 or dmma or vbatched" -x -q -m gpu -p no:cacheprovider --timeout 200 2>&1 | tail -3
timeout 300 python bench.py --workload f64-128x128x128:16384 --no-cpu-baseline --no-e2e 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('f64-128', round(d['value'],2), round(d['roofline']['frac'],3))"
for o in 16,32,64,128,192,256 16,32,64 64,128; do timeout 120 python tools/vb_bench.py --mode vb --dtype f64 --orders $o --batch 16384 --reps 5 | cut -c1-200 | sed "s/^/orders=$o /"; done
timeout 120 python tools/vb_bench.py --mode vb --dtype f64 --orders 16,32,64 --batch 16384 --reps 5 --nmax 64 | cut -c1-200 | sed "s/^/nmax64 /"
