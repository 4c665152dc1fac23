#!/bin/bash
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
for r in 1 2 3; do for v in 0 2 1; do
 KAMI_VB_VIEWS=$v timeout 300 python tools/vb_bench.py --mode vb --batch 65536 --dtype f16 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('views=$v', round(d['tflops'],1), round(d['frac_hbm'],3))"
done; done
