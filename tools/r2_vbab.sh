#!/bin/bash
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
timeout 900 python -m pytest tests/test_gpu_vbatched.py tests/test_gpu_spmm.py tests/test_gpu_grid8.py -x -q -m gpu 2>&1 | tail -3
for r in 1 2; do for srt in 0 1; do
 KAMI_VB_SORT=$srt timeout 100 python tools/vb_bench.py --mode vb --batch 65536 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('sort=$srt mix', round(d['tflops'],1), round(d['frac_hbm'],3), d['kernel'])"
for o in 16 64 256; do
 KAMI_VB_SORT=$srt timeout 100 python tools/vb_bench.py --mode vb --batch 65536 --orders $o --nmax $o | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('sort=$srt uniform $o', round(d['tflops'],1), round(d['frac_hbm'],3))"
done; done; done
timeout 100 python tools/vb_bench.py --mode ptr --shape 200x128x128 --batch 16384 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('ptr 200x128x128', round(d['tflops'],1), round(d['frac_hbm'],3))"
KAMI_VB_SORT=1 timeout 300 python tools/trace_vb.py mix 65536 | tail -4
