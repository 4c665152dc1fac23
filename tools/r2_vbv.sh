#!/bin/bash
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
timeout 900 python -m pytest tests/test_gpu_vbatched.py tests/test_gpu_grid8.py tests/test_gpu_steady.py tests/test_gpu_spmm.py -x -q -m gpu 2>&1 | tail -3
for v in 0 1; do for b in 16384 65536; do
 KAMI_VB_VIEWS=$v timeout 300 python tools/vb_bench.py --mode vb --batch $b --dtype f16 | sed "s/^/views=$v /"
done; done
KAMI_VB_VIEWS=1 timeout 300 python tools/vb_bench.py --mode vb --batch 65536 --dtype bf16 | sed "s/^/views=1 /"
for v in 0 1; do KAMI_VB_VIEWS=$v timeout 300 python tools/vb_bench.py --mode ptr --shape 200x128x128 --batch 16384 | sed "s/^/views=$v /"; done
