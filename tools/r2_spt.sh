#!/bin/bash
# SpMM with A by one TMA box per nonzero block: parity, steady state, throughput
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
timeout 900 python -m pytest tests/test_gpu_spmm.py tests/test_gpu_steady.py -k "spmm" -q --timeout 300 -p no:cacheprovider -x 2>&1 | tail -5
for sh in 256x256x256:8000 256x128x128:20000 224x96x160:20000 128x128x128:40000 64x64x64:65536 256x256x64:16000; do
  IFS=: read shape batch <<< "$sh"
  timeout 300 python tools/vb_bench.py --mode spmm --shape $shape --batch $batch --reps 10
  timeout 300 python tools/vb_bench.py --mode zmorton --shape $shape --batch $batch --reps 10
done
