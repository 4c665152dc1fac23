#!/bin/bash
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
timeout 900 python -m pytest tests/test_gpu_spmm.py -q --timeout 300 -p no:cacheprovider -x 2>&1 | tail -5
for sh in 256x256x256:8000 256x128x128:20000 224x96x160:20000 128x128x128:40000; do
  IFS=: read shape batch <<< "$sh"
  timeout 300 python tools/vb_bench.py --mode spmm --shape $shape --batch $batch --reps 10
  timeout 300 python tools/vb_bench.py --mode zmorton --shape $shape --batch $batch --reps 10
done
