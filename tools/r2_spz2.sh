#!/bin/bash
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
timeout 900 python -m pytest tests/test_gpu_spmm.py -q --timeout 120 -p no:cacheprovider -x 2>&1 | tail -2
for sh in 256x256x256:8000 256x128x128:20000 224x96x160:20000 128x128x128:40000 64x64x64:65536; do
  IFS=: read shape batch <<< "$sh"
  timeout 60 python tools/vb_bench.py --mode spmm --shape $shape --batch $batch --reps 10
  for al in 1d; do timeout 60 python tools/vb_bench.py --mode zmorton --shape $shape --batch $batch --reps 10 --algo $al 2>&1 | tail -1; done
done
