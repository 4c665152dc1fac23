#!/bin/bash
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
timeout 900 python -m pytest tests/test_gpu_spmm.py tests/test_gpu_steady.py tests/test_gpu_vbatched.py -x -q -m gpu -p no:cacheprovider --timeout 120 2>&1 | tail -12
for sh in 256x256x256:8000 256x128x128:20000 224x96x160:20000 128x128x128:40000 64x64x64:65536; do
  IFS=: read shape batch <<< "$sh"
  timeout 60 python tools/vb_bench.py --mode spmm --shape $shape --batch $batch --reps 10 | cut -c1-150
  timeout 60 python tools/vb_bench.py --mode zmorton --shape $shape --batch $batch --reps 10 | cut -c1-150
done
timeout 60 python tools/vb_bench.py --mode vb --batch 65536 --reps 10 | cut -c1-150
