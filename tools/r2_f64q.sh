#!/bin/bash
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_steady.py tests/test_gpu_vbatched.py -k "f64 or dmma or fp64" -x -q -m gpu -p no:cacheprovider --timeout 120 2>&1 | tail -2
for w in f64-16 f64-32 f64-64; do
  timeout 300 python bench.py --workload $w --no-cpu-baseline --no-e2e 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$w', round(d['value'],2), round(d['roofline']['frac'],3), d['clocks']['sm_mhz'])"
done
for pf in 0 1; do KAMI_VB_PREFETCH=$pf timeout 60 python tools/vb_bench.py --mode vb --batch 65536 --reps 10 | cut -c1-160 | sed "s/^/prefetch=$pf /"; done
