#!/bin/bash
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
timeout 900 python -m pytest tests/test_gpu_vbatched.py tests/test_gpu_parity.py tests/test_gpu_steady.py -k "f64 or dmma or vbatched" -x -q -m gpu -p no:cacheprovider --timeout 200 2>&1 | tail -3
timeout 300 python bench.py --workload f64-128x128x128:16384 --no-cpu-baseline --no-e2e 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('f64-128', round(d['value'],2), round(d['roofline']['frac'],3))"
timeout 300 python bench.py --workload f64-96x40x72:32768 --no-cpu-baseline --no-e2e 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('f64-96x40x72', round(d['value'],2), round(d['roofline']['frac'],3))"
