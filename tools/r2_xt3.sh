#!/bin/bash
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
timeout 900 python -m pytest tests/test_gpu_xt.py -x -q -m gpu -p no:cacheprovider --timeout 120 2>&1 | tail -3
#timeout 600 python tools/xt_ab.py
#timeout 300 python bench.py --workload f64-32 --no-cpu-baseline --no-e2e 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('f64-32', d['value'], d['roofline']['frac'], d['clocks'])"
#timeout 300 python bench.py --workload f64-64 --no-cpu-baseline --no-e2e 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('f64-64', d['value'], d['roofline']['frac'], d['clocks'])"
