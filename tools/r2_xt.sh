#!/bin/bash
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
timeout 900 python -m pytest tests/test_gpu_xt.py -x -q -m gpu -p no:cacheprovider --timeout 120 2>&1 | tail -4
timeout 600 python tools/xt_ab.py
