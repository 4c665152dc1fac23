#!/bin/bash
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
mkdir -p gpurun_out/r2
timeout 1500 python -m pytest tests/test_gpu_grid8.py tests/test_gpu_f64_general.py tests/test_gpu_parity.py -q --timeout 600 -p no:cacheprovider 2>&1 | tail -15
timeout 1500 python tools/variant_sweep_r2.py > gpurun_out/r2/variant_sweep.log 2>&1; tail -3 gpurun_out/r2/variant_sweep.log
cp profiles/r2/variant_sweep_r2.json gpurun_out/r2/
./tools/r2_evidence.sh
