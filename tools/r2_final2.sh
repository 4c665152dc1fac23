#!/bin/bash
# planner data + BF16 sweep with the pair-tile XT kernel and the refit model
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
mkdir -p gpurun_out/r2g
timeout 1500 python tools/variant_sweep_r2.py --out gpurun_out/r2g/variant_sweep_r2.json > gpurun_out/r2g/variant.log 2>&1; echo "variant rc=$?"
timeout 1500 python tools/bf16_sweep.py --out gpurun_out/r2g/bf16_sweep.json > gpurun_out/r2g/sweep.log 2>&1; echo "sweep rc=$?"
timeout 900 python -m pytest tests/test_gpu_planner*.py tests/test_gpu_xt.py -q -m gpu -p no:cacheprovider --timeout 120 2>&1 | tail -2
