#!/bin/bash
# planner data refresh (variant sweep), thin shapes with the refit model, oracle checks of the changed pipelines
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
mkdir -p gpurun_out/r2f
timeout 1500 python tools/variant_sweep_r2.py --out gpurun_out/r2f/variant_sweep_r2.json > gpurun_out/r2f/variant.log 2>&1; echo "variant rc=$?"
grep "f64-32\|32x192x16" gpurun_out/r2f/variant.log
timeout 600 python tools/xt_ab.py > gpurun_out/r2f/xt_ab.log 2>&1; echo "xt rc=$?"
timeout 600 python tools/sanitize_cases.py 2>&1 | tail -22
