#!/bin/bash
# transposed-product kernel: GPU tests, variant sweep (planner check data),
# BF16 sweep with the new AUTO, sanitizers on the new / changed pipelines
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
mkdir -p gpurun_out/r2x
timeout 900 python -m pytest tests/test_gpu_xt.py tests/test_gpu_parity.py -x -q -m gpu -p no:cacheprovider --timeout 300 2>&1 | tail -3
timeout 1500 python tools/variant_sweep_r2.py > gpurun_out/r2x/variant.log 2>&1; echo "variant rc=$?"; tail -2 gpurun_out/r2x/variant.log
cp profiles/r2/variant_sweep_r2.json gpurun_out/r2x/ 2>/dev/null
timeout 1500 python tools/bf16_sweep.py --out gpurun_out/r2x/bf16_sweep.json > gpurun_out/r2x/sweep.log 2>&1; echo "sweep rc=$?"; tail -3 gpurun_out/r2x/sweep.log
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 30 python tools/sanitize_cases.py > gpurun_out/r2x/san_$tool.log 2>&1
  echo "== $tool rc=$?"; tail -5 gpurun_out/r2x/san_$tool.log
done
