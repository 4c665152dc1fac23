#!/bin/bash
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
mkdir -p gpurun_out/r2s
timeout 1500 python tools/bf16_sweep.py --out gpurun_out/r2s/bf16_sweep.json > gpurun_out/r2s/sweep.log 2>&1; echo "sweep rc=$?"; tail -2 gpurun_out/r2s/sweep.log | cut -c1-200
