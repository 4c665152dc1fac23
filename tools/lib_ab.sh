#!/bin/bash
# same-box A/B of two library builds (KAMI_LIB) on bench workloads, interleaved
# usage: LIBB=paper_conf_sc_wangdltsl25_b200/libkami_old.so WL="lr-8 lr-16" tools/lib_ab.sh
mkdir -p gpurun_out/lab
for rep in a b; do for w in ${WL:-lr-8 lr-16 lr-32 f16-64}; do
  timeout 300 python bench.py --workload $w --steps 50 --warmup 5 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 > gpurun_out/lab/${w}_A_$rep.json
  KAMI_LIB=$PWD/${LIBB:-paper_conf_sc_wangdltsl25_b200/libkami_old.so} timeout 300 python bench.py --workload $w --steps 50 --warmup 5 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 > gpurun_out/lab/${w}_B_$rep.json
done; done
python tools/summarize.py gpurun_out/lab/*.json
