#!/bin/bash
# FP64 k-permutation (bank conflicts), thin warp kernels, 8-grid fix: parity + perf + ncu check
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
mkdir -p gpurun_out/r2b4
timeout 1800 python -m pytest tests/test_gpu_thin.py tests/test_gpu_grid8.py tests/test_gpu_f64_general.py tests/test_gpu_steady.py tests/test_gpu_vbatched.py tests/test_gpu_f4.py tests/test_gpu_spmm.py -q --timeout 600 -p no:cacheprovider -k "f64 or thin or grid8 or zmorton or axpby_f64" 2>&1 | tail -8
line() { python -c "import json,sys; d=json.loads(open('$1').read().strip().splitlines()[-1]); print('$2', round(d['value'],2), d['roofline']['kernel'], d['roofline']['bound'], round(d['roofline']['frac'],3), d['clocks']['sm_mhz'])" 2>/dev/null || echo "$2 FAILED"; }
for wl in f64-64 f64-32 f64-16 f64-128x128x128:16384 f64-256x256x256:2048 f64-96x40x72:32768 f64-48x48x48; do
  timeout 300 python bench.py --workload $wl --steps 20 --warmup 5 --no-cpu-baseline --no-e2e > gpurun_out/r2b4/t.json 2>/dev/null
  line gpurun_out/r2b4/t.json "$wl"
done
M=l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum,smsp__sass_data_bytes_mem_shared_op_ld.sum,smsp__inst_executed_op_shared_ld.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum,gpu__time_duration.sum,sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active
for w in f64-64 f64-32 f64-128x128x128:8192; do
  timeout 300 ncu --metrics $M --clock-control none -k regex:kami_ -c 1 --csv python tools/prof_one.py --workload $w --iters 1 2>/dev/null | grep -v "^==" | tail -8
done
