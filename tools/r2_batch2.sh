#!/bin/bash
# round 2 batch 2: TS tuning, CA SMEM bytes (ncu), TMA row-width ubench, variant sweep
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
mkdir -p gpurun_out/r2 gpurun_out/ca
timeout 600 python -m pytest tests/test_gpu_f64_general.py -q -x --timeout 300 -p no:cacheprovider 2>&1 | tail -3
line() { python -c "import json,sys; d=json.loads(open('$1').read().strip().splitlines()[-1]); print('$2', round(d['value'],2), d['roofline']['kernel'], round(d['roofline']['frac'],3), d['clocks']['sm_mhz'])" 2>/dev/null || echo "$2 FAILED"; }
for wl in f16-64 f16-128 f16-32; do
 for tune in "0,0,0" "0,0,2" "3,0,0" "4,0,0" "6,0,0" "8,0,0" "0,4,0" "0,8,0" "4,8,2" "6,16,2"; do
  KAMI_TS_TUNE=$tune timeout 300 python bench.py --workload $wl --algo 1d_tmem --steps 20 --warmup 5 --no-cpu-baseline --no-e2e > gpurun_out/r2/t.json 2>/dev/null
  line gpurun_out/r2/t.json "ts1d $wl tune=$tune"
 done
 timeout 300 python bench.py --workload $wl --algo 1d --steps 20 --warmup 5 --no-cpu-baseline --no-e2e > gpurun_out/r2/t.json 2>/dev/null
 line gpurun_out/r2/t.json "ss $wl"
done
for wl in f64-128x128x128:16384 f64-256x256x256:2048 f64-96x40x72:32768 f64-48x48x48 f64-24x40x56:65536; do
  timeout 300 python bench.py --workload $wl --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/r2/t.json 2>/dev/null
  line gpurun_out/r2/t.json "gen $wl"
done
M=smsp__sass_data_bytes_mem_shared_op_ld.sum,smsp__sass_data_bytes_mem_shared_op_st.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum,smsp__inst_executed_pipe_tensor.sum,gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,l1tex__m_xbar2l1tex_read_bytes_mem_global_op_tma_ld.sum,l1tex__m_l1tex2xbar_write_bytes_mem_global_op_tma_st.sum
run() { timeout 300 ncu --metrics $M --clock-control none -k regex:kami_ -c 1 --csv --log-file gpurun_out/ca/$1.csv python tools/prof_one.py --workload $2 --algo $3 --p $4 --batch $5 --iters 1 > /dev/null 2>&1; }
run f16-64_ts1d f16-64 1d_tmem 0 8192
run f16-64_ts3d f16-64 3d_tmem 0 8192
run f16-128_ts1d f16-128 1d_tmem 0 4096
run f16-128_ts3d f16-128 3d_tmem 0 4096
run f16-32_ts1d f16-32 1d_tmem 0 8192
run f16-32_tc16 f16-32 1d 0 8192
run f16-64_tc16 f16-64 auto 0 8192
run f16-128_tc16 f16-128 auto 0 4096
run f16-64_nonca f16-64 nonca 0 8192
run f16-64_nonca8 f16-64 nonca 8 8192
run f16-64_3d f16-64 3d 0 8192
run f16-64_2d f16-64 2d 0 8192
run f16-128_nonca16 f16-128 nonca 16 4096
run f16-32_nonca f16-32 nonca 0 8192
ls gpurun_out/ca | wc -l
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -Ipaper_conf_sc_wangdltsl25_b200/csrc -o tools/ubench_tma tools/ubench_tma.cu -lcuda && timeout 300 ./tools/ubench_tma > gpurun_out/r2/ubench_tma.json
timeout 1200 python tools/variant_sweep_r2.py > gpurun_out/r2/variant_sweep.log 2>&1; tail -5 gpurun_out/r2/variant_sweep.log
cp profiles/r2/variant_sweep_r2.json gpurun_out/r2/ 2>/dev/null
