#!/bin/bash
# ncu shared-memory traffic per MMA for each CA schedule vs the non-CA baseline
# (the CA claim of BASELINE.json north_star).  One launch per variant.
M=smsp__sass_data_bytes_mem_shared_op_ld.sum,smsp__sass_data_bytes_mem_shared_op_st.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum,smsp__inst_executed_pipe_tensor.sum,smsp__inst_executed_pipe_fp64.sum,sm__inst_executed_pipe_uma.sum,gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,l1tex__m_xbar2l1tex_read_bytes_mem_global_op_tma_ld.sum,l1tex__m_l1tex2xbar_write_bytes_mem_global_op_tma_st.sum
mkdir -p gpurun_out/ca
run() { # tag workload algo p batch
  timeout 300 ncu --metrics $M --clock-control none -k regex:kami_ -c 1 --csv --log-file gpurun_out/ca/$1.csv \
    python tools/prof_one.py --workload $2 --algo $3 --p $4 --batch $5 --iters 1 > /dev/null 2>&1
}
for a in 1d 2d 3d nonca; do run f64-32_$a f64-32 $a 0 8192; run f64-64_$a f64-64 $a 0 4096; done
run f64-64_1dm8 f64-64 1d 8 4096
run f64-64_nonca16 f64-64 nonca 16 4096
run f64-64_nonca8 f64-64 nonca 8 4096
run f64-32_nonca8 f64-32 nonca 8 8192
run f16-64_nonca8 f16-64 nonca 8 8192
run f16-128_nonca16 f16-128 nonca 16 4096
run f16-64_w1d f16-64 1d 4 8192
for a in 2d 3d nonca; do run f16-64_$a f16-64 $a 0 8192; done
run f16-32_w1d f16-32 1d 2 8192
for a in 2d nonca; do run f16-32_$a f16-32 $a 0 8192; done
run f16-64_tc16 f16-64 auto 0 8192
run f16-128_tc16 f16-128 auto 0 4096
run f16-128_w1d f16-128 1d 8 4096
run f16-128_2d f16-128 2d 0 4096
ls gpurun_out/ca
