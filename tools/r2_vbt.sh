#!/bin/bash
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
mkdir -p gpurun_out/vbt
KAMI_VB_SORT=0 timeout 120 python tools/vb_bench.py --mode vb --batch 65536 > gpurun_out/vbt/a.out 2> gpurun_out/vbt/a.err; echo "rc=$?"
tail -3 gpurun_out/vbt/a.out; tail -5 gpurun_out/vbt/a.err
KAMI_VB_SORT=0 timeout 120 python tools/vb_bench.py --mode vb --batch 4096 > gpurun_out/vbt/b.out 2> gpurun_out/vbt/b.err; echo "rc=$?"
tail -3 gpurun_out/vbt/b.out; tail -5 gpurun_out/vbt/b.err
