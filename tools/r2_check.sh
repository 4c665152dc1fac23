#!/bin/bash
# round 2 re-entry: whole GPU suite, smoke, default bench line, f2/f3 baselines
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
mkdir -p gpurun_out/r2c
timeout 1800 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider > gpurun_out/r2c/gputest.log 2>&1
echo "gputest rc=$?"; tail -6 gpurun_out/r2c/gputest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2c/smoke.log 2>&1; echo "smoke rc=$?"; tail -3 gpurun_out/r2c/smoke.log
timeout 600 python bench.py > gpurun_out/r2c/bench.json 2> gpurun_out/r2c/bench.err; echo "bench rc=$?"; cat gpurun_out/r2c/bench.json
for b in 65536; do timeout 300 python tools/vb_bench.py --mode vb --batch $b --dtype f16; done
timeout 300 python tools/vb_bench.py --mode spmm 2>&1 | tail -8
