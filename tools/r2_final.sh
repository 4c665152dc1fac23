#!/bin/bash
# round 2 final evidence on one box: whole GPU suite, smoke, default bench line,
# every bench workload, planner data, BF16 sweep (graph-timed)
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
O=gpurun_out/r2z; mkdir -p $O
timeout 2400 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider > $O/gputest.log 2>&1; echo "gputest rc=$?"; tail -3 $O/gputest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"; cat $O/smoke.log
timeout 600 python bench.py > $O/bench_default.json 2> $O/bench_default.err; echo "bench rc=$?"; cut -c1-400 $O/bench_default.json
bash tools/r2_lines.sh > $O/lines.log 2>&1; cat $O/lines.log; cp -r gpurun_out/r2l $O/ 2>/dev/null
timeout 900 python tools/variant_sweep_r2.py --out $O/variant_sweep_r2.json > $O/variant.log 2>&1; echo "variant rc=$?"
timeout 1500 python tools/bf16_sweep.py --out $O/bf16_sweep.json > $O/sweep.log 2>&1; echo "sweep rc=$?"
