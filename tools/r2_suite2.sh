#!/bin/bash
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
mkdir -p gpurun_out/r2y
timeout 2400 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider > gpurun_out/r2y/gputest.log 2>&1; echo "gputest rc=$?"; tail -4 gpurun_out/r2y/gputest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -5
timeout 600 python bench.py > gpurun_out/r2y/bench_default.json 2> gpurun_out/r2y/bench_default.err; echo "bench rc=$?"; cut -c1-300 gpurun_out/r2y/bench_default.json
