#!/bin/bash
# variant sweep refresh + the whole GPU suite + smoke
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
mkdir -p gpurun_out/r2h
timeout 900 python tools/variant_sweep_r2.py --out gpurun_out/r2h/variant_sweep_r2.json > gpurun_out/r2h/variant.log 2>&1; echo "variant rc=$?"
timeout 2400 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider > gpurun_out/r2h/gputest.log 2>&1; echo "gputest rc=$?"; tail -4 gpurun_out/r2h/gputest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -3
