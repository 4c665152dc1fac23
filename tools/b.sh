#!/bin/bash
# build libkami.so and say loudly whether it worked
cd "$(dirname "$0")/.." && python -m paper_conf_sc_wangdltsl25_b200.build > /tmp/kami_build.log 2>&1
rc=$?
if [ $rc -ne 0 ]; then echo "BUILD FAILED"; grep -E "error" -A3 /tmp/kami_build.log | head -20; exit 1; fi
echo "BUILD OK"; grep -h "spill stores" paper_conf_sc_wangdltsl25_b200/_build/*.log | grep -v " 0 bytes spill" | head -3
