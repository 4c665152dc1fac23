#!/bin/bash
# round 2: the whole GPU suite + compute-sanitizer on one small case per instantiation
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
mkdir -p gpurun_out/r2/san
timeout 3000 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider > gpurun_out/r2/gputest.log 2>&1
tail -25 gpurun_out/r2/gputest.log
for tool in memcheck racecheck synccheck; do
  timeout 1200 compute-sanitizer --tool $tool --print-limit 30 python tools/sanitize_cases.py > gpurun_out/r2/san/$tool.log 2>&1
  echo "== $tool rc=$?"; tail -4 gpurun_out/r2/san/$tool.log
done
