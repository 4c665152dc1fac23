#!/bin/bash
# what the driver runs at round end: build, GPU suite, smoke, bench (N=1)
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
mkdir -p gpurun_out/r2f
timeout 3000 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider > gpurun_out/r2f/gputest.log 2>&1
tail -6 gpurun_out/r2f/gputest.log
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -3
timeout 900 python bench.py > gpurun_out/r2f/bench.json 2> gpurun_out/r2f/bench.err; tail -c 1500 gpurun_out/r2f/bench.json
