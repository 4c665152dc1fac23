#!/bin/bash
# full ncu captures (source-level stall sampling) of the low-rank and headline tcgen05 launches
mkdir -p gpurun_out/r1b
for w in ${WORKLOADS:-lr-16 f16-64}; do
  ncu --set full --clock-control none --import-source on -k regex:kami_ -s 2 -c 1 -f \
      -o gpurun_out/r1b/full_$w python tools/prof_one.py --workload $w --iters 3 > gpurun_out/r1b/full_$w.log 2>&1
done
python tools/mix_bw.py > gpurun_out/r1b/mix_bw.json 2>&1
