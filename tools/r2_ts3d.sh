#!/bin/bash
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
O=gpurun_out/r2t; mkdir -p $O
for al in 1d_tmem 3d_tmem; do
  timeout 300 ncu --set full --import-source on --clock-control none -k regex:kami_ -s 2 -c 1 -f -o $O/$al python tools/prof_one.py --workload f16-64 --algo $al --iters 3 > /dev/null 2>&1
  ncu -i $O/$al.ncu-rep --page source --csv --print-source sass > $O/src_$al.csv 2>/dev/null
  ncu -i $O/$al.ncu-rep --page raw --csv --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed > $O/raw_$al.csv 2>/dev/null
  rm -f $O/$al.ncu-rep
  echo "== $al"; python tools/ncu_stalls.py $O/src_$al.csv 8
done
