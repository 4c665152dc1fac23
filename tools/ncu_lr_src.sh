mkdir -p gpurun_out/lrn
for w in lr-16 lr-32; do
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:kami_ -s 2 -c 1 -f -o gpurun_out/lrn/full_$w python tools/prof_one.py --workload $w --iters 3 > gpurun_out/lrn/full_$w.log 2>&1
  ncu -i gpurun_out/lrn/full_$w.ncu-rep --page source --csv --print-source sass > gpurun_out/lrn/src_$w.csv 2>/dev/null
  ncu -i gpurun_out/lrn/full_$w.ncu-rep --page raw --csv > gpurun_out/lrn/raw_$w.csv 2>/dev/null
done
ls -la gpurun_out/lrn
