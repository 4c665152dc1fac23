mkdir -p gpurun_out/tf
for L in libkami_old.so libkami.so libkami_old.so libkami.so; do echo -n "tf32-64 $L: "; KAMI_LIB=paper_conf_sc_wangdltsl25_b200/$L timeout 120 python bench.py --workload tf32-64 --steps 30 --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],2), round(d['roofline']['frac'],3), d['clocks']['sm_mhz'])"; done
timeout 300 ncu --set full --clock-control none --import-source on -k regex:kami_ -s 2 -c 1 -f -o gpurun_out/tf/full_tf32 python tools/prof_one.py --workload tf32-64 --iters 3 > gpurun_out/tf/full.log 2>&1
ncu -i gpurun_out/tf/full_tf32.ncu-rep --page source --csv --print-source sass > gpurun_out/tf/src_tf32.csv 2>/dev/null
