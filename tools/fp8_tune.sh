for i in 1 2; do for w in e4m3-64 f16-32; do for t in "0,0,0,-1,0,0" "0,2,0,-1,2,0" "0,1,0,-1,2,0" "3,0,0,-1,0,0" "4,0,0,-1,0,0" "8,0,0,-1,0,0"; do
  echo -n "$w $t: "; KAMI_TC_TUNE=$t timeout 120 python bench.py --workload $w --steps 30 --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],2), round(d['roofline']['frac'],3), d['clocks']['sm_mhz'])"
done; done; done
