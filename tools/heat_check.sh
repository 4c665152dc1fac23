for i in 1 2 3; do python bench.py --steps 30 --warmup 5 --no-cpu-baseline --no-e2e | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],1), d['clocks'])"; done
python tools/tc_tune.py --workload f16-64 --tunes 0,0,0,-1
timeout 300 python tools/bf16_sweep.py --orders 128,192,256 --out /tmp/x.json > /dev/null 2>&1
for i in 1 2 3; do python bench.py --steps 30 --warmup 5 --no-cpu-baseline --no-e2e | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],1), d['clocks'])"; done
python tools/tc_tune.py --workload f16-64 --tunes 0,0,0,-1
