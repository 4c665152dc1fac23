#!/bin/bash
# which classes of the mixed-size batch are slow: sub-mixes by m / n / k order sets
python -m paper_conf_sc_wangdltsl25_b200.build > /dev/null
run() { timeout 60 python tools/vb_bench.py --mode vb --reps 10 "$@" | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(' '.join(sys.argv[1:]), round(d['frac_hbm'],3), round(d['ms'],3))" "$@"; }
run --batch 65536
run --batch 40000 --orders 64,128,192,256
run --batch 65536 --morders 16,32
run --batch 65536 --morders 64,128,192,256
run --batch 65536 --norders 16,32
run --batch 65536 --norders 64,128,192,256
run --batch 65536 --korders 16,32
run --batch 65536 --korders 64,128,192,256
run --batch 65536 --morders 16,32 --norders 128,192,256
run --batch 65536 --morders 128,192,256 --norders 16,32
run --batch 65536 --morders 192 
run --batch 65536 --morders 128,256
