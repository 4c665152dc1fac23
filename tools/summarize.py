import json, sys
for f in sys.argv[1:]:
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
    except Exception as e:
        print(f, "ERR", e)
        continue
    if "roofline" not in d:
        print(f"{f:40s} {d.get('value', 0):9.4g} {d.get('unit', '')} ({d.get('impl', '?')})")
        continue
    r = d["roofline"]
    print(f"{f:40s} {d['value']:9.2f} TF {d['ms_per_step']:8.4f} ms {r['bound']:6s} {r['achieved']:8.1f} {r['unit']} "
          f"frac {r['frac']:.3f} roof {r['frac_of_roofline_tflops']:.3f} {r['kernel']} sm {d['clocks']['sm_mhz']} {d['clocks']['reasons']}")
