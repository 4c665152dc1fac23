"""Top SASS lines by warp-stall samples from an `ncu --page source --csv
--print-source sass` export (with the dominant stall reasons), plus the
kernel-wide stall breakdown.   python tools/ncu_stalls.py file.csv [N]"""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hdr, data = rows[1], rows[2:]
i_s, i_src, i_ex = hdr.index("Warp Stall Sampling (All Samples)"), hdr.index("Source"), hdr.index("Instructions Executed")
cols = [i for i, h in enumerate(hdr) if h.startswith("stall_") and "Not Issued" not in h]
tot = sum(float(r[i_s] or 0) for r in data)
agg = {}
for r in data:
    for i in cols:
        agg[hdr[i]] = agg.get(hdr[i], 0) + float(r[i] or 0)
print("samples", tot, "| by reason:", ", ".join(f"{k[6:]} {v / tot * 100:.1f}%" for v, k in
                                                 sorted(((v, k) for k, v in agg.items()), reverse=True)[:8]))
for r in sorted(data, key=lambda r: -float(r[i_s] or 0))[: int(sys.argv[2]) if len(sys.argv) > 2 else 20]:
    st = sorted(((float(r[i] or 0), hdr[i][6:]) for i in cols), reverse=True)[:2]
    print(f"{r[0][-5:]} {float(r[i_s]) / tot * 100:5.1f}% exec {r[i_ex]:>8} {r[i_src].strip()[:58]:58} {st}")
