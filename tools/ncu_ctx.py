"""Context of given SASS addresses in an ncu source CSV (and the role split).
    python tools/ncu_ctx.py src.csv addr1 addr2 ...  (last 5 hex digits)"""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hdr, data = rows[1], rows[2:]
i_s = hdr.index("Warp Stall Sampling (All Samples)")
i_src = hdr.index("Source")
i_ex = hdr.index("Instructions Executed")
addr = [r[0] for r in data]
for t in sys.argv[2:]:
    idx = [i for i, a in enumerate(addr) if a.endswith(t)][0]
    print("-----", t)
    for r in data[max(0, idx - 12):idx + 2]:
        print(r[0][-5:], r[i_ex].rjust(9), r[i_s].rjust(6), r[i_src][:96])
