"""Top SASS lines by warp-stall samples from an `ncu --page source --csv` dump:
    python tools/ncu_src_top.py file.source.csv [N]"""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
N = int(sys.argv[2]) if len(sys.argv) > 2 else 25
hdr = rows[1]
si = hdr.index("Warp Stall Sampling (All Samples)")
tot = 0
lines = []
for r in rows[2:]:
    if len(r) <= si:
        continue
    try:
        s = int(r[si])
    except ValueError:
        continue
    tot += s
    lines.append((s, r[0], r[1].strip()))
lines.sort(reverse=True)
print("total samples", tot)
for s, a, src in lines[:N]:
    print(f"{s:7d} {100.0 * s / max(tot, 1):5.1f}%  {a[-5:]}  {src[:90]}")
