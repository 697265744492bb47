"""Top SASS lines by warp-stall samples from `ncu --page source --csv --print-source sass`."""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
h = rows[1]
data = []
for r in rows[2:]:   # the first kernel only (a capture with several ends at the next "Kernel Name" row)
    if r and r[0] == "Kernel Name":
        break
    data.append(r)
i_src, i_s = h.index("Source"), h.index("Warp Stall Sampling (All Samples)")
data = [r for r in data if len(r) > i_s and (r[i_s] or '0').isdigit()]
tot = sum(int(r[i_s] or 0) for r in data)
top = sorted(data, key=lambda r: -int(r[i_s] or 0))[: int(sys.argv[2]) if len(sys.argv) > 2 else 25]
print("total samples", tot)
for r in top:
    print(f"{int(r[i_s]):6d} {100 * int(r[i_s]) / max(tot, 1):5.1f}%  {r[0][-5:]}  {r[i_src].strip()[:90]}")
