"""Top SASS lines by warp-stall samples from `ncu --page source --csv --print-source sass`,
with each line's dominant stall reasons, plus the kernel-wide stall-reason totals.

usage: python tools/sass_hot.py SOURCE.csv [N] [ADDR_LO ADDR_HI]"""
import csv
import sys
from collections import Counter

rows = list(csv.reader(open(sys.argv[1])))
h = rows[1]
n = int(sys.argv[2]) if len(sys.argv) > 2 else 40
lo = int(sys.argv[3], 16) if len(sys.argv) > 3 else None
hi = int(sys.argv[4], 16) if len(sys.argv) > 4 else None
ia, isrc, ist = h.index("Address"), h.index("Source"), h.index("Warp Stall Sampling (All Samples)")
ie = h.index("Instructions Executed")
stall_cols = [i for i, c in enumerate(h) if c.startswith("stall_") and "Not Issued" not in c]
seen, data, base = set(), [], None
for r in rows[2:]:
    try:
        key = r[ia]
        if key in seen:
            continue
        seen.add(key)
        addr = int(key, 16)
        if base is None:
            base = addr
        off = addr - base
        if lo is not None and not (lo <= off < hi):
            continue
        st = Counter({h[i][6:]: int(r[i] or 0) for i in stall_cols})
        data.append((int(r[ist] or 0), off, addr, r[isrc][:70], r[ie], st))
    except (ValueError, IndexError):
        pass
tot = sum(d[0] for d in data) or 1
agg = Counter()
for d in data:
    agg.update(d[5])
print("total samples", tot, " by reason:", ", ".join(f"{k} {100 * v / tot:.1f}%" for k, v in agg.most_common(8)))
for d in sorted(data, key=lambda d: -d[0])[:n]:
    top = ", ".join(f"{k} {v}" for k, v in d[5].most_common(2) if v)
    print(f"{100 * d[0] / tot:5.1f}% {d[1]:#07x} {d[3]:70s} exec={d[4]:>9s} [{top}]")
