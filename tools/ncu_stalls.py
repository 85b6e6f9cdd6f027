"""Stall-reason totals of a kernel (whole kernel and the top-N SASS sites) from the SASS source page.
usage: python tools/ncu_stalls.py REPORT_OR_EXPORT_PREFIX [topN]"""
import csv
import io
import os
import sys
from collections import Counter

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from ncu_csv import page  # noqa: E402

rows = list(csv.reader(io.StringIO(page(sys.argv[1], "sass"))))
top = int(sys.argv[2]) if len(sys.argv) > 2 else 12
hi = next(i for i, r in enumerate(rows) if r and r[0] == "Address")
h = rows[hi]
cols = [i for i, c in enumerate(h) if c.startswith("stall_") and "Not Issued" not in c]
iS, iI, iSrc = h.index("Warp Stall Sampling (All Samples)"), h.index("Instructions Executed"), h.index("Source")
tot = Counter()
sites = []
for r in rows[hi + 1:]:
    if len(r) < len(h) or r[0] == "Address":
        continue
    c = Counter({h[i]: float(r[i] or 0) for i in cols})
    tot.update(c)
    sites.append((float(r[iS] or 0), r[0], r[iSrc].strip(), c, int(float(r[iI] or 0))))
T = sum(tot.values()) or 1
print("kernel stall mix: " + ", ".join(f"{k[6:]} {100 * v / T:.1f}%" for k, v in tot.most_common(8)))
for s, a, src, c, n in sorted(sites, reverse=True)[:top]:
    mix = ", ".join(f"{k[6:]} {100 * v / (s or 1):.0f}%" for k, v in c.most_common(3) if v)
    print(f"{100 * s / T:5.1f}% x{n:<11d} {a} {src[:60]:60s} [{mix}]")
