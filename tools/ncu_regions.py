"""Share of warp instructions / stall samples per source region of the Map kernel.
usage: python tools/ncu_regions.py report.ncu-rep"""
import collections, csv, io, os, sys
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from ncu_csv import page
out = page(sys.argv[1], "src")
cur = hdr = None; data = []
for r in csv.reader(io.StringIO(out)):
    if not r: continue
    if r[0] == "File Path": cur = r[1].split('/')[-1]; continue
    if r[0] == "Line No":
        hdr = r; iS = hdr.index("Warp Stall Sampling (All Samples)"); iI = hdr.index("Instructions Executed"); continue
    if hdr is None or not r[0]: continue
    try: data.append((cur, int(r[0]), int(r[iI] or 0), int(r[iS] or 0)))
    except ValueError: pass
REG = [l.split("|") for l in open(sys.argv[2]).read().split("\n") if l.strip()] if len(sys.argv) > 2 else []
tot = sum(d[2] for d in data) or 1; tots = sum(d[3] for d in data) or 1
acc = collections.Counter(); accs = collections.Counter()
for f, l, i, s in data:
    name = "other:" + str(f)
    for rf, a, b, n in REG:
        if f == rf and int(a) <= l <= int(b): name = n
    acc[name] += i; accs[name] += s
print(f"total {tot / 1e9:.2f} G warp instructions")
for n, i in acc.most_common(): print(f"{n:30s} {100 * i / tot:5.1f}%i {100 * accs[n] / tots:5.1f}%stall")
