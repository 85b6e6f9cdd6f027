"""Aggregate ncu source-page metrics per CUDA source line (needs -lineinfo builds).
usage: python tools/ncu_lines.py report.ncu-rep [topN]"""
import csv, io, os, sys
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from ncu_csv import page
rep = sys.argv[1]; top = int(sys.argv[2]) if len(sys.argv) > 2 else 30
out = page(rep, "src")
rows = list(csv.reader(io.StringIO(out)))
agg = []
cur_file = None; hdr = None; cur = None
for r in rows:
    if not r: continue
    if r[0] == "File Path": cur_file = r[1].split('/')[-1]; continue
    if r[0] == "Line No": hdr = r; iS = hdr.index("Warp Stall Sampling (All Samples)"); iI = hdr.index("Instructions Executed"); continue
    if hdr is None or r[0] == "Function Name": continue
    if r[0]:  # source line row (aggregated)
        try: agg.append((int(r[iS] or 0), int(r[iI] or 0), f"{cur_file}:{r[0]}", r[1].strip()[:90]))
        except ValueError: pass
tot_s = sum(a[0] for a in agg) or 1; tot_i = sum(a[1] for a in agg) or 1
print(f"total samples {tot_s}, instructions {tot_i}")
print("-- by stall samples"); [print(f"{100*s/tot_s:5.1f}% {100*i/tot_i:5.1f}%i {loc:18s} {src}") for s, i, loc, src in sorted(agg, reverse=True)[:top]]
print("-- by instructions"); [print(f"{100*s/tot_s:5.1f}% {100*i/tot_i:5.1f}%i {loc:18s} {src}") for s, i, loc, src in sorted(agg, key=lambda a: -a[1])[:top]]
