"""Instruction mix of one kernel by SASS opcode (and average active threads), from the ncu
source page.  usage: python tools/ncu_opmix.py report.ncu-rep [topN]"""
import collections, csv, io, subprocess, sys
rep = sys.argv[1]; top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
hdr = None; agg = collections.Counter(); thr = collections.Counter(); tot = 0
for r in csv.reader(io.StringIO(out)):
    if r and r[0] == "Address":
        hdr = r; iI = hdr.index("Instructions Executed"); iS = hdr.index("Source")
        iT = hdr.index("Thread Instructions Executed"); continue
    if hdr is None or len(r) < len(hdr): continue
    try: n = int(r[iI] or 0); t = int(r[iT] or 0)
    except ValueError: continue
    toks = r[iS].split()
    if not toks: continue
    op = toks[1] if toks[0].startswith("@") else toks[0]
    op = op.split(".")[0]
    agg[op] += n; thr[op] += t; tot += n
print(f"total warp instructions {tot / 1e9:.3f} G")
for op, n in agg.most_common(top):
    print(f"{op:10s} {n / 1e9:7.3f} G {100 * n / tot:5.1f}%  avg threads {thr[op] / max(n, 1):5.1f}")
