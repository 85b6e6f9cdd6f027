"""Executed warp instructions by opcode class (ALU / FMA-pipe integer / memory / control) per
source region, from an ncu export (SASS page joined with the cuda,sass page for line info).
usage: python tools/ncu_opmix2.py EXPORT_PREFIX REGIONS_FILE"""
import csv
import io
import os
import sys
from collections import Counter, defaultdict

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from ncu_csv import page  # noqa: E402

ALU = ("LOP3", "IADD3", "SHF", "PRMT", "SEL", "ISETP", "FLO", "BREV", "VIMNMX", "POPC", "LEA", "IABS", "FSEL",
       "FSETP", "FMNMX", "P2R", "R2P", "PLOP3", "VIADD", "ISCADD", "IMNMX", "LOP", "BMSK", "SGXT")
FMA = ("IMAD", "FFMA", "FADD", "FMUL", "HFMA2", "IMUL", "FADD2", "FFMA2", "FMUL2")


def klass(op):
    o = op.split()[0]
    if o.startswith("@"):
        o = op.split()[1]
    b = o.split(".")[0]
    if b in ALU:
        return "alu"
    if b in FMA:
        return "fma"
    if b in ("LDS", "STS", "ATOMS", "LDG", "STG", "REDG", "ATOMG", "LD", "ST", "LDSM", "SHFL", "MATCH", "LDL", "STL",
             "RED", "ATOM", "UBLKCP", "SYNCS", "REDUX", "VOTE", "CCTL", "MEMBAR", "FENCE"):
        return "mem/sync"
    return "ctl/other"


def main():
    prefix, regf = sys.argv[1], sys.argv[2]
    regs = [l.split("|") for l in open(regf).read().split("\n") if l.strip()]
    rows = list(csv.reader(io.StringIO(page(prefix, "src"))))
    cur_file, cur_line, hdr = None, None, None
    acc = defaultdict(Counter)
    for r in rows:
        if not r:
            continue
        if r[0] == "File Path":
            cur_file = r[1].split("/")[-1]
            continue
        if r[0] == "Line No":
            hdr = r
            iI = hdr.index("Instructions Executed")
            continue
        if hdr is None or r[0] == "Function Name":
            continue
        if r[0]:
            try:
                cur_line = int(r[0])
            except ValueError:
                pass
            continue
        if len(r) > iI and r[2].startswith("0x"):
            name = "other:" + str(cur_file)
            for rf, a, b, n in regs:
                if cur_file == rf and int(a) <= cur_line <= int(b):
                    name = n
            acc[name][klass(r[3].strip())] += float(r[iI] or 0)
    T = sum(sum(c.values()) for c in acc.values()) or 1
    print(f"{'region':32s} {'share':>6s}  alu    fma    mem    ctl")
    for name, c in sorted(acc.items(), key=lambda x: -sum(x[1].values())):
        t = sum(c.values())
        print(f"{name:32s} {100 * t / T:5.1f}%  " + "  ".join(f"{100 * c[k] / T:4.1f}%" for k in ("alu", "fma", "mem/sync", "ctl/other")))
    # fallback: use the sass page (no line info) for the global mix
    srows = list(csv.reader(io.StringIO(page(prefix, "sass"))))
    hi = next(i for i, r in enumerate(srows) if r and r[0] == "Address")
    h = srows[hi]
    iI, iSrc = h.index("Instructions Executed"), h.index("Source")
    tot = Counter()
    for r in srows[hi + 1:]:
        if len(r) <= iI or r[0] == "Address":
            continue
        n = float(r[iI] or 0)
        tot[klass(r[iSrc].strip())] += n
    T = sum(tot.values())
    print(f"total {T / 1e9:.2f} G: " + ", ".join(f"{k} {100 * v / T:.1f}%" for k, v in tot.most_common()))


main()
