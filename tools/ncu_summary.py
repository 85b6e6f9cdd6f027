"""Summarise ncu reports (run here, on the CPU box, over reports brought back in gpurun_out/).

usage: python tools/ncu_summary.py OUT.md report1.ncu-rep [report2 ...]
       python tools/ncu_summary.py --launches OUT.txt launches.csv
"""
import csv
import io
import os
import subprocess
import sys

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from ncu_csv import page  # noqa: E402
from collections import defaultdict

METRICS = [
    ("gpu__time_duration.sum", "duration"),
    ("dram__bytes_read.sum", "dram read"),
    ("dram__bytes_write.sum", "dram write"),
    ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "DRAM % peak"),
    ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "SM % peak"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "occupancy %"),
    ("launch__registers_per_thread", "regs/thread"),
    ("launch__grid_size", "grid"),
    ("launch__block_size", "block"),
    ("smsp__inst_executed.sum", "warp instructions"),
    ("l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "smem bank conflicts"),
    ("smsp__issue_active.avg.pct_of_peak_sustained_active", "issue active %"),
    ("sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active", "ALU pipe %"),
    ("sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active", "FMA pipe %"),
    ("sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active", "FMA pipe cycles %"),
    ("sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active", "LSU pipe %"),
    ("smsp__thread_inst_executed_per_inst_executed.ratio", "threads / instruction"),
    ("l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "smem wavefronts"),
    ("l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_atom.sum", "smem bank conflicts (atomics)"),
    ("smsp__inst_executed_op_shared_atom.sum", "shared atomics (warp inst)"),
    ("l1tex__m_xbar2l1tex_read_sectors_mem_global_op_atom.sum", "global atomic sectors"),
    ("l1tex__m_l1tex2xbar_write_sectors_mem_global_op_red.sum", "global RED sectors"),
]


def raw(rep):
    rows = list(csv.reader(io.StringIO(page(rep, "raw"))))
    hi = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    return rows[hi], rows[hi + 1], rows[hi + 2:]


def top_stalls(rep, idx=0, n=6):
    out = page(rep, "sass", ["--launch-skip", str(idx), "--launch-count", "1"])
    rows = list(csv.reader(io.StringIO(out)))
    if len(rows) < 3:
        return []
    h = rows[1]
    iS, iI, iSrc = h.index("Warp Stall Sampling (All Samples)"), h.index("Instructions Executed"), h.index("Source")
    data = []
    for r in rows[2:]:
        try:
            data.append((int(r[iS] or 0), int(r[iI] or 0), r[iSrc].strip()))
        except (ValueError, IndexError):
            pass
    tot = sum(d[0] for d in data) or 1
    return [(100.0 * s / tot, i, src) for s, i, src in sorted(data, reverse=True)[:n]]


def main():
    if sys.argv[1] == "--launches":
        out, path = sys.argv[2], sys.argv[3]
        rows = list(csv.reader(open(path)))
        hi = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
        h = rows[hi]
        agg = defaultdict(lambda: [0, 0.0])
        for r in rows[hi + 1:]:
            try:
                v = float(r[h.index("Metric Value")].replace(",", ""))
            except (ValueError, IndexError):
                continue
            name = r[h.index("Kernel Name")]
            agg[name][0] += 1
            agg[name][1] += v
        tot = sum(v[1] for v in agg.values())
        with open(out, "w") as f:
            f.write(f"# per-kernel device time from {path} (ncu gpu__time_duration.sum, serialised, cold cache)\n")
            f.write("# total_ms share launches kernel\n")
            for name, (c, v) in sorted(agg.items(), key=lambda x: -x[1][1]):
                f.write(f"{v / 1e6:10.3f} {100 * v / tot:6.2f}% {c:6d}  {name[:140]}\n")
        return
    out = sys.argv[1]
    with open(out, "w") as f:
        for rep in sys.argv[2:]:
            h, units, rows = raw(rep)
            for idx, r in enumerate(rows):
                f.write(f"## {rep.split('/')[-1]} — {r[h.index('Kernel Name')][:120]}\n\n")
                for m, label in METRICS:
                    if m in h:
                        f.write(f"- {label}: {r[h.index(m)]} {units[h.index(m)]}\n")
                f.write("\nTop SASS stall sites (share of warp-stall samples, executions, instruction):\n\n")
                for share, inst, src in top_stalls(rep, idx):
                    f.write(f"- {share:5.1f}%  x{inst}  `{src[:90]}`\n")
                f.write("\n")


if __name__ == "__main__":
    main()
