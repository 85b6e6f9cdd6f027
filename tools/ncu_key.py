"""Key metrics of each kernel in an ncu report (duration, DRAM bytes, instructions, issue, SMEM
bank conflicts, pipe utilisation).  usage: python tools/ncu_key.py report.ncu-rep"""
import csv, io, subprocess, sys
out = subprocess.run(["ncu", "-i", sys.argv[1], "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
h = rows[0]
want = ["Kernel Name", "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "smsp__inst_executed.sum",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active", "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum",
        "smsp__thread_inst_executed_per_inst_executed.ratio", "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
        "smsp__inst_executed_op_shared_atom.sum", "smsp__inst_executed_op_global_atom.sum", "smsp__inst_executed_op_global_red.sum",
        "smsp__sass_inst_executed_op_shared_atom.sum", "smsp__sass_inst_executed_op_global_atom.sum", "smsp__sass_inst_executed_op_global_red.sum",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed"]
idx = {n: h.index(n) for n in want if n in h}
for r in rows[2:]:
    for n, i in idx.items():
        print(f"{n:60s} {rows[1][i]:>10s} {r[i]}")
    print()
