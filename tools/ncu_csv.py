"""ncu page text from a report (runs `ncu -i`) or from CSVs exported on the GPU box by
tools/r03/ncu_export.sh (a report with source is too large to bring back): pass the report path, or
the export prefix gpurun_out/<tag>/<NAME> (files <NAME>_raw.csv, <NAME>_src.csv.gz, <NAME>_sass.csv.gz)."""
import gzip
import os
import subprocess

_PAGES = {"raw": (["--page", "raw", "--csv"], "_raw.csv"),
          "src": (["--page", "source", "--csv", "--print-source", "cuda,sass"], "_src.csv.gz"),
          "sass": (["--page", "source", "--csv", "--print-source", "sass"], "_sass.csv.gz")}


def page(rep, which, extra=()):
    args, suffix = _PAGES[which]
    if rep.endswith(".ncu-rep"):
        return subprocess.run(["ncu", "-i", rep, *args, *extra], capture_output=True, text=True).stdout
    path = rep + suffix
    if not os.path.exists(path):
        return ""
    opener = gzip.open if path.endswith(".gz") else open
    with opener(path, "rt") as f:
        return f.read()
