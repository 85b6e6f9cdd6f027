"""Write profiles/traffic.json: DRAM bytes (dram__bytes_read.sum + dram__bytes_write.sum) per
launch of the dominant kernels, from `ncu --set full` captures brought back in gpurun_out/.

usage: python tools/make_traffic.py OUT.json WORKLOAD=report.ncu-rep|export-prefix [WORKLOAD=... ...]
(bench.py reads OUT.json for the roofline `traffic` field; the report names are recorded)."""
import csv
import io
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from ncu_csv import page  # noqa: E402  (a report, or the CSV export prefix of tools/r03/ncu_export.sh)


def launches(rep):
    rows = list(csv.reader(io.StringIO(page(rep, "raw"))))
    hi = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    rows = rows[hi:]
    h = rows[0]
    iname, ir, iw = h.index("Kernel Name"), h.index("dram__bytes_read.sum"), h.index("dram__bytes_write.sum")
    units = rows[1]
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
    for r in rows[2:]:
        rd = float(r[ir].replace(",", "")) * scale[units[ir]]
        wr = float(r[iw].replace(",", "")) * scale[units[iw]]
        yield r[iname], rd + wr


def main():
    out = sys.argv[1]
    res = json.load(open(out)) if os.path.exists(out) else {}
    for arg in sys.argv[2:]:
        wl, rep = arg.split("=", 1)
        agg = {}
        for name, b in launches(rep):
            key = "k_onesweep" if "k_onesweep" in name else "k_map" if "k_map" in name else None
            if key:
                agg.setdefault(key, []).append(b)
        for key, v in agg.items():
            res.setdefault(wl, {})[key] = {"bytes_per_launch": int(sum(v) / len(v)), "launches": len(v),
                                           "source": os.path.basename(rep)}
    json.dump(res, open(out, "w"), indent=1, sort_keys=True)
    print(json.dumps(res, indent=1))


if __name__ == "__main__":
    main()
