"""Regenerate the bench table of profiles/r01/SUMMARY.md from the committed bench lines
(between the <!-- table --> markers)."""
import json
import os
import re

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
D = os.path.join(ROOT, "profiles", "r01")
NAMES = {"C5": "WordCount 8 GiB, Zipf V=1M", "C2": "StringMatch 4 GiB", "C3": "KMeans 64M x 8 fp32, k=32",
         "C4": "InvertedIndex 8 GiB"}


def main():
    rows = ["| cfg | workload | GB/s (input) | ms/step | dominant kernel (share of step) | achieved GB/s | frac of "
            "measured HBM | ncu DRAM bytes / launch | e2e GB/s (host buffers) | CPU oracle GB/s (1 core) |",
            "|---|---|---|---|---|---|---|---|---|---|"]
    for w in ("C5", "C2", "C3", "C4"):
        d = json.load(open(os.path.join(D, f"bench_{w}.json")))
        r = d["roofline"]
        tr = f"{r['traffic'] / 1e9:.2f} G" if r.get("traffic") else "—"
        rows.append(f"| {w} | {NAMES[w]} | {d['value']:.1f} | {d['ms_per_step']:.2f} | {r['kernel']} "
                    f"({r.get('share_of_step', 0):.2f}) | {r['achieved']:.0f} | {r['frac']:.3f} | {tr} | "
                    f"{d['e2e']['value']:.1f} | {d['cpu_baseline']['value']:.4g} |")
    p = os.path.join(D, "SUMMARY.md")
    s = open(p).read()
    s = re.sub(r"<!-- table -->.*<!-- /table -->", "<!-- table -->\n" + "\n".join(rows) + "\n<!-- /table -->", s,
               flags=re.S)
    open(p, "w").write(s)
    print("\n".join(rows))


if __name__ == "__main__":
    main()
