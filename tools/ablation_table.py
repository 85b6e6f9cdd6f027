"""Regenerate the table of profiles/r01/ablation.md from an ablation.jsonl (tools/ablation.sh):
Map kernel device time (ms, the library's CUDA events) per config and memory mode."""
import json
import sys

NAMES = {"C5": "C5 WordCount 8 GiB (Zipf V=1M)", "C2": "C2 StringMatch 4 GiB", "C3": "C3 KMeans 64M pts, k=32",
         "C4": "C4 InvertedIndex 8 GiB"}


def main():
    src = sys.argv[1]
    t = {}
    for line in open(src):
        line = line.strip()
        if not line.startswith("{"):
            continue
        d = json.loads(line)
        c = d["config"]
        comb = "n/a" if c["workload"] in ("C2", "C4") else ("on" if c.get("map_combiner", True) else "off")
        t[(c["workload"], comb, c["map_mode"])] = d["phases_ms"]["map"]
    print("| config | combiner | SIO | SO | SI | G | G / SIO |")
    print("|---|---|---|---|---|---|---|")
    for w in ("C5", "C2", "C3", "C4"):
        for comb in ("on", "off", "n/a"):
            row = [t.get((w, comb, m)) for m in ("SIO", "SO", "SI", "G")]
            if row[0] is None:
                continue
            cells = " | ".join(f"{v:.2f}" if v is not None else "—" for v in row)
            ratio = f"{row[3] / row[0]:.2f}x" if row[3] and row[0] else "—"
            print(f"| {NAMES[w]} | {comb} | {cells} | {ratio} |")


if __name__ == "__main__":
    main()
