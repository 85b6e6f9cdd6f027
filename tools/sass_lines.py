"""SASS of one kernel grouped by CUDA source line (needs a -lineinfo build).
usage: python tools/sass_lines.py build/map.o KERNEL_SUBSTRING FILE:LO-HI"""
import os
import re
import subprocess
import sys
import tempfile

obj, kname, rng = sys.argv[1], sys.argv[2], sys.argv[3]
fname, span = rng.split(":")
lo, hi = map(int, span.split("-"))
with tempfile.TemporaryDirectory() as d:
    subprocess.run(["cuobjdump", "-xelf", "all", os.path.abspath(obj)], cwd=d, capture_output=True)
    cub = [f for f in os.listdir(d) if f.endswith(".cubin")][0]
    txt = subprocess.run(["nvdisasm", "-g", "-c", os.path.join(d, cub)], capture_output=True, text=True).stdout
inside, cur, n = False, None, 0
for l in txt.split("\n"):
    if l.startswith("//----") and ".text." in l:
        inside = kname in l
        continue
    if not inside:
        continue
    m = re.search(r'//## File ".*/([\w.]+)", line (\d+)', l)
    if m:
        cur = (m.group(1), int(m.group(2)))
        continue
    m = re.match(r"\s+/\*([0-9a-f]+)\*/\s+(.*?);", l)
    if m and cur and cur[0] == fname and lo <= cur[1] <= hi:
        print(f"{m.group(1)} {cur[1]:5d}  {m.group(2).strip()}")
        n += 1
print(f"# {n} instructions", file=sys.stderr)
