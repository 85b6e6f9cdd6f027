"""quick WC check with the L2 tables forced on (BMR_TABLE_MIN_BYTES=0): pages from argv"""
import os, sys, time
os.environ.setdefault("BMR_TABLE_MIN_BYTES", "0")
sys.path.insert(0, os.getcwd())
import numpy as np, torch
import paper_conf_ipps_jim11_b200 as bmr
from gen import pygen
from oracle import oracle
from tests.helpers import decode
pages = int(sys.argv[1]) if len(sys.argv) > 1 else 4
g = pygen.host_text(pygen.spec_wc(1_000_000, 5), pages)
d = torch.from_numpy(g["data"]).cuda(); o = torch.from_numpy(g["offsets"].view(np.int64)).cuda()
t0 = time.time()
with bmr.Job("wc") as job:
    job.map(d, o, g["n"]); print("mapped", flush=True)
    job.group(); print("grouped", time.time() - t0, flush=True)
    job.reduce(); r = job.fetch(); st = job.stats()
got = decode("wc", r); exp = decode("wc", oracle.run("wc", [(g["data"], g["offsets"], g["n"], 0, 0)]))
print("equal", got == exp, len(got), len(exp), {k: st[k] for k in ("pairs", "words_combined", "pairs_hashed", "replays")})
if got != exp:
    diff = [k for k in set(got) | set(exp) if got.get(k) != exp.get(k)][:10]
    print([(k, got.get(k), exp.get(k)) for k in diff])
