import sys, numpy as np, torch
sys.path.insert(0, '.')
import paper_conf_ipps_jim11_b200 as bmr
from gen import pygen
from oracle import oracle
from tests.helpers import decode
from tests.test_gpu_multirank import shards_text, run_virtual, union_dict
spec = pygen.spec_wc(1_000_000, 5)
whole = pygen.host_text(spec, 4)
exp = decode("wc", oracle.run("wc", [(whole["data"], whole["offsets"], whole["n"], 0, 0)]))
for flags, R in [(bmr.FLAG_NO_COMBINE, 1), (0, 1), (0, 2), (bmr.FLAG_NO_COMBINE, 1), (bmr.FLAG_NO_COMBINE, 2), (bmr.FLAG_NO_COMBINE, 1)]:
    sh = shards_text(spec, 4, R)
    got = union_dict(run_virtual("wc", sh, R, flags=flags), "wc")
    bad = {k: (got.get(k), exp.get(k)) for k in set(got) | set(exp) if got.get(k) != exp.get(k)}
    print(flags, R, "keys", len(got), len(exp), "sum", sum(got.values()), sum(exp.values()), "bad", len(bad), "empty", got.get(b''), list(bad.items())[:3])
