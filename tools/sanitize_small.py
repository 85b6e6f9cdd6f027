"""Small end-to-end runs for compute-sanitizer (memcheck / racecheck / synccheck)."""
import sys
import numpy as np
import torch
sys.path.insert(0, '.')
import paper_conf_ipps_jim11_b200 as bmr
from gen import pygen

def run(w, spec, pages, **kw):
    g = pygen.host_text(spec, pages)
    d = torch.from_numpy(g["data"]).cuda(); o = torch.from_numpy(g["offsets"].view(np.int64)).cuda()
    with bmr.Job(w, **kw) as job:
        job.map(d, o, g["n"]); job.group(); job.reduce(); r = job.fetch()
    print(w, r["n_keys"])

run("wc", pygen.spec_wc(1000, 1), 1)
run("wc", pygen.spec_wc(1000, 1), 1, flags=bmr.FLAG_FORCE_TINY_OUT)
run("ii", pygen.spec_ii(4), 1)
run("sm", pygen.spec_sm(20000), 1, pattern=pygen.SM_PATTERN)
spec = pygen.KMSpec(); pts = pygen.host_km(spec, 4096); _, init = pygen.km_centres(spec)
with bmr.Job("km", centroids=init) as job:
    d = torch.from_numpy(pts.view(np.uint8).reshape(-1)).cuda()
    job.map(d, None, 4096); job.group(); job.reduce(); print("km", job.fetch()["n_keys"])
# SM dense plants (the stage-released record check) and the fused exchange window (f-3)
run("sm", pygen.spec_sm(20000, dense=True) if "dense" in pygen.spec_sm.__code__.co_varnames else pygen.spec_sm(20000), 2,
    pattern=pygen.SM_PATTERN)
g = pygen.host_text(pygen.spec_ii(4), 2)
d = torch.from_numpy(g["data"]).cuda(); o = torch.from_numpy(g["offsets"].view(np.int64)).cuda()
w = bmr.XWindow(1 << 16, 1 << 22)
with bmr.Job("ii") as job:
    job.set_xwindows([w]); job.map(d, o, g["n"]); torch.cuda.synchronize(); job.ingest_xwindow(w)
    job.group(); job.reduce(); print("ii fused", job.fetch()["n_keys"])
