import sys, numpy as np, torch
sys.path.insert(0, '.')
import paper_conf_ipps_jim11_b200 as bmr
from gen import pygen
spec = pygen.spec_wc(1_000_000, 5)
g = pygen.host_text(spec, 4)
d = torch.from_numpy(g["data"]).cuda(); o = torch.from_numpy(g["offsets"].view(np.int64)).cuda()
job = bmr.Job("wc", rank=0, nranks=1, flags=bmr.FLAG_NO_COMBINE)
job.map(d, o, g["n"])
ent, heap, counts, eb = job.partition()
torch.cuda.synchronize()
e = ent.cpu().numpy().view(np.uint64).reshape(-1, 2)
klen = e[:, 0] & 0xFFFF
print("entries", len(e), "counts", counts.tolist(), "klen0", int((klen == 0).sum()), "v!=1", int((e[:, 1] != 1).sum()))
print("stats", job.stats())
job2 = bmr.Job("wc")
job2.map(d, o, g["n"]); job2.group()
print("stats plain", job2.stats())
