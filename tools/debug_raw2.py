import sys, numpy as np, torch
sys.path.insert(0, '.')
import paper_conf_ipps_jim11_b200 as bmr
from gen import pygen
from tests.test_gpu_multirank import shards_text
spec = pygen.spec_wc(1_000_000, 5)
for flags, R in [(0, 1), (0, 2), (bmr.FLAG_NO_COMBINE, 1), (bmr.FLAG_NO_COMBINE, 1), (bmr.FLAG_NO_COMBINE, 2)]:
    sh = shards_text(spec, 4, R)
    for r in range(R):
        g = sh[r]
        d = torch.from_numpy(g["data"]).cuda(); o = torch.from_numpy(g["offsets"].view(np.int64)).cuda()
        job = bmr.Job("wc", rank=r, nranks=R, flags=flags)
        job.map(d, o, g["n"])
        ent, heap, counts, eb = job.partition()
        torch.cuda.synchronize()
        e = ent.cpu().numpy().view(np.uint64).reshape(-1, 2)
        klen = e[:, 0] & 0xFFFF
        st = job.stats()
        print(flags, R, r, "entries", len(e), "klen0", int((klen == 0).sum()), "pairs", st["pairs"], "flushes", st["flushes"], "cap", st["capacity_pairs"])
        job.close()
