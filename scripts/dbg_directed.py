"""Debug: int / top_run cases through the directed levels (R28), stats per call."""
import numpy as np, torch, sys, json
sys.path.insert(0, ".")
import paper_conf_ipps_ribizela19_b200 as ss
import datagen
import oracle as osel
def bits(v):
    a = np.asarray(v); return int(a.view(np.uint32 if a.itemsize == 4 else np.uint64))
for dt in (np.int32, np.int64):
    n = 4194311
    x = datagen.int_uniform(n, dt, seed=n % 1000)
    xd = torch.from_numpy(x).cuda()
    for d in (1, 0):
        c = ss.Context(0, directed=d)
        for k in (0, 1, n // 2, n - 1):
            v = c.select(xd, k)
            st = c.stats()
            ok = bits(v) == bits(osel.select(x, k))
            print(dt.__name__, "dir", d, "k", k, "ok", ok, json.dumps({q: st[q] for q in ("levels", "equality_exit", "n_level", "spec_levels", "fused_levels", "incomplete_rounds")}))
        c.close()
