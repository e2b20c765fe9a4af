import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import datagen, oracle
import paper_conf_ipps_ribizela19_b200 as ss
for log2n, kw in ((20, dict(spec_min_n=1)), (22, dict(spec_min_n=1)), (26, {})):
    n = (1 << log2n) + 13
    x = datagen.uniform(n, np.float32, seed=21)
    xd = torch.from_numpy(x).cuda()
    c = ss.Context(0, **kw)
    print(log2n, c.config)
    for k in (0, n // 3, n // 2, n - 1):
        v = c.select(xd, k)
        st = c.stats()
        print(k, v, st["n_level"], st["bucket"], "spec", st["spec_levels"], "fused", st["fused_levels"], st["bytes_algorithmic"] / n)
