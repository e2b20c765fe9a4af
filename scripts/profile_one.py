"""Run a few selections for ncu: `python scripts/profile_one.py [log2n] [mode] [b]`
(mode: exact, approx, multi (b = number of ranks), upper (b = log2 of n - k))."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import datagen
import paper_conf_ipps_ribizela19_b200 as ss
log2n = int(sys.argv[1]) if len(sys.argv) > 1 else 28
mode = sys.argv[2] if len(sys.argv) > 2 else "exact"
b = int(sys.argv[3]) if len(sys.argv) > 3 else {"exact": 256, "multi": 8, "upper": 20}.get(mode, 1024)
n = 1 << log2n
x = torch.from_numpy(datagen.uniform(n, np.float32, seed=datagen.dataset_seed(5, 0))).cuda()
import json
ctx = ss.Context(0, **json.loads(os.environ.get('SS_CFG', '{}')))
for _ in range(3):
    if mode == "exact":
        ctx.configure(b_exact=b); v = ctx.select(x, n // 2)
    elif mode == "multi":
        v = ctx.select_multi(x, [datagen.rank(n, 100 + i) for i in range(b)])
    elif mode == "upper":
        v = ctx.select_upper(x, n - (1 << b))[0]
    else:
        v = ctx.approx_select(x, n // 2, b)
torch.cuda.synchronize()
print(v, ctx.stats())
