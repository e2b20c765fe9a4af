"""Debug driver: one sharded call on virtual ranks (for compute-sanitizer runs).
python scripts/dbg_sharded.py <case> <P> [gather_log2]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import numpy as np
import oracle
from test_sharded_gpu import _run, _shards, _bits
case = sys.argv[1] if len(sys.argv) > 1 else "empty"
P = int(sys.argv[2]) if len(sys.argv) > 2 else 2
g = int(sys.argv[3]) if len(sys.argv) > 3 else 14
n = (1 << 20) // P + 17
shards = _shards(case, P, n, np.float32, seed=100 + P)
full = np.concatenate(shards)
ks = [full.size // 2]
out, stats = _run(shards, ks, P, shard_gather_log2=g)
print(out, _bits(oracle.select(full, ks[0])), stats[0][0]["n_level"][:6], stats[0][0]["shard_levels"])
