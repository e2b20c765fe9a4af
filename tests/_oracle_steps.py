"""CPU reference implementation of the sharded driver's Steps interface,
built from the oracle (test infrastructure only).  Lets the host protocol of
paper_conf_ipps_ribizela19_b200.sharded run under gloo without a GPU."""
import numpy as np
import torch

import oracle


class OracleSteps:
    def __init__(self, seed: int = 0x5A17):
        self.seed = seed

    def sample(self, x, level, slot_begin, count):
        a = x.numpy()
        if count == 0 or a.size == 0:
            return torch.from_numpy(a[:0].copy())
        idx = oracle.sample_indices(self.seed, level, a.size, slot_begin, count)
        return torch.from_numpy(a[idx].copy())

    def tree(self, x_like, keys, b):
        spl = oracle.pick_splitters(keys.numpy(), b)
        fixed, eq = oracle.equality_fixup(spl)
        return torch.from_numpy(oracle.heap_tree(fixed)), torch.from_numpy(fixed), torch.from_numpy(eq)

    def count(self, x, tree, b):
        a = x.numpy()
        if a.size == 0:
            return torch.zeros(b, dtype=torch.int64), np.zeros(0, np.uint8)
        counts, orc = oracle.count_buckets(a, tree.numpy())
        return torch.from_numpy(counts), orc

    def search(self, totals, b, k, eq):
        t = totals.numpy()
        r = 0
        for j in range(b):
            if r <= k < r + t[j]:
                return j, k - r, int(t[j]), bool(eq.numpy()[j])
            r += t[j]
        raise AssertionError("rank outside the totals")

    def filter(self, x, orc, j, expected):
        a = x.numpy()
        out = oracle.filter_bucket(a, orc, j) if a.size else a[:0]
        assert out.size == expected
        return torch.from_numpy(out.copy())

    def splitter_value(self, x_like, spl, j):
        return spl.numpy()[j - 1]

    def select(self, x, k):
        return oracle.select(x.numpy(), k)
