"""Atomics ablation on B200 (§V.E, Fig. 8
right L1093-1120): time the plain Fig. 4 count kernel with each bucket
increment strategy over inputs with d distinct values, n = 2^28 fp32, b = 256.

    python scripts/atomics_ablation.py [--log2n 28] [--b 256] [--reps 5] [--out FILE]

Inputs are generated on the device (torch): d = 1 (all 42.0), d in {16, 128,
1024} (uniform choice of the values 0..d-1 as floats), d = n (U[0,1)).  The
tree comes from the library's own sample + tree steps.  Prints one JSON line
per (d, mode) and a markdown table; every mode's totals are checked equal to
the first mode's (parity against the oracle is tests/test_gpu_ablation.py).
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch
    import paper_conf_ipps_ribizela19_b200 as ss
    p = argparse.ArgumentParser()
    p.add_argument("--log2n", type=int, default=28)
    p.add_argument("--b", type=int, default=256)
    p.add_argument("--reps", type=int, default=5)
    p.add_argument("--out", default="")
    a = p.parse_args()
    n, b = 1 << a.log2n, a.b
    ctx = ss.Context(0)
    g = torch.Generator(device="cuda:0").manual_seed(77)
    modes = ["shared", "shared_wa", "shared_fig6", "global", "global_wa"]
    rows = []
    for d in [1, 16, 128, 1024, n]:
        if d == 1:
            x = torch.full((n,), 42.0, device="cuda:0")
        elif d == n:
            x = torch.rand(n, device="cuda:0", generator=g)
        else:
            x = torch.randint(0, d, (n,), device="cuda:0", generator=g).float()
        keys = torch.empty(4096, dtype=torch.int32, device="cuda:0")
        ctx.step_sample(x, 0, 0, 4096, keys)
        tree = torch.empty(b - 1, dtype=torch.int32, device="cuda:0")
        spl = torch.empty(b - 1, dtype=torch.int32, device="cuda:0")
        eq = torch.empty(b, dtype=torch.uint8, device="cuda:0")
        ctx.step_tree(0, keys, b, True, tree, spl, eq)
        ref = None
        for mode in modes:
            tot = torch.zeros(b, dtype=torch.int64, device="cuda:0")
            for _ in range(2):
                ctx.step_count_ablation(x, tree, b, mode, tot)
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            st = torch.cuda.current_stream()
            ms = []
            for _ in range(a.reps):
                e0.record(st)
                ctx.step_count_ablation(x, tree, b, mode, tot)
                e1.record(st)
                torch.cuda.synchronize()
                ms.append(e0.elapsed_time(e1))
            t = tot.cpu()
            assert int(t.sum()) == n
            if ref is None:
                ref = t
            assert torch.equal(t, ref), (d, mode)
            best = min(ms)
            row = {"d": d, "mode": mode, "b": b, "n": n, "ms_min": best, "ms_mean": sum(ms) / len(ms),
                   "elem_per_s": n / (best * 1e-3), "gbs": 4 * n / (best * 1e-3) / 1e9,
                   "max_bucket_frac": float(t.max()) / n}
            rows.append(row)
            print(json.dumps(row), flush=True)
        del x
        torch.cuda.empty_cache()
    ctx.close()
    print("\n| d | " + " | ".join(modes) + " |")
    print("|---|" + "---|" * len(modes))
    for d in sorted({r["d"] for r in rows}):
        cells = [f"{r['ms_min'] * 1e3:.0f} us ({r['gbs']:.0f} GB/s)" for m in modes for r in rows
                 if r["d"] == d and r["mode"] == m]
        print(f"| {'n' if d == n else d} | " + " | ".join(cells) + " |")
    if a.out:
        with open(a.out, "w") as f:
            json.dump(rows, f, indent=1)


if __name__ == "__main__":
    main()
