"""Latency probe of the small kernels (K1 sample/sort/tree, base case, small levels).
Not part of the product; prints per-kernel device times."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import datagen
import paper_conf_ipps_ribizela19_b200 as ss

ctx = ss.Context(0)
dev = "cuda:0"


def ev_time(fn, reps=200):
    fn(); torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(reps):
        fn()
    b.record(); torch.cuda.synchronize()
    return a.elapsed_time(b) / reps * 1e3


x = torch.from_numpy(datagen.uniform(1 << 28, np.float32, seed=5)).to(dev)
for s in (1024, 4096, 16384):
    keys = torch.empty(s, dtype=torch.int32, device=dev)
    t_s = ev_time(lambda: ctx.step_sample(x, 0, 0, s, keys))
    tree = torch.empty(1024, dtype=torch.int32, device=dev)
    spl = torch.empty(1024, dtype=torch.int32, device=dev)
    eq = torch.empty(1024, dtype=torch.uint8, device=dev)
    for b in (64, 256):
        t_t = ev_time(lambda: ctx.step_tree(0, keys, b, True, tree, spl, eq))
        print(f"s={s:5d} b={b:4d}: sample (grid kernel) {t_s:7.1f} us   sort+tree (1 CTA) {t_t:7.1f} us", flush=True)

ctx.configure(profile=1)
for n in (1000, 3712, 16384, 1 << 17, 1 << 20, 1 << 22):
    xs = x[:n].clone()
    for _ in range(3):
        ctx.select(xs, n // 2)
    torch.cuda.synchronize()
    ctx.profile_totals(reset=True)
    t0 = time.perf_counter()
    R = 50
    for _ in range(R):
        ctx.select(xs, n // 2)
    wall = (time.perf_counter() - t0) / R * 1e6
    pr = ctx.profile_totals(reset=True)
    st = ctx.stats()
    per = [[round(pr["ms_sum"][l][q] / max(1, pr["count"][l][q]) * 1e3, 1) for q in range(3)] for l in range(st["levels"] + 1)]
    print(f"n={n:8d}: wall/call {wall:7.1f} us levels={st['levels']} n_level={st['n_level']} per-kernel us={per}", flush=True)
ctx.configure(profile=0)
for n in (1000, 3712, 16384, 1 << 17, 1 << 20, 1 << 22):
    xs = x[:n].clone()
    for _ in range(3):
        ctx.select(xs, n // 2)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    R = 50
    for _ in range(R):
        ctx.select(xs, n // 2)
    wall = (time.perf_counter() - t0) / R * 1e6
    print(f"profile=0 n={n:8d}: wall/call {wall:7.1f} us", flush=True)
