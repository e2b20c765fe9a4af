#!/usr/bin/env python
"""Benchmark of the B200 SampleSelect hot path (BASELINE.json metric:
exact-select elements/s & % of HBM roofline, n=2^28 fp32, 1/2/4/8 B200).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
    torchrun --nproc-per-node N --master-addr 127.0.0.1 bench.py --gpus N ...

A step is one exact selection (the whole hot path: sample/tree, classify+
count, prefix/search, filter, recursion, base case) of rank k over n = 2^28
uniform fp32 elements resident in HBM, through the C ABI, result returned to
the host.  Inputs are 1 GiB (> 126 MB L2), so no L2 flush is needed between
steps.  Prints ONE JSON line on rank 0.

--impl reference times the CPU oracle (test infrastructure: sort-and-index)
on bounded samples of the same workload on the host cores.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

METRIC = "exact-select elements/s & % of HBM roofline, n=2^28 fp32, 1/2/4/8 B200"
UNIT = "elements/s"


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=50)
    p.add_argument("--warmup", type=int, default=5)
    p.add_argument("--impl", choices=["ours", "reference"], default="ours")
    p.add_argument("--log2n", type=int, default=28, help="elements per GPU = 2^log2n")
    p.add_argument("--dtype", default="float32", choices=["float32", "float64", "int32", "int64"])
    p.add_argument("--kind", default="uniform")
    p.add_argument("--mode", default="exact", choices=["exact", "approx", "upper", "multi", "quick"],
                   help="upper: top-k fusion (select + all larger elements, §IV.I), k = n - --upper-count")
    p.add_argument("--upper-count", type=int, default=1 << 20, help="upper mode: n - k elements returned")
    p.add_argument("--ranks", type=int, default=8, help="multi mode: number of ranks (seeded, uniform)")
    p.add_argument("--b", type=int, default=0, help="buckets (exact default 256, approx 1024)")
    p.add_argument("--e2e-steps", type=int, default=0, help="host-buffer steps (default: min(steps, 10))")
    p.add_argument("--cpu-seconds", type=float, default=10.0, help="CPU-oracle baseline budget")
    p.add_argument("--no-cpu", action="store_true")
    p.add_argument("--classify", type=int, default=0, help="0 auto (cell LUT where it applies), 1 tree walk")
    p.add_argument("--events", default="separate", choices=["timed", "separate"],
                   help="CUDA events around K2 inside the timed loop (timed: they break the PDL overlap "
                        "of the kernel chain) or in a second timed pass of the same length (separate)")
    return p.parse_args()


# ---------------------------------------------------------------- helpers --
def measured_peak():
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(path) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, b.copy_(a) read+write)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md: 6.65 TB/s)"


class ClockSampler:
    """NVML sampling of SM clock + throttle reasons during the timed region."""

    REASONS = {
        "gpu_idle": 0x1, "applications_clocks_setting": 0x2, "sw_power_cap": 0x4,
        "hw_slowdown": 0x8, "sync_boost": 0x10, "sw_thermal_slowdown": 0x20,
        "hw_thermal_slowdown": 0x40, "hw_power_brake_slowdown": 0x80,
        "display_clock_setting": 0x100,
    }

    def __init__(self, device: int, period_s: float = 0.001):
        self.device, self.period = device, period_s
        self.samples, self.reasons, self.max_mhz = [], set(), None
        self._stop = threading.Event()
        self._t = None
        self.ok = False
        try:
            import pynvml
            pynvml.nvmlInit()
            # CUDA_VISIBLE_DEVICES remaps indices; match by UUID
            import torch
            h = None
            uuid = getattr(torch.cuda.get_device_properties(device), "uuid", None)
            if uuid is not None:
                try:
                    h = pynvml.nvmlDeviceGetHandleByUUID(("GPU-" + str(uuid)).encode())
                except Exception:
                    h = None
            if h is None:
                vis = os.environ.get("CUDA_VISIBLE_DEVICES")
                idx = int(vis.split(",")[device]) if vis else device
                h = pynvml.nvmlDeviceGetHandleByIndex(idx)
            self._nv, self._h = pynvml, h
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(h, pynvml.NVML_CLOCK_SM)
            self.ok = True
        except Exception as e:  # pragma: no cover
            self.err = str(e)

    def _run(self):
        nv, h = self._nv, self._h
        while not self._stop.is_set():
            try:
                self.samples.append(nv.nvmlDeviceGetClockInfo(h, nv.NVML_CLOCK_SM))
                r = nv.nvmlDeviceGetCurrentClocksEventReasons(h)
                for name, bit in self.REASONS.items():
                    if r & bit and name != "gpu_idle":
                        self.reasons.add(name)
            except Exception:
                pass
            time.sleep(self.period)

    def __enter__(self):
        if self.ok:
            self._t = threading.Thread(target=self._run, daemon=True)
            self._t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self._t:
            self._t.join()

    def summary(self):
        if not self.ok or not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons),
                    "samples": len(self.samples)}
        return {"sm_mhz": statistics.median(self.samples), "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons), "samples": len(self.samples)}


def cpu_oracle_baseline(x: np.ndarray, budget_s: float):
    """The oracle as it stands (qsort sort-and-index, 1 thread) on a bounded
    sample: the first min(n, 2^24) elements of the same input."""
    import oracle
    m = min(x.size, 1 << 24)
    sample = np.ascontiguousarray(x[:m])
    oracle.build()
    runs, t0 = 0, time.perf_counter()
    while True:
        oracle.select(sample, m // 2)
        runs += 1
        el = time.perf_counter() - t0
        if el >= budget_s or runs >= 100:
            break
    return {"value": runs * m / el, "unit": UNIT, "cores": 1, "kind": "oracle",
            "sample": f"oracle.select (qsort sort-and-index, 1 thread) on the first {m} elements "
                      f"of the same input, k={m // 2}, {runs} run(s), {el:.1f} s"}


def make_input(args, rank: int):
    import datagen
    n = 1 << args.log2n
    seed = datagen.dataset_seed(5, 0) + 7919 * rank
    x = datagen.make(args.kind, n, np.dtype(args.dtype), seed)
    return x


# ------------------------------------------------------------- reference --
def run_reference(args, rank, world):
    if rank != 0:
        return 0
    x = make_input(args, 0)
    import oracle
    oracle.build()
    m = min(x.size, 1 << 22)
    sample = np.ascontiguousarray(x[:m])
    kind = args.mode
    b = args.b or (256 if kind == "exact" else 1024)

    def step():
        if kind in ("exact", "quick"):
            oracle.select(sample, m // 2)
        elif kind == "upper":
            oracle.select_upper(sample, m - min(args.upper_count, m))
        else:
            oracle.approx_select(sample, m // 2, b, oracle.sample_size(b), 0x5A17)
    for _ in range(args.warmup):
        step()
    t0 = time.perf_counter()
    for _ in range(args.steps):
        step()
    el = time.perf_counter() - t0
    value = args.steps * m / el
    cfg = {"workload": f"{kind} select n=2^{args.log2n} {args.dtype} {args.kind}, k=n/2",
           "n": 1 << args.log2n, "sample_elements_per_step": m}
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * el / args.steps,
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": _dt_name(args.dtype),
        "data": "synthetic", "config": cfg,
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": 1, "kind": "oracle",
                         "sample": f"oracle {dict(exact='select', upper='select_upper').get(kind, 'approx_select')} "
                                   f"(CPU, 1 thread) on the first {m} elements of the workload per step"},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


def _dt_name(d):
    return {"float32": "f32", "float64": "f64", "int32": "i32", "int64": "i64"}[d]


# ------------------------------------------------------------------- ours --
def run_ours(args, rank, world, local_rank):
    import torch
    import paper_conf_ipps_ribizela19_b200 as ss

    dev = local_rank
    torch.cuda.set_device(dev)
    x = make_input(args, rank)
    n = x.size
    xh = torch.from_numpy(x).pin_memory()
    xd = xh.to(f"cuda:{dev}", non_blocking=False)
    torch.cuda.synchronize()
    ctx = ss.Context(dev)
    if args.classify:
        ctx.configure(classify=args.classify)
    upper = args.mode == "upper"
    multi = args.mode == "multi"
    quick = args.mode == "quick"
    exact = args.mode in ("exact", "upper", "multi", "quick")
    b = args.b or (256 if exact else 1024)
    if exact:
        ctx.configure(b_exact=b)
    if world > 1:
        from paper_conf_ipps_ribizela19_b200 import sharded
        group_n = n * world
        k = group_n // 2
        sel = sharded.ShardedSelect(sharded.CudaSteps(ctx), sharded.TorchDistComm(), b=b)

        def step(inp):
            return sel.select(inp, k)
    elif multi:
        ks = np.random.default_rng(12345).integers(0, n, args.ranks).tolist()
        k = ks[0]

        def step(inp):
            return ctx.select_multi(inp, ks)
    elif quick:
        k = n // 2

        def step(inp):
            return ctx.quickselect(inp, k)
    elif upper:
        k = n - args.upper_count
        outbuf = torch.empty(args.upper_count, dtype=xd.dtype, device=xd.device)

        def step(inp):
            return ctx.select_upper(inp, k, out=outbuf)
    else:
        k = n // 2
        if exact:
            def step(inp):
                return ctx.select(inp, k)
        else:
            def step(inp):
                return ctx.approx_select(inp, k, b)

    stream = torch.cuda.current_stream(dev)

    def barrier():
        if world > 1:
            torch.distributed.barrier()

    # ---- warm-up
    for _ in range(max(3, args.warmup)):
        step(xd)
    torch.cuda.synchronize()

    # ---- timed region.  profile=2: the library records CUDA events around
    # the dominant kernel (level-0 count) on the call's stream and accumulates
    # its device time over the timed calls (read once afterwards, so nothing
    # but the select calls runs between steps).
    ctx.configure(profile=2 if args.events == "timed" else 0)
    ctx.profile_totals(reset=True)
    barrier()
    torch.cuda.synchronize()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with ClockSampler(dev) as clk:
        ev0.record(stream)
        for _ in range(args.steps):
            step(xd)
        ev1.record(stream)
        torch.cuda.synchronize()
    barrier()
    ms = ev0.elapsed_time(ev1) / args.steps
    prof_timed = ctx.profile_totals(reset=True)
    upper_ms = []
    if args.events == "separate":
        ctx.configure(profile=2)
        for _ in range(args.steps):
            step(xd)
            if upper:
                upper_ms.append(ctx.stats()["ms_upper_gather"])
        torch.cuda.synchronize()
        prof_timed = ctx.profile_totals(reset=True)
    # per-kernel breakdown (all kernels timed; separate, informational pass)
    ctx.configure(profile=1)
    for _ in range(min(args.steps, 10)):
        step(xd)
    torch.cuda.synchronize()
    prof = ctx.profile_totals(reset=True)
    last = ctx.stats()
    ctx.configure(profile=0)

    def kavg(level, q, pr=None):
        pr = pr or prof
        cnt = pr["count"][level][q]
        return pr["ms_sum"][level][q] / cnt if cnt else 0.0
    if world > 1:
        t = torch.tensor([ms], device=f"cuda:{dev}", dtype=torch.float64)
        torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
        ms = float(t.item())
    total_elems = n * world
    value = total_elems / (ms * 1e-3)

    # ---- end-to-end through the public API with HOST buffers
    e2e_steps = args.e2e_steps or min(args.steps, 10)
    xhn = xh.numpy()
    if world == 1 and not upper and not multi and not quick:
        step_h = (lambda: ctx.select(xhn, k)) if exact else (lambda: ctx.approx_select(xhn, k, b))
        step_h()
        torch.cuda.synchronize()
        t0 = torch.cuda.Event(enable_timing=True)
        t1 = torch.cuda.Event(enable_timing=True)
        t0.record(stream)
        for _ in range(e2e_steps):
            step_h()
        t1.record(stream)
        torch.cuda.synchronize()
        e2e_ms = t0.elapsed_time(t1) / e2e_steps
        est = ctx.stats()
        e2e = {"value": total_elems / (e2e_ms * 1e-3), "unit": UNIT,
               "h2d_bytes_per_step": int(est["h2d_bytes"]), "d2h_bytes_per_step": int(est["d2h_bytes"]),
               "ms_per_step": e2e_ms, "steps": e2e_steps}
    else:
        e2e = None

    if rank != 0:
        return 0

    # ---- roofline of the dominant kernel (level 0's count pass).  Exact
    # selection at this size runs the fused filter on level 0 (window_kernel:
    # reads the level once, writes the window = the next level); otherwise
    # the paper's count kernel (reads the level, writes one oracle byte per
    # element when exact).  Bytes per launch: DESIGN.md §7.
    peak, peak_src = measured_peak()
    S = np.dtype(args.dtype).itemsize
    fused0 = exact and bool(last.get("fused_levels", 0) & 1)
    if multi or quick:
        kname = ("whole call (shared sample + count, bucket extractions, per-rank tails)" if multi else
                 "whole call (QuickSelect baseline: per level pivot + partition + decide, SURVEY NEXT-3)")
        k2_bytes = float(last["bytes_algorithmic"])
        tkey = f"{args.mode}_{args.dtype}_2p{args.log2n}"
    elif upper:
        kname = "upper_gather_kernel (top-k pass: read the input, write the elements > result)"
        k2_bytes = S * n + S * int(last["upper_greater"])
        tkey = f"upper_{args.dtype}_2p{args.log2n}"
    elif fused0:
        kname = "window_kernel (fused count + filter, level 0)"
        k2_bytes = S * n + S * int(last["n_level"][1])
        tkey = f"window_{args.mode}_{args.dtype}_2p{args.log2n}"
    else:
        kname = "count_kernel (K2, level 0)"
        k2_bytes = (S + (1 if exact else 0)) * n          # read S*n, write n oracle bytes
        tkey = f"count_{args.mode}_{args.dtype}_2p{args.log2n}"
    k2_avg = float(np.mean(upper_ms)) if upper and upper_ms else (ms if multi or quick else kavg(0, 1, prof_timed))
    achieved = k2_bytes / (k2_avg * 1e-3) / 1e9
    traffic = None
    tpath = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(tpath):
        try:
            with open(tpath) as f:
                traffic = json.load(f).get(tkey)
        except Exception:
            traffic = None
    path_bytes = float(last["bytes_algorithmic"])
    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": max(3, args.warmup), "ms_per_step": ms, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": _dt_name(args.dtype), "data": "synthetic",
        "config": {"workload": f"{args.mode} select n=2^{args.log2n} {args.dtype} {args.kind} per GPU, "
                               + (f"k=N-{args.upper_count} (+ all larger elements), b={b}" if upper else
                                  f"{args.ranks} seeded uniform ranks in one call, b={b}" if multi else
                                  "k=N/2, one median-of-256-sample pivot per level" if quick else f"k=N/2, b={b}"),
                   "n_per_gpu": n, "k": k, "b": b, "kind": args.kind,
                   "l2": "inputs larger than L2 (1 GiB input vs 126 MB L2); no flush"},
        "roofline": {"bound": "hbm", "kernel": kname, "achieved": achieved,
                     "peak": peak, "unit": "GB/s", "frac": achieved / peak, "traffic": traffic,
                     "peak_source": peak_src, "algorithmic_bytes": k2_bytes, "avg_ms": k2_avg,
                     "share_of_step": k2_avg / ms,
                     "events": ("CUDA events around the kernel on the call's stream, inside the timed loop"
                                if args.events == "timed" else
                                f"CUDA events around the kernel on the call's stream, over a second timed pass of "
                                f"{args.steps} steps right after the headline loop (events between the "
                                f"kernels would break their PDL overlap in the headline loop)")},
        "path_roofline": {"algorithmic_bytes_per_step": path_bytes,
                          "achieved_gbs": path_bytes / (ms * 1e-3) / 1e9,
                          "frac_of_peak": path_bytes / (ms * 1e-3) / 1e9 / peak,
                          "frac_of_8tbs": path_bytes / (ms * 1e-3) / 8e12},
        "kernels_ms": {"avg_per_level": [[kavg(l, q) for q in range(3)] for l in range(last["levels"] + 1)],
                       "sum_of_kernels": sum(kavg(l, q) for l in range(last["levels"] + 1) for q in range(3)),
                       "levels": last["levels"], "n_level": last["n_level"]},
        "gpu_launches": int(prof_timed["launches"]),
        "clocks": clk.summary(),
        "e2e": e2e,
    }
    if not args.no_cpu and world == 1:
        line["cpu_baseline"] = cpu_oracle_baseline(x, args.cpu_seconds)
    print(json.dumps(line), flush=True)
    ctx.close()
    return 0


def main():
    args = parse()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        return run_reference(args, rank, world)
    if world > 1:
        import torch
        torch.cuda.set_device(local_rank)
        torch.distributed.init_process_group("nccl", device_id=torch.device(f"cuda:{local_rank}"))
    try:
        return run_ours(args, rank, world, local_rank)
    finally:
        if world > 1:
            import torch
            torch.distributed.destroy_process_group()


if __name__ == "__main__":
    sys.exit(main())
