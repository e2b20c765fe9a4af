#!/usr/bin/env python
"""Benchmark of the B200 SampleSelect hot path (BASELINE.json metric:
exact-select elements/s & % of HBM roofline, n=2^28 fp32, 1/2/4/8 B200).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
    python bench.py --config c1|c2|c3|c4       # BASELINE.json configs 1-4 (one JSON line each)

A step is one exact selection -- the whole hot path: sample + splitter tree,
classify + count, prefix / bucket search, filter, the recursion and the base
case -- of rank k over n = 2^28 uniform fp32 elements per GPU resident in HBM,
through the C ABI, result returned to the host.  N = 1 is the single-GPU path
(ss_select); N > 1 launches one rank per GPU (re-executing itself under
torch.distributed.run when WORLD_SIZE is unset) and runs ss_select_sharded
over NCCL, 2^28 elements per rank (weak scaling).  The headline input is 1 GiB
per GPU (> 126 MB L2): no L2 flush is needed between steps; configs with
inputs <= 2^26 elements flush L2 (a 2x L2 scratch write) between timed steps
and time each step with its own CUDA events.  Rank 0 prints ONE JSON line.

--impl reference times the CPU oracle (test infrastructure: sort-and-index)
on bounded samples of the same workload on the host cores.
"""
from __future__ import annotations

import argparse
import json
import os
import socket
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

METRIC = "exact-select elements/s & % of HBM roofline, n=2^28 fp32, 1/2/4/8 B200"
UNIT = "elements/s"
L2_BYTES = 126 * 1024 * 1024


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=50)
    p.add_argument("--warmup", type=int, default=5)
    p.add_argument("--impl", choices=["ours", "reference"], default="ours")
    p.add_argument("--config", default="headline", choices=["headline", "c1", "c2", "c3", "c4"],
                   help="headline: BASELINE config 5 (2^28 fp32 per GPU); c1..c4: BASELINE configs 1-4")
    p.add_argument("--log2n", type=int, default=28, help="elements per GPU = 2^log2n")
    p.add_argument("--dtype", default="float32", choices=["float32", "float64", "int32", "int64"])
    p.add_argument("--kind", default="uniform")
    p.add_argument("--mode", default="exact", choices=["exact", "approx", "upper", "multi", "quick"],
                   help="upper: top-k fusion (select + all larger elements, §IV.I), k = n - --upper-count")
    p.add_argument("--upper-count", type=int, default=1 << 20, help="upper mode: n - k elements returned")
    p.add_argument("--ranks", type=int, default=8, help="multi mode: number of ranks (seeded, uniform)")
    p.add_argument("--b", type=int, default=0, help="buckets (exact default 256, approx 1024)")
    p.add_argument("--fused", type=int, default=1, help="0: the paper's oracle-byte filter on every level")
    p.add_argument("--rotate", type=int, default=1, help="rotate this many distinct input buffers")
    p.add_argument("--flush", action="store_true", help="flush L2 between timed steps (per-step events)")
    p.add_argument("--e2e-steps", type=int, default=0, help="host-buffer steps (default: min(steps, 10))")
    p.add_argument("--cpu-seconds", type=float, default=10.0, help="CPU-oracle baseline budget")
    p.add_argument("--no-cpu", action="store_true")
    p.add_argument("--cfg", default="", help="extra ss_config fields as JSON, e.g. '{\"upper_onepass\": 0}'")
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


def host_info():
    model = None
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for line in out.splitlines():
            if line.startswith("Model name"):
                model = line.split(":", 1)[1].strip()
    except Exception:
        pass
    return {"nproc": os.cpu_count(), "lscpu_model": model, "OMP_NUM_THREADS": os.environ.get("OMP_NUM_THREADS")}


def cpu_baselines(x: np.ndarray, k: int, budget_s: float):
    """The CPU baselines, timed on this host in the same run:
    (i) the oracle as it stands (qsort sort-and-index, 1 thread) on a bounded
    sample -- the reported `cpu_baseline` -- and, on the FULL input,
    (ii) std::nth_element on 1 core (the paper's reference check, L601-603)
    and (iii) __gnu_parallel::nth_element on all host cores after a warm-up."""
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
    line = {"value": runs * m / el, "unit": UNIT, "cores": 1, "kind": "oracle",
            "sample": f"oracle.select (qsort sort-and-index, 1 thread) on the first {m} elements "
                      f"of the same input, k={m // 2}, {runs} run(s), {el:.1f} s",
            "host": host_info()}
    if x.dtype in (np.float32, np.float64):
        try:
            import cpu_baseline
            t1, v1 = cpu_baseline.nth_element(x, k, parallel=False, reps=1)
            cpu_baseline.nth_element(x[: 1 << 20], 1 << 19, parallel=True, reps=1)   # OpenMP pool start-up
            tp, vp = cpu_baseline.nth_element(x, k, parallel=True, reps=2)
            line["nth_element_1core"] = {"value": x.size / t1, "unit": UNIT, "cores": 1, "seconds": t1,
                                         "sample": f"std::nth_element, full input n={x.size}, k={k}, 1 run"}
            line["gnu_parallel_nth_element"] = {
                "value": x.size / tp, "unit": UNIT, "cores": cpu_baseline.threads(), "seconds": tp,
                "sample": f"__gnu_parallel::nth_element, full input n={x.size}, k={k}, best of 2 after a warm-up"}
            line["nth_element_agrees"] = bool(np.asarray(v1).tobytes() == np.asarray(vp).tobytes())
        except Exception as e:  # pragma: no cover
            line["nth_element_error"] = str(e)
    return line


def make_input(args, rank: int, log2n=None, kind=None, dtype=None, config_id=5, dataset=0):
    import datagen
    n = 1 << (log2n or args.log2n)
    seed = datagen.dataset_seed(config_id, dataset) + 7919 * rank
    return datagen.make(kind or args.kind, n, np.dtype(dtype or args.dtype), seed)


def _dt_name(d):
    return {"float32": "f32", "float64": "f64", "int32": "i32", "int64": "i64"}[str(np.dtype(d))]


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


# ------------------------------------------------------------------- ours --
def _workload_label(args, b, world, levels):
    if args.mode == "upper":
        return f"k=N-{args.upper_count} (+ all larger elements), b={b}"
    if args.mode == "multi":
        return f"{args.ranks} seeded uniform ranks in one call, b={b}"
    if args.mode == "quick":
        return "k=N/2, QuickSelect baseline: one median-of-256-sample pivot per level"
    if args.mode == "approx":
        return f"k=N/2, approximate, one level with b={b} buckets"
    if world > 1:
        return (f"k=N/2 of the union (N = {world} x 2^{args.log2n}), sharded levels: fused window "
                f"(2 splitters from a 4096-key sample) per rank, then gather + single-GPU b={b} levels")
    if args.fused == 0:
        return f"k=N/2, the paper's level on every level: b={b} tree, oracle bytes, filter kernel"
    return (f"k=N/2; level 0: fused window [klo, khi) from a 16384-key sample (two order statistics by "
            f"digit narrowing, K1w) -- one pass counts #{{x < klo}} and copies the window (reading R21); "
            f"deeper fused levels directed by the previous level's 1024-bin key histogram (reading R28); "
            f"levels below 2^16 elements the paper's b={b} tree + oracle-byte filter; base case on an "
            f"8-CTA cluster; level sizes {levels} (a trailing 0: the answer came from a one-key bin, "
            f"an equality exit)")


def run_ours(args, rank, world, local_rank):
    import torch
    import paper_conf_ipps_ribizela19_b200 as ss

    dev = local_rank
    torch.cuda.set_device(dev)
    x = make_input(args, rank)
    n = x.size
    xh = torch.from_numpy(x).pin_memory()
    xds = [xh.to(f"cuda:{dev}", non_blocking=False) for _ in range(max(1, args.rotate))]
    xd = xds[0]
    torch.cuda.synchronize()
    ctx = ss.Context(dev)
    if args.classify:
        ctx.configure(classify=args.classify)
    if not args.fused:
        ctx.configure(fused_filter=0)
    if args.cfg:
        ctx.configure(**json.loads(args.cfg))
    upper = args.mode == "upper"
    multi = args.mode == "multi"
    quick = args.mode == "quick"
    exact = args.mode in ("exact", "upper", "multi", "quick")
    b = args.b or (256 if exact else 1024)
    if exact:
        ctx.configure(b_exact=b)
    if world > 1:
        from paper_conf_ipps_ribizela19_b200.sharded import ShardedSelect
        sel = ShardedSelect(ctx)
        group_n = n * world
        k = group_n // 2

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

    # ---- warm-up (every rotated buffer once)
    for i in range(max(3, args.warmup, len(xds))):
        step(xds[i % len(xds)])
    torch.cuda.synchronize()

    # ---- timed region.  profile=2: the library records CUDA events around
    # the dominant kernel (level-0 count / window) on the call's stream and
    # accumulates its device time over the timed calls (read once afterwards).
    ctx.configure(profile=2 if args.events == "timed" else 0)
    ctx.profile_totals(reset=True)
    barrier()
    torch.cuda.synchronize()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with ClockSampler(dev) as clk:
        ev0.record(stream)
        for i in range(args.steps):
            step(xds[i % len(xds)])
        ev1.record(stream)
        torch.cuda.synchronize()
    barrier()
    ms = ev0.elapsed_time(ev1) / args.steps
    prof_timed = ctx.profile_totals(reset=True)
    launches_timed = prof_timed["launches"]
    upper_ms = []
    if args.events == "separate":
        ctx.configure(profile=2)
        barrier()
        for i in range(args.steps):
            step(xds[i % len(xds)])
            if upper:
                upper_ms.append(ctx.stats()["ms_upper_gather"])
        torch.cuda.synchronize()
        prof_timed = ctx.profile_totals(reset=True)
    # per-kernel breakdown (all kernels timed; separate, informational pass)
    ctx.configure(profile=1)
    barrier()
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

    # ---- end-to-end through the public API with HOST buffers: the step's
    # input goes host -> device inside the timed region, the result comes back
    e2e_steps = args.e2e_steps or min(args.steps, 10)
    xhn = xh.numpy()
    e2e = None
    if not upper and not multi and not quick:
        if world == 1:
            step_h = (lambda: ctx.select(xhn, k)) if exact else (lambda: ctx.approx_select(xhn, k, b))
            h2d_note = "ss_select_host: the call copies the pinned host input to device workspace"
        else:
            def step_h():
                xd.copy_(xh, non_blocking=True)        # this rank's shard, pinned host -> device
                return sel.select(xd, k)
            h2d_note = "each rank copies its pinned host shard to the device, then ss_select_sharded"
        step_h()
        torch.cuda.synchronize()
        barrier()
        t0 = torch.cuda.Event(enable_timing=True)
        t1 = torch.cuda.Event(enable_timing=True)
        t0.record(stream)
        for _ in range(e2e_steps):
            step_h()
        t1.record(stream)
        torch.cuda.synchronize()
        e2e_ms = t0.elapsed_time(t1) / e2e_steps
        if world > 1:
            t = torch.tensor([e2e_ms], device=f"cuda:{dev}", dtype=torch.float64)
            torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
            e2e_ms = float(t.item())
        est = ctx.stats()
        e2e = {"value": total_elems / (e2e_ms * 1e-3), "unit": UNIT,
               "h2d_bytes_per_step": int(x.nbytes) if world > 1 else int(est["h2d_bytes"]),
               "d2h_bytes_per_step": int(est["d2h_bytes"]), "ms_per_step": e2e_ms, "steps": e2e_steps,
               "how": h2d_note}

    if rank != 0:
        ctx.close()
        return 0

    # ---- roofline of the dominant kernel: level 0's fused window (reads the
    # level once, writes the window = the next level) or the paper's count
    # kernel (reads the level, writes one oracle byte per element when exact).
    # Bytes per launch: DESIGN.md §7.  Sharded: this rank's level-0 window.
    peak, peak_src = measured_peak()
    S = np.dtype(args.dtype).itemsize
    fused0 = exact and bool(last.get("fused_levels", 0) & 1)
    if multi or quick:
        kname = ("whole call (shared sample + count, bucket extractions, per-rank tails)" if multi else
                 "whole call (QuickSelect baseline: per level pivot + partition + decide, SURVEY NEXT-3)")
        k2_bytes = float(last["bytes_algorithmic"])
        tkey = f"{args.mode}_{args.dtype}_2p{args.log2n}"
    elif upper and last.get("upper_onepass"):
        # one-pass top-k: level 0 reads the input once, writes its window (the
        # next level) and streams the keys above it to the output; the bytes
        # count every key > result as streamed (the few inside the window are
        # appended by the tail instead: an overcount of at most n_1 elements)
        kname = "window_kernel (one-pass top-k level 0: count + window copy + keys above the window)"
        k2_bytes = S * n + S * int(last["n_level"][1]) + S * int(last["upper_greater"])
        tkey = f"window_upper_{args.dtype}_2p{args.log2n}"
    elif upper:
        kname = "upper_gather_kernel (top-k pass: read the input, write the elements > result)"
        k2_bytes = S * n + S * int(last["upper_greater"])
        tkey = f"upper_{args.dtype}_2p{args.log2n}"
    elif world > 1:
        kname = "window_kernel (fused count + filter, sharded level 0, this rank's shard)"
        k2_bytes = S * n + S * (int(last["n_level"][1]) / world if last["levels"] > 1 else 0)
        tkey = f"window_sharded_{args.dtype}_2p{args.log2n}"
    elif fused0:
        kname = "window_kernel (fused count + filter, level 0)"
        k2_bytes = S * n + S * int(last["n_level"][1])
        tkey = f"window_{args.mode}_{args.dtype}_2p{args.log2n}"
    elif not exact and last.get("spec_levels", 0) & 1:
        kname = "window_kernel<APX> (approximate: one-pass splitter window, level 0)"
        k2_bytes = S * n                                   # one read; the window's ranks stay on chip
        tkey = f"window_approx_{args.dtype}_2p{args.log2n}"
    else:
        kname = "count_kernel (K2, level 0)"
        k2_bytes = (S + (1 if exact else 0)) * n          # read S*n, write n oracle bytes
        tkey = f"count_{args.mode}_{args.dtype}_2p{args.log2n}"
    up_two = upper and not last.get("upper_onepass")
    k2_avg = float(np.mean(upper_ms)) if up_two and upper_ms else (ms if multi or quick else kavg(0, 1, prof_timed))
    achieved = k2_bytes / (k2_avg * 1e-3) / 1e9 if k2_avg else 0.0
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
                               + _workload_label(args, b, world, last["n_level"]),
                   "n_per_gpu": n, "k": k, "b": b, "kind": args.kind, "fused_filter": args.fused,
                   **({"ss_config": json.loads(args.cfg)} if args.cfg else {}),
                   **({"upper_path": "one pass" if last.get("upper_onepass") else "two passes"} if upper else {}),
                   "input_buffers": len(xds),
                   "l2": "inputs larger than L2 (1 GiB input vs 126 MB L2); no flush"
                   if n * S > 2 * L2_BYTES else "WARNING: input fits L2 and is not flushed (use --config)"},
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
                          "frac_of_peak": path_bytes / (ms * 1e-3) / 1e9 / (peak * (world if world > 1 else 1)),
                          "frac_of_8tbs": path_bytes / (ms * 1e-3) / (8e12 * world)},
        "kernels_ms": {"avg_per_level": [[kavg(l, q) for q in range(3)] for l in range(last["levels"] + 1)],
                       "sum_of_kernels": sum(kavg(l, q) for l in range(last["levels"] + 1) for q in range(3)),
                       "levels": last["levels"], "n_level": last["n_level"],
                       "shard_levels": last.get("shard_levels", 0)},
        "gpu_launches": int(launches_timed),
        "clocks": clk.summary(),
        "e2e": e2e,
    }
    if not args.no_cpu and world == 1:
        line["cpu_baseline"] = cpu_baselines(x, n // 2, args.cpu_seconds)
    print(json.dumps(line), flush=True)
    ctx.close()
    return 0


# ------------------------------------------------- BASELINE configs 1-4 --
class Flusher:
    """Writes a 2x-L2 scratch buffer: the next step starts with a cold L2."""

    def __init__(self, dev):
        import torch
        self.buf = torch.empty(2 * L2_BYTES // 4, dtype=torch.int32, device=f"cuda:{dev}")

    def __call__(self):
        self.buf.fill_(1)


def timed_steps(step, steps, warmup, flusher, stream):
    """Per-step device ms (CUDA events around each call; the L2 flush between
    steps is outside the events)."""
    import torch
    for _ in range(max(3, warmup)):
        step()
    torch.cuda.synchronize()
    out = []
    for _ in range(steps):
        if flusher:
            flusher()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        step()
        b.record(stream)
        torch.cuda.synchronize()
        out.append(a.elapsed_time(b))
    return out


def _bits(v):
    v = np.asarray(v)
    u = np.uint32 if v.dtype.itemsize == 4 else np.uint64
    return int(v.reshape(1).view(u)[0])


def run_configs(args):
    import torch
    import oracle
    import datagen
    import paper_conf_ipps_ribizela19_b200 as ss
    torch.cuda.set_device(0)
    stream = torch.cuda.current_stream(0)
    ctx = ss.Context(0)
    peak, peak_src = measured_peak()
    fl = Flusher(0)
    steps = args.steps
    cases = []
    with ClockSampler(0) as clk:
        if args.config == "c1":           # n = 2^16 median, 10 datasets, latency-bound
            n = 1 << 16
            for d in range(10):
                x = datagen.uniform(n, np.float32, datagen.dataset_seed(1, d))
                xd = torch.from_numpy(x).cuda()
                k = n // 2
                v = ctx.select(xd, k)
                t_or = time.perf_counter()
                ref = oracle.select(x, k)
                t_or = time.perf_counter() - t_or
                import cpu_baseline
                t_nth, _ = cpu_baseline.nth_element(x, k, parallel=False, reps=5)
                ms = timed_steps(lambda: ctx.select(xd, k), steps, args.warmup, fl, stream)
                cases.append({"dataset": d, "k": k, "us_mean": 1e3 * float(np.mean(ms)),
                              "us_min": 1e3 * float(np.min(ms)), "elements_per_s": n / (1e-3 * float(np.mean(ms))),
                              "parity_bit_exact": _bits(v) == _bits(ref), "cpu_oracle_s": t_or,
                              "cpu_nth_element_1core_s": t_nth, "launches": ctx.stats()["launches"]})
            metric = "exact-median latency (us), n=2^16 uniform fp32, 1 B200"
        elif args.config == "c2":         # n = 2^24 fp32 / fp64, uniform / normal, k in {1, n/2, n-1}
            n = 1 << 24
            for dt in (np.float32, np.float64):
                for kind in ("uniform", "normal"):
                    x = datagen.make(kind, n, dt, datagen.dataset_seed(2, 0))
                    xd = torch.from_numpy(x).cuda()
                    for k in (1, n // 2, n - 1):
                        v = ctx.select(xd, k)
                        ok = oracle.count_less(x, v) <= k < oracle.count_leq(x, v)
                        ms = timed_steps(lambda: ctx.select(xd, k), steps, args.warmup, fl, stream)
                        st = ctx.stats()
                        t = float(np.mean(ms))
                        cases.append({"dtype": _dt_name(dt), "kind": kind, "k": k, "ms_mean": t,
                                      "ms_min": float(np.min(ms)), "elements_per_s": n / (1e-3 * t),
                                      "path_bytes": st["bytes_algorithmic"],
                                      "path_frac_of_peak": st["bytes_algorithmic"] / (1e-3 * t) / 1e9 / peak,
                                      "read_once_frac_of_peak": x.itemsize * n / (1e-3 * t) / 1e9 / peak,
                                      "n_level": st["n_level"], "count_invariant_holds": bool(ok)})
            metric = "exact-select elements/s & % of HBM roofline, n=2^24 fp32/fp64, 1 B200 (L2 flushed)"
        elif args.config == "c3":         # n = 2^26 adversarial
            n = 1 << 26
            for kind in ("distinct16", "equal", "distinct1024", "perm"):
                x = datagen.make(kind, n, np.float32, datagen.dataset_seed(3, 0))
                xd = torch.from_numpy(x).cuda()
                for k in (0, n // 2, n - 1, datagen.rank(n, 3)):
                    v = ctx.select(xd, k)
                    ok = oracle.count_less(x, v) <= k < oracle.count_leq(x, v)
                    ms = timed_steps(lambda: ctx.select(xd, k), steps, args.warmup, fl, stream)
                    st = ctx.stats()
                    t = float(np.mean(ms))
                    cases.append({"kind": kind, "k": k, "ms_mean": t, "elements_per_s": n / (1e-3 * t),
                                  "path_frac_of_peak": st["bytes_algorithmic"] / (1e-3 * t) / 1e9 / peak,
                                  "read_once_frac_of_peak": 4 * n / (1e-3 * t) / 1e9 / peak,
                                  "equality_exit": st["equality_exit"], "levels": st["levels"],
                                  "count_invariant_holds": bool(ok)})
            metric = "exact-select elements/s, n=2^26 fp32 adversarial (16 / 1024 distinct, all-equal, permutation)"
        else:                             # c4: approximate, rank error vs speed
            n = 1 << 28
            per_b = {bb: {"rel_rank_err": [], "value_rel_err": [], "ms": []} for bb in (64, 256, 1024)}
            exact_ms = []
            for d in range(10):
                x = datagen.uniform(n, np.float32, datagen.dataset_seed(4, d))
                xd = torch.from_numpy(x).cuda()
                ks = np.random.default_rng(datagen.dataset_seed(4, d) + 1).integers(0, n, 10)
                for k in ks.tolist():
                    ex = ctx.select(xd, k)
                    exact_ms += timed_steps(lambda: ctx.select(xd, k), 1, 1, None, stream)
                    for bb in per_b:
                        v, r = ctx.approx_select(xd, k, bb)
                        per_b[bb]["ms"] += timed_steps(lambda: ctx.approx_select(xd, k, bb), 1, 1, None, stream)
                        per_b[bb]["rel_rank_err"].append(abs(r - k) / n)
                        per_b[bb]["value_rel_err"].append(abs(float(v) - float(ex)) / max(abs(float(ex)), 1e-30))
                del xd
            em = float(np.mean(exact_ms))
            for bb, dd in per_b.items():
                t = float(np.mean(dd["ms"]))
                cases.append({"b": bb, "calls": len(dd["ms"]), "ms_mean": t, "elements_per_s": n / (1e-3 * t),
                              "read_once_frac_of_peak": 4 * n / (1e-3 * t) / 1e9 / peak,
                              "speedup_vs_exact": em / t,
                              "rel_rank_err_mean": float(np.mean(dd["rel_rank_err"])),
                              "rel_rank_err_max": float(np.max(dd["rel_rank_err"])),
                              "bound_4_over_b": 4.0 / bb,
                              "value_rel_err_mean": float(np.mean(dd["value_rel_err"])),
                              "value_rel_err_max": float(np.max(dd["value_rel_err"]))})
            cases.append({"exact_ms_mean": em, "exact_elements_per_s": n / (1e-3 * em)})
            metric = "approximate select ms & relative rank error vs b, n=2^28 fp32 (10 datasets x 10 random k)"
    line = {"metric": metric, "config_id": args.config, "unit": "see cases", "n_gpus": 1, "steps": steps,
            "warmup": max(3, args.warmup), "data": "synthetic (datagen, DESIGN.md §5)",
            "l2": "flushed between timed steps (2x L2 scratch write), per-step CUDA events"
            if args.config != "c4" else "inputs 1 GiB > L2; per-call CUDA events",
            "peak_gbs": peak, "peak_source": peak_src, "cases": cases, "clocks": clk.summary()}
    print(json.dumps(line), flush=True)
    ctx.close()
    return 0


# ------------------------------------------------------------------ main --
def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def main():
    args = parse()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if "WORLD_SIZE" not in os.environ and args.gpus > 1:
        # one process per GPU: re-execute under torch.distributed.run
        cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
               "--master-addr=127.0.0.1", f"--master-port={_free_port()}", os.path.abspath(__file__),
               *sys.argv[1:]]
        return subprocess.call(cmd)
    if args.impl == "reference":
        return run_reference(args, rank, world)
    if world != args.gpus:
        raise SystemExit(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={world}")
    if args.config != "headline":
        if world > 1:
            return 0 if rank else run_configs(args)
        return run_configs(args)
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
