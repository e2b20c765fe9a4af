"""Device timeline of one selection (profile=3: %globaltimer stamps inside the
kernels, PDL overlap intact).  `python scripts/timeline.py [log2n] [b] [mode]`
WS_DEBUG=1 / TL_DEBUG=1 print the phase stamps of level 0's K1w / level 1's
window kernel; they need a library built with SS_NVCC_EXTRA=-DSS_PHASE_STAMPS=1
(e.g. into build_variants/ and loaded with SS_LIB=...)."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import datagen
import paper_conf_ipps_ribizela19_b200 as ss

log2n = int(sys.argv[1]) if len(sys.argv) > 1 else 28
b = int(sys.argv[2]) if len(sys.argv) > 2 else 256
mode = sys.argv[3] if len(sys.argv) > 3 else "exact"
bd = int(sys.argv[4]) if len(sys.argv) > 4 else 0
n = 1 << log2n
x = torch.from_numpy(datagen.uniform(n, np.float32, seed=datagen.dataset_seed(5, 0))).cuda()
import json
ctx = ss.Context(0, **json.loads(os.environ.get('SS_CFG', '{}')))
if mode == "exact":
    ctx.configure(b_exact=b, b_deep=bd)
run = (lambda: ctx.select(x, n // 2)) if mode == "exact" else (lambda: ctx.approx_select(x, n // 2, b))
for _ in range(5):
    run()
torch.cuda.synchronize()
ctx.configure(profile=3)
R = 20
acc = None
for _ in range(R):
    run()
    st = ctx.stats()
    tl = np.array(ctx.raw_tl(), dtype=np.float64)
    acc = tl if acc is None else acc + tl
tl = acc / R
names = ["K1", "K2", "K5"]
if os.environ.get("WS_DEBUG"):        # level-0 K1w phase stamps (tl_phase, last CTA to pass)
    names_k1w = ["keys loaded", "min/max", "pass 1", "pass 2", "pass 3", "candidates", "ranked"]
    for i, nm in enumerate(names_k1w):
        l, q = divmod(80 + i, 3)
        if tl[l][q][1] > 0:
            print(f"  K1w {nm}: first {tl[l][q][0]:8.1f}  last {tl[l][q][1]:8.1f}")
if os.environ.get("TL_DEBUG"):       # window_kernel phase stamps of level 1 (tl_phase)
    for sl, nm in ((90, "L1 window: setup done"), (91, "L1 window: stream done"), (92, "L1 window: ticket")):
        l, q = divmod(sl, 3)
        print(f"  {nm}: first {tl[l][q][0]:8.1f}  last {tl[l][q][1]:8.1f}")
print(f"n=2^{log2n} b={b} b_deep={bd} {mode}: n_level={st['n_level']}  (mean of {R} calls, us after init)")
for l in range(min(8, tl.shape[0])):
    for q in range(3):
        s0, s1 = tl[l][q]
        if s0 >= 0 and s1 > 0:
            print(f"  L{l} {names[q]}: start {s0:8.1f}  end {s1:8.1f}  dur {s1 - s0:7.1f}")
ctx.configure(profile=0)
torch.cuda.synchronize()
ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
ev0.record()
for _ in range(R):
    run()
ev1.record(); torch.cuda.synchronize()
print(f"  per call (events, profile=0): {ev0.elapsed_time(ev1) / R * 1e3:.1f} us")
