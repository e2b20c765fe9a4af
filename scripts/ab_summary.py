"""Summarise gpurun_out/ab.log: ms/step and per-level kernel ms per run."""
import json, sys
for line in open(sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/ab.log"):
    line = line.strip()
    if line.startswith("=="):
        print(line); continue
    try:
        d = json.loads(line)
    except Exception:
        print("  ", line[:300]); continue
    km = d.get("kernels_ms", {})
    lv = [" ".join(f"{x*1e3:6.1f}" for x in l) for l in km.get("avg_per_level", [])]
    print(f"   {d['ms_per_step']*1e3:7.1f} us/step  K2 frac {d['roofline']['frac']:.3f} | " + " | ".join(lv))
