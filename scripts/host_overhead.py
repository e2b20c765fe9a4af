"""Host-side overhead probe of one select call (not part of the product)."""
import os, sys, time, ctypes
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_ipps_ribizela19_b200 as ss
from paper_conf_ipps_ribizela19_b200 import _abi

ctx = ss.Context(0)
x = torch.rand(1000, device="cuda")
L = _abi.lib()
def t(fn, R=2000):
    for _ in range(50): fn()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(R): fn()
    return (time.perf_counter() - t0) / R * 1e6
print(f"ctypes ss_abi_version: {t(lambda: L.ss_abi_version()):.2f} us")
print(f"ctx._args(tensor): {t(lambda: ctx._args(x)):.2f} us")
print(f"ctx._stream(None): {t(lambda: ctx._stream(None)):.2f} us")
print(f"select n=1000: {t(lambda: ctx.select(x, 500), 500):.2f} us")
xs = torch.rand(1 << 16, device="cuda")
print(f"select n=2^16: {t(lambda: ctx.select(xs, 1 << 15), 500):.2f} us")
xb = torch.rand(1 << 28, device="cuda")
print(f"select n=2^28: {t(lambda: ctx.select(xb, 1 << 27), 50):.2f} us")
ctx.close()
