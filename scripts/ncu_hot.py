"""Hot SASS lines of one kernel in an ncu report: python scripts/ncu_hot.py rep.ncu-rep <kernel-regex> [launch-skip] [N]"""
import csv, io, subprocess, sys
rep, kre = sys.argv[1], sys.argv[2]
skip = sys.argv[3] if len(sys.argv) > 3 else "0"
N = int(sys.argv[4]) if len(sys.argv) > 4 else 40
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "-k", f"regex:{kre}", "-s", skip, "-c", "1",
                      "--print-source", "sass"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr = next(r for r in rows if r and r[0] == "Address")
data = [r for r in rows if r and r[0].startswith("0x")]
ie, iss = hdr.index("Instructions Executed"), hdr.index("Warp Stall Sampling (All Samples)")
f = lambda x: int(x) if x.strip() else 0
tot = sum(f(r[ie]) for r in data)
print(f"{len(data)} SASS lines, {tot} warp instructions, {sum(f(r[iss]) for r in data)} stall samples")
# group consecutive lines into blocks with equal exec counts
blocks, cur = [], None
for i, r in enumerate(data):
    c = f(r[ie])
    if cur and cur[1] == c:
        cur[2] += 1; cur[3] += f(r[iss])
    else:
        cur = [i, c, 1, f(r[iss]), r[1].strip()[:60]]; blocks.append(cur)
blocks.sort(key=lambda b: -b[1] * b[2])
for b in blocks[:N]:
    print(f"line {b[0]:5d}  exec {b[1]:9d} x {b[2]:3d} instr = {b[1]*b[2]:10d}  stalls {b[3]:6d}  {b[4]}")
