"""One line per kernel of an ncu report: name, duration, DRAM bytes, warp instructions, issue-active %.
python scripts/ncu_brief.py rep.ncu-rep"""
import csv, io, subprocess, sys
out = subprocess.run(["ncu", "-i", sys.argv[1], "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr = rows[0]
col = {h: i for i, h in enumerate(hdr)}
for r in rows[2:]:
    g = lambda k: r[col[k]] if k in col else "?"
    print(f"{g('Kernel Name')[:48]:48s} {float(g('gpu__time_duration.sum')):9.2f} us  "
          f"rd {float(g('dram__bytes_read.sum')):8.4f} GB  wr {float(g('dram__bytes_write.sum'))/1e3 if 'Mbyte' in '' else float(g('dram__bytes_write.sum')):9.4f}  "
          f"inst {float(g('smsp__inst_executed.sum')):12.0f}  issue {g('smsp__issue_active.avg.pct_of_peak_sustained_active')}%")
