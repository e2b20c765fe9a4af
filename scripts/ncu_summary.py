"""Summarise ncu --set full reports: `python scripts/ncu_summary.py rep.ncu-rep [...]` (reads via ncu -i)."""
import csv, io, subprocess, sys

WANT = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "launch__grid_size", "launch__block_size", "launch__registers_per_thread",
    "sm__warps_active.avg.per_cycle_active", "smsp__inst_executed.sum",
    "smsp__issue_active.avg.pct_of_peak_sustained_active",
    "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
    "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
    "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
    "sm__pipe_shared_cycles_active.avg.pct_of_peak_sustained_active",
    "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum",
    "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum",
    "l1tex__data_pipe_lsu_wavefronts_mem_shared.avg.pct_of_peak_sustained_elapsed",
    "smsp__inst_executed_op_shfl.sum" , "sm__cycles_elapsed.avg.per_second",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
]
STALLS = "smsp__average_warp_latency_issue_stalled_"


def main():
    for rep in sys.argv[1:]:
        out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
        rows = list(csv.reader(io.StringIO(out)))
        hdr, units = rows[0], rows[1]
        for r in rows[2:]:
            d = dict(zip(hdr, r))
            print(f"== {rep}: {d.get('Kernel Name', '?')[:70]}")
            for w in WANT:
                if w in d:
                    print(f"  {w} = {d[w]} {units[hdr.index(w)]}")
            st = sorted(((float(d[k] or 0), k[len(STALLS):]) for k in d if k.startswith(STALLS) and k.endswith(".ratio")),
                        reverse=True)[:8]
            print("  stalls (cycles/issued inst):", ", ".join(f"{n.replace('.ratio','')} {v:.2f}" for v, n in st))


if __name__ == "__main__":
    main()
