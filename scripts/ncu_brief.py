"""Key counters + stall reasons of every kernel in an .ncu-rep (for quick reading here)."""
import csv
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
        "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_tensor_subpipe_dmma_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_tensor_subpipe_dmma.sum",
        "sm__inst_executed.avg.per_cycle_active", "lts__t_sector_hit_rate.pct",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum", "launch__grid_size", "launch__block_size"]
out = subprocess.run(["ncu", "-i", sys.argv[1], "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
h = rows[0]
for v in rows[2:]:
    print(v[h.index("Kernel Name")][:100])
    for k in KEYS:
        if k in h:
            print(f"  {k:62s} {v[h.index(k)]}")
    st = []
    for i, x in enumerate(h):
        if x.startswith("smsp__pcsamp_warps_issue_stalled_") and not x.endswith("not_issued"):
            try:
                st.append((float(v[i]), x.replace("smsp__pcsamp_warps_issue_stalled_", "")))
            except ValueError:
                pass
    tot = sum(a for a, _ in st) or 1
    print("  stalls:", ", ".join(f"{n} {a / tot * 100:.0f}%" for a, n in sorted(st, reverse=True)[:7]))
