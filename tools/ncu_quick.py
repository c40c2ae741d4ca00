"""Print the key counters of one ncu capture (run here on the .ncu-rep brought back)."""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
h = rows[0]
keys = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_sector_hit_rate.pct",
        "smsp__inst_executed.sum", "sm__issue_active.avg.pct_of_peak_sustained_elapsed",
        "l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__cycles_active.avg", "sm__cycles_elapsed.avg", "smsp__warps_active.avg.per_cycle_active"]
stall = [k for k in h if k.startswith("smsp__average_warps_issue_stalled_") and k.endswith("per_issue_active.ratio")]
for r in rows[2:]:
    print(r[h.index("Kernel Name")][:60], r[h.index("Grid Size")], r[h.index("Block Size")])
    for k in keys:
        if k in h:
            print(f"  {k:70s} {r[h.index(k)]}")
    st = sorted(((float(r[h.index(k)] or 0), k) for k in stall), reverse=True)[:7]
    for v, k in st:
        print(f"  stall {k[34:-27]:30s} {v:.2f}")
