"""Hot SASS instructions and stall reasons of one ncu --set full capture (run here, no GPU).

  python tools/sass_hot.py gpurun_out/prof_sweep.ncu-rep [top]
"""
import collections
import csv
import io
import subprocess
import sys


def main(rep, top=30):
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    h, v = rows[0], rows[2]
    keys = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
            "l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed",
            "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "smsp__issue_active.avg.pct_of_peak_sustained_active",
            "sm__warps_active.avg.pct_of_peak_sustained_active", "smsp__warps_eligible.avg.per_cycle_active",
            "smsp__inst_executed.sum", "launch__registers_per_thread", "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active",
            "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "sm__cycles_elapsed.avg.per_second"]
    for i, n in enumerate(h):
        if n in keys:
            print(f"{n:70s} {v[i]} {rows[1][i]}")
    st = [(float(v[i]), n) for i, n in enumerate(h)
          if n.startswith("smsp__average_warps_issue_stalled_") and n.endswith("_per_issue_active.ratio")]
    for x, n in sorted(st, reverse=True)[:8]:
        print(f"  stall {n[34:-23]:24s} {x:.3f}")
    src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(src)))
    hdr, data = rows[1], rows[2:]
    ai, si = hdr.index("Address"), hdr.index("Source")
    wi, ie = hdr.index("Warp Stall Sampling (All Samples)"), hdr.index("Instructions Executed")
    tot = 0
    byop, cnt, lst = collections.Counter(), collections.Counter(), []
    for k, r in enumerate(data):
        if len(r) <= wi:
            continue
        s = int(r[wi] or 0)
        tot += s
        toks = r[si].split()
        op = (toks[1] if toks and toks[0].startswith("@") and len(toks) > 1 else (toks[0] if toks else "")).split(".")[0]
        byop[op] += s
        cnt[op] += int(r[ie] or 0)
        lst.append((s, k))
    print("samples", tot)
    for op, s in byop.most_common(16):
        print(f"  {op:10s} {100 * s / tot:5.1f}%  executed {cnt[op]}")
    for s, k in sorted(lst, reverse=True)[:top]:
        ctx = " | ".join(data[j][si].strip()[:40] for j in range(max(0, k - 2), k))
        print(f"{100 * s / tot:5.1f}% {data[k][si].strip()[:60]:60s}  after: {ctx}")


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 30)
