"""Summarise ncu outputs into profiles/ (run here, no GPU needed).

  python tools/ncu_summary.py launches gpurun_out/launches.csv profiles/rNN_launches.md [steps_hint]
  python tools/ncu_summary.py full gpurun_out/prof_sweep.ncu-rep profiles/rNN_sweep_full.md [n]

`launches`: per-kernel share of device time (cold-cache, serialised launches:
compare SHARES, not absolute times).  `full`: DRAM bytes, throughput, occupancy,
registers and top stall reasons of the captured launch(es); also writes
profiles/ncu_sweep_summary.json (per-launch DRAM bytes) that bench.py reads
for the roofline `traffic` field.
"""
import collections
import csv
import io
import json
import os
import subprocess
import sys


def read_csv(path):
    lines = open(path).read().splitlines()
    start = next(i for i, l in enumerate(lines) if l.startswith('"ID"'))
    return list(csv.DictReader(io.StringIO("\n".join(lines[start:]))))


def short(name):
    return name.split("(")[0][:80]


def launches(src, dst):
    rows = [r for r in read_csv(src) if r["Metric Name"] == "gpu__time_duration.sum"]
    agg = collections.OrderedDict()
    for r in rows:
        k = short(r["Kernel Name"])
        v = float(r["Metric Value"].replace(",", ""))
        unit = r["Metric Unit"]
        v = v / 1e3 if unit == "ns" else (v * 1e3 if unit == "ms" else v)  # -> us
        a = agg.setdefault(k, [0, 0.0, r["Grid Size"], r["Block Size"]])
        a[0] += 1
        a[1] += v
    tot = sum(a[1] for a in agg.values())
    out = ["# ncu launch list (gpu__time_duration.sum, --clock-control none)", "",
           f"source: `{src}`; {len(rows)} launches; total {tot / 1e3:.2f} ms", "",
           "| kernel | launches | total us | share | avg us | last grid | block |", "|---|---|---|---|---|---|---|"]
    for k, (n, t, g, b) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
        out.append(f"| `{k}` | {n} | {t:.1f} | {t / tot * 100:.1f}% | {t / n:.2f} | {g} | {b} |")
    open(dst, "w").write("\n".join(out) + "\n")
    print("\n".join(out))


METRICS = ["dram__bytes_read.sum", "dram__bytes_write.sum", "gpu__time_duration.sum", "dram__throughput.avg.pct_of_peak_sustained_elapsed",
           "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "sm__warps_active.avg.pct_of_peak_sustained_active",
           "launch__registers_per_thread", "launch__occupancy_limit_registers", "launch__occupancy_limit_shared_mem",
           "sm__maximum_warps_per_active_cycle_pct", "lts__t_bytes.sum", "l1tex__t_bytes.sum",
           "sm__throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sector_hit_rate.pct",
           "launch__grid_size", "launch__block_size", "smsp__inst_executed.sum",
           "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active",
           "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "achieved_occupancy",
           "sm__warps_active.avg.per_cycle_active"]


def full(src, dst, n=None):
    raw = subprocess.run(["ncu", "-i", src, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = read_csv_text(raw)
    out = [f"# ncu --set full summary: `{os.path.basename(src)}`", ""]
    js = []
    for r in rows:
        name = short(r.get("Kernel Name", "?"))
        out.append(f"## `{name}` grid {r.get('Grid Size')} block {r.get('Block Size')}")
        out.append("")
        out.append("| metric | value |")
        out.append("|---|---|")
        for m in METRICS:
            if m in r:
                out.append(f"| {m} | {r[m]} |")
        rd = to_bytes(r, "dram__bytes_read.sum")
        wr = to_bytes(r, "dram__bytes_write.sum")
        t = to_ns(r, "gpu__time_duration.sum")
        if rd is not None and wr is not None and t:
            out.append(f"| DRAM bytes (read+write) | {rd + wr:.4e} |")
            out.append(f"| DRAM GB/s (bytes / duration, serialised cold launch) | {(rd + wr) / t:.1f} |")
            js.append({"kernel": name, "dram_bytes_per_launch": rd + wr, "read": rd, "write": wr, "ns": t})
        out.append("")
    # stall reasons (source page, summed)
    src_csv = subprocess.run(["ncu", "-i", src, "--page", "details", "--csv", "--section", "WarpStateStats"],
                             capture_output=True, text=True).stdout
    if src_csv.strip():
        out.append("## WarpStateStats section")
        out.append("")
        out.append("```")
        out.extend(src_csv.strip().splitlines()[:40])
        out.append("```")
    open(dst, "w").write("\n".join(out) + "\n")
    print("\n".join(out))
    if js and n:
        summ = {"n": int(n), "source": os.path.basename(src), **js[0]}
        json.dump(summ, open(os.path.join(os.path.dirname(dst), "ncu_sweep_summary.json"), "w"), indent=1)


def read_csv_text(txt):
    lines = txt.splitlines()
    try:
        start = next(i for i, l in enumerate(lines) if l.startswith('"ID"'))
    except StopIteration:
        return []
    rd = list(csv.reader(io.StringIO("\n".join(lines[start:]))))
    hdr, units = rd[0], rd[1]
    rows = []
    for row in rd[2:]:
        d = {}
        for h, u, v in zip(hdr, units, row):
            d[h] = v
            d[h + "@unit"] = u
        rows.append(d)
    return rows


def to_bytes(r, k):
    if k not in r:
        return None
    v = float(r[k].replace(",", ""))
    u = r.get(k + "@unit", "byte")
    return v * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1e3, "MB": 1e6, "GB": 1e9}.get(u, 1)


def to_ns(r, k):
    if k not in r:
        return None
    v = float(r[k].replace(",", ""))
    u = r.get(k + "@unit", "ns")
    return v * {"ns": 1, "us": 1e3, "usecond": 1e3, "nsecond": 1, "ms": 1e6, "msecond": 1e6}.get(u, 1)


if __name__ == "__main__":
    mode, src, dst = sys.argv[1:4]
    if mode == "launches":
        launches(src, dst)
    else:
        full(src, dst, sys.argv[4] if len(sys.argv) > 4 else None)
