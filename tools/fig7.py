"""Fig 7-style potential-speedup view of the finest-level operations:

    Speedup = 100% / %Roofline  x  100% / %Theoretical AI

per level-0 kernel of an ncu launch list (gpu__time_duration, dram__bytes_read / _write per launch),
with %Roofline = algorithmic bytes / time / peak HBM and %Theoretical AI = algorithmic bytes / DRAM
bytes (observed AI over the compulsory-miss AI).  Algorithmic bytes per fine point are those
of DESIGN.md §7 (Table IV decomposed).  Run here on a launch list brought back from the GPU:

  python tools/fig7.py gpurun_out/launches.csv 512 [peak_gbs] > profiles/r02_fig7.md
"""
import collections
import csv
import io
import json
import os
import re
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

# (name prefix, template args) -> (operation, algorithmic bytes per fine point)
B_PER_PT = [
    ("sweep2p_kernel<2>", "two-sweep pass + restriction (pencil)", 25.0),
    ("sweep2p_kernel<0>", "two-sweep pass (pencil)", 24.0),
    ("sweep2p_kernel<1>", "two-sweep pass + r (pencil)", 32.0),
    # SW_PEER (256): the exchange fused into the pass -- ghost slabs from the owners' fields
    ("sweep2p_kernel<258>", "two-sweep pass + restriction, exchange fused (pencil, SW_PEER)", 25.0),
    ("sweep2p_kernel<256>", "two-sweep pass, exchange fused (pencil, SW_PEER)", 24.0),
    ("sweep_col_kernel<0>", "fused sweep (column)", 24.0),
    ("sweep_col_kernel<1>", "fused sweep + r (column)", 32.0),
    ("sweep_col_kernel<2>", "fused sweep + restriction (column)", 25.0),
    ("interp4_kernel", "interpolation+increment", 17.0),
    ("interp_kernel", "interpolation+increment", 17.0),
    ("sweep_kernel<1, 0>", "applyOp (paper kernel set)", 16.0),
    ("sweep_kernel<2, 0>", "maxNormRes", 16.0),
    ("smooth_kernel<1>", "smooth+residual (paper kernel set)", 40.0),
    ("smooth_kernel<0>", "smooth (paper kernel set)", 32.0),
    ("restrict_kernel", "restriction", 9.0),
    ("zero_kernel", "initZero (per coarse point: 8 B)", 1.0),
    # the N4 variants' level-0 kernels (one-brick family): variable coefficients read c too (32 B/pt);
    # 4^3 bricks (generic.cu) move the paper's bytes
    ("sweep_kernel<0, 64>", "fused sweep, variable coefficients (one-brick)", 32.0),
    ("sweep_kernel<0, 65>", "fused sweep + r, variable coefficients (one-brick)", 40.0),
    ("sweep_kernel<0, 66>", "fused sweep + restriction, variable coefficients (one-brick)", 33.0),
    ("sweep_kernel<0, 68>", "interpolation + fused sweep, variable coefficients (one-brick)", 33.0),
    ("sweep_kernel<2, 64>", "maxNormRes, variable coefficients", 24.0),
    ("sweep_kernel<0, 0>", "fused sweep (one-brick)", 24.0),
    ("sweep_kernel<0, 2>", "fused sweep + restriction (one-brick)", 25.0),
    ("sweep_kernel<0, 4>", "interpolation + fused sweep (one-brick)", 25.0),
    ("sweep_col_kernel<128>", "maxNormRes (TMA column kernel)", 16.0),
    ("sweep_col_kernel<64>", "fused sweep, variable coefficients (column)", 32.0),
    ("sweep_col_kernel<65>", "fused sweep + r, variable coefficients (column)", 40.0),
    ("sweep_col_kernel<66>", "fused sweep + restriction, variable coefficients (column)", 33.0),
    ("sweep_col_kernel<192>", "maxNormRes, variable coefficients (column)", 24.0),
    ("unnamed>::gsweep_kernel<4, 0, 0>", "fused sweep, 4^3 bricks", 24.0),
    ("unnamed>::gsweep_kernel<4, 0, 2>", "fused sweep + restriction, 4^3 bricks", 25.0),
    ("unnamed>::gsweep_kernel<4, 0, 4>", "interpolation + fused sweep, 4^3 bricks", 25.0),
    ("unnamed>::gsweep_kernel<4, 2, 0>", "maxNormRes, 4^3 bricks", 16.0),
    ("mirror_kernel", "mirror exchange (Dirichlet / Neumann faces)", 0.0),
]


def read_csv(path):
    lines = open(path).read().splitlines()
    start = next(i for i, l in enumerate(lines) if l.startswith('"ID"'))
    return list(csv.DictReader(io.StringIO("\n".join(lines[start:]))))


def classify(name):
    name = name[5:] if name.startswith("void ") else name
    # (the one-brick sweep kernel's thread-count template argument does not change the operation)
    name = re.sub(r"^sweep_kernel<(\d+), (\d+), \d+>", r"sweep_kernel<\1, \2>", name)
    for pre, op, b in B_PER_PT:
        if name.startswith(pre):
            return op, b
    return None, None


def main():
    src, n = sys.argv[1], int(sys.argv[2])
    if len(sys.argv) > 3:
        peak = float(sys.argv[3])
    else:
        mp = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
        peak = float(mp.get("hbm_gbs") or mp.get("hbm_copy_gbs"))
    pts = float(n) ** 3
    per = collections.defaultdict(dict)
    for r in read_csv(src):
        d = per[r["ID"]]
        d["name"] = r["Kernel Name"]
        v = float(r["Metric Value"].replace(",", ""))
        u = r["Metric Unit"]
        if r["Metric Name"] == "gpu__time_duration.sum":
            d["us"] = v / 1e3 if u == "ns" else (v * 1e3 if u == "ms" else v)
        elif r["Metric Name"].startswith("dram__bytes"):
            scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(u, 1)
            d["dram"] = d.get("dram", 0.0) + v * scale
    agg = collections.OrderedDict()
    for d in per.values():
        op, b = classify(d["name"])
        if op is None or "us" not in d or "dram" not in d:
            continue
        alg = b * pts
        if alg == 0.0:
            continue
        if op.startswith("initZero"):
            alg = 8.0 * pts / 8.0  # x of level 1 = one eighth of the fine points, 8 B each
        # level-0 launches only: their DRAM traffic is within a factor 2 of the algorithmic bytes
        if not (0.5 * alg <= d["dram"] <= 2.5 * alg):
            continue
        a = agg.setdefault(op, [0, 0.0, 0.0, alg])
        a[0] += 1
        a[1] += d["us"]
        a[2] += d["dram"]
    print(f"# Fig 7-style potential speed-up, finest level ({n}^3), one B200\n")
    print(f"Source: `{os.path.relpath(src, ROOT)}` (ncu launch list, cold-cache serialised launches); "
          f"peak HBM {peak:.0f} GB/s (MEASURED_PEAKS.json).  Speedup = 1/%Roofline x 1/%TheoreticalAI "
          f"(P:L300).\n")
    print("| operation | launches | us / launch | algorithmic GB | DRAM GB | achieved GB/s | %Roofline | "
          "%Theoretical AI | potential speed-up |")
    print("|---|---|---|---|---|---|---|---|---|")
    for op, (cnt, us, dram, alg) in agg.items():
        t = us / cnt * 1e-6
        dr = dram / cnt
        ach = alg / t / 1e9
        roof = ach / peak
        ai = alg / dr
        print(f"| {op} | {cnt} | {us / cnt:.1f} | {alg / 1e9:.3f} | {dr / 1e9:.3f} | {ach:.0f} | {100 * roof:.1f}% | "
              f"{100 * ai:.1f}% | {1 / (roof * ai):.2f}x |")


if __name__ == "__main__":
    main()
