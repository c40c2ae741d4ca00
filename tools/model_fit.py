"""Latency/throughput model fits (the paper's f(x) = x / (alpha + x/beta),
P:L214-238) from tools/config_sweep.py output.  Runs here (no GPU).

  python tools/model_fit.py gpurun_out/configs.json profiles/r01_model_fit.md

Per op kind, every timed invocation is a sample (x = points the op touches, t = device time);
t = alpha + x / beta is fitted by least squares on relative error (weights 1/t), so alpha is
the per-invocation latency (launch + ramp + tail) and beta the asymptotic throughput.  The
exchange is fitted on bytes.  The Fig 7-style view splits each V-cycle level's time into
alpha * invocations (latency share) and x / beta (throughput share).
"""
import collections
import json
import sys

import numpy as np

OPS = ["sweep", "applyOp", "smooth", "restrict", "interp", "zero", "exchange", "bottom"]
# algorithmic bytes per point: fused sweep 24 (+r 32), applyOp 16, smooth+r 40,
# restriction 9 per fine point, interpolation 17 per fine point, initZero 8 per coarse point
BPP = {"sweep": 24.0, "applyOp": 16.0, "smooth": 40.0, "restrict": 9.0, "interp": 17.0, "zero": 8.0}


def samples(runs):
    """(op, x, ms) per timed invocation.  x: cells of the level the op runs on (restrict / interp:
    fine level; zero: the coarse level it zeroes; exchange: ghost bytes of the level)."""
    out = []
    for r in runs:
        n = r["n"]
        gm = r.get("ghost_mode", 0)
        nbot = sum(1 for rec in r["records"] if OPS[rec[1]] == "bottom")
        for lvl, op, ms in r["records"]:
            nl = n >> lvl
            name = OPS[op]
            if name == "exchange":
                # bytes of one x-exchange: the ghost cells within the exchange depth d of the owned box
                # (the copy transports move only those; NCCL whole bricks, d = 8)
                k = (r.get("ca_period") or [0] * 16)[lvl]
                d = 8 if r.get("transport") == 1 else min(k if k else (2 if lvl == 0 else 8), 8)
                x = ((nl + 2 * d) ** 3 - nl ** 3) * 8.0 if gm == 1 else None
            elif name == "bottom":
                if nbot > 1:  # one record per bottom sweep (launched sweeps)
                    name, x = "bottom_sweep", float(nl ** 3)
                elif lvl < r["levels"] - 1:  # the cluster coarse solve of levels lvl .. L-1
                    name, x = "coarse_cluster", float(nl ** 3)
                else:  # the resident kernel: all sweeps in one launch
                    x = nl ** 3 * float(r.get("bottom", 100))
            else:
                x = float(nl ** 3)
            if x:
                out.append((name, x, ms, r["tag"], r.get("temporal_blocking", 3), lvl, r.get("fusion", [0])[0]))
    return out


def fit(xs, ts):
    xs, ts = np.asarray(xs), np.asarray(ts)
    w = 1.0 / ts
    A = np.stack([np.ones_like(xs), xs], 1) * w[:, None]
    (alpha, inv_beta), *_ = np.linalg.lstsq(A, ts * w, rcond=None)
    alpha = max(alpha, 0.0)
    pred = alpha + xs * inv_beta
    return alpha, 1.0 / inv_beta if inv_beta > 0 else float("inf"), float(np.max(np.abs(pred - ts) / ts))


def main():
    runs = json.load(open(sys.argv[1]))
    dst = sys.argv[2]
    S = samples(runs)
    lines = ["# Latency / throughput fits (N3): t = alpha + x / beta per op invocation", "",
             f"Source: `{sys.argv[1]}` (tools/config_sweep.py on one B200; CUDA events around every op of an",
             "instrumented V-cycle; sizes 8^3 .. 1024^3 from the levels of the 32^3 .. 1024^3 runs).", "",
             "| op (runs) | samples | alpha (us) | beta (Gpts/s) | beta x alg. B/pt (GB/s) | max rel. misfit |",
             "|---|---|---|---|---|---|"]
    groups = {
        "applyOp + smooth+residual (paper set, 2 kernels)": [s for s in S if s[0] == "sweep" and s[3] == "fit_paper"],
        "restriction (paper set)": [s for s in S if s[0] == "restrict" and s[3] == "fit_paper"],
        "interpolation (paper set)": [s for s in S if s[0] == "interp" and s[3] == "fit_paper"],
        "initZero (paper set)": [s for s in S if s[0] == "zero" and s[3] == "fit_paper"],
        "fused sweep, streaming kernel (>= 256^3, tb=0)": [s for s in S if s[0] == "sweep" and s[4] == 0 and
                                                          s[6] != 1 and s[3] in ("c2", "c3_fusion") and
                                                          s[1] >= 256 ** 3],
        "fused sweep, one-brick CTAs (<= 128^3)": [s for s in S if s[0] == "sweep" and s[4] == 0 and
                                                   s[6] != 1 and s[3] in ("c2", "c3_fusion") and s[1] <= 128 ** 3],
        "bottom sweep, launched (paper set)": [s for s in S if s[0] == "bottom_sweep" and s[3] == "fit_paper"],
        "bottom, 100 sweeps in one resident CTA": [s for s in S if s[0] == "bottom"],
        "coarse levels <= 64 bricks, one cluster launch (x = cells of its top level)":
            [s for s in S if s[0] == "coarse_cluster"],
        "exchange, self (local copies)": [s for s in S if s[0] == "exchange" and s[3] == "c3"],
    }
    fits = {}
    for name, ss in groups.items():
        if len(ss) < 3:
            continue
        if len({s[1] for s in ss}) < 2:  # one size only: the mean time is all latency
            t = np.array([s[2] for s in ss])
            lines.append(f"| {name} (one size: mean time) | {len(ss)} | {t.mean() * 1e3:.1f} | — | — | "
                         f"{float(np.max(np.abs(t - t.mean()) / t)):.2f} |")
            continue
        a, b, mis = fit([s[1] for s in ss], [s[2] for s in ss])
        fits[name] = (a, b)
        key = name.split(",")[0].split(" ")[0]
        bpp = {"applyOp": 56, "restriction": 9, "interpolation": 17, "initZero": 8, "fused": 24,
               "bottom": 24}.get(key)
        if name.startswith("exchange"):
            lines.append(f"| {name} | {len(ss)} | {a * 1e3:.1f} | — | {b / 1e6:.1f} (bytes) | {mis:.2f} |")
        elif name.startswith("bottom, 100") or name.startswith("coarse levels"):
            lines.append(f"| {name} | {len(ss)} | {a * 1e3:.1f} | {b / 1e6:.2f} (pt-sweeps) | — | {mis:.2f} |")
        else:
            gbs = f"{b / 1e6 * bpp:.0f}" if bpp else "—"
            lines.append(f"| {name} | {len(ss)} | {a * 1e3:.1f} | {b / 1e6:.2f} | {gbs} | {mis:.2f} |")
    lines += ["", "alpha is what one invocation costs at any size (launch inside a CUDA graph, ramp, tail);",
              "x / beta is the bandwidth part.  At 512^3 the level-0 ops run at their throughput; from",
              "64^3 down every op is latency-bound (x / beta < alpha).", ""]
    # Fig 7-style view on the default 512^3 cycle
    for tag in ("c3_fusion", "fit_default"):
        rr = [r for r in runs if r["tag"] == tag and r["n"] == 512 and "fusion" not in r]
        if rr:
            r = rr[0]
            break
    else:
        r = None
    if r is not None and "fused sweep, one-brick CTAs (<= 128^3)" in fits:
        a, b = fits["fused sweep, one-brick CTAs (<= 128^3)"]
        per = collections.defaultdict(lambda: [0.0, 0])
        for lvl, op, ms in r["records"]:
            per[lvl][0] += ms
            per[lvl][1] += 1
        lines += ["## Where the default 512^3 V-cycle's time goes (Fig 7-style)", "",
                  f"Measured per level (instrumented cycle, `{r['tag']}`), and the latency share alpha x ops with",
                  f"alpha = {a * 1e3:.1f} us (one-brick fused-sweep fit; the streaming kernels' alpha is similar).", "",
                  "| level | n | ops | measured ms | latency alpha x ops (ms) | latency share |", "|---|---|---|---|---|---|"]
        tot = sum(v[0] for v in per.values())
        lat = 0.0
        for lvl in sorted(per):
            ms, cnt = per[lvl]
            la = a * cnt
            lat += la
            lines.append(f"| {lvl} | {r['n'] >> lvl} | {cnt} | {ms:.3f} | {la:.3f} | {min(1.0, la / ms):.0%} |")
        lines += ["", f"Total {tot:.2f} ms; latency floor {lat:.2f} ms ({lat / tot:.0%}).  Removing every launch",
                  "and ramp of levels >= 2 (a resident coarse solver, N2) can save at most the latency",
                  "share of those levels.", ""]
    open(dst, "w").write("\n".join(lines) + "\n")
    print("\n".join(lines))


if __name__ == "__main__":
    main()
