"""Markdown summary of tools/config_sweep.py output (runs here, no GPU).

  python tools/configs_table.py gpurun_out/configs.json profiles/r01_configs.md
"""
import json
import sys

OPS = ["sweep", "applyOp", "smooth", "restrict", "interp", "zero", "exchange", "bottom"]


def desc(r):
    parts = []
    fu = r.get("fusion", [0])[0]
    parts.append({0: "fusion auto(full)", 1: "paper kernel set", 2: "fused sweep", 3: "full fusion"}[fu])
    tb = r.get("temporal_blocking", 3) if fu != 1 else 0
    if r.get("var_coef") or r.get("brick_edge") == 4:
        tb = 0  # (the one-brick kernel family)
    parts.append({0: "1 sweep/pass", 1: "2 sweeps/pass (one-brick CTA streams)", 2: "2 sweeps/pass (warp streams)",
                  3: "2 sweeps/pass (2x2-brick pencils)"}[tb])
    if r.get("ghost_mode"):
        parts.append(f"self-exchange k={r['ca_period'][0]}")
    if r.get("pre") is not None:
        parts.append(f"s={r['pre']}")
    if r.get("smoother") in (1, 2):
        parts.append({1: "Chebyshev smoother", 2: "red-black Gauss-Seidel smoother"}[r["smoother"]])
    if r.get("bottom_solver") == 1:
        parts.append("CG bottom")
    if r.get("bc"):
        parts.append({1: "Dirichlet", 2: "Neumann"}[r["bc"]])
    if r.get("var_coef"):
        parts.append("variable coefficients")
    if r.get("brick_edge") == 4:
        parts.append("4^3 bricks")
    return ", ".join(parts)


def main():
    runs = json.load(open(sys.argv[1]))
    out = ["# Configs 1, 2, 3, 5 on one B200 (SURVEY §8(d))", "",
           f"Source: `{sys.argv[1]}` from `tools/config_sweep.py` (CUDA events around graph-replayed V-cycles,",
           "mean of 5 after 3 warm-up; sin right-hand side; device-resident inputs).  DOF/s = n^3 / time.", ""]
    sect = [("c1", "Config 1: 64^3, L = 4, solve to 1e-10"), ("c2", "Config 2: 256^3, L = 6 (256 -> 8)"),
            ("c3", "Config 3: 512^3, L = 6, self-exchange mode (ghost shell on every axis, local copies)"),
            ("c3_fusion", "Config 3: 512^3, L = 6, fusion variants (no ghosts)"),
            ("c5", "Config 5 at P = 1: 1024^3, L = 7 (global coarsest 16^3)")]
    for tag, title in sect:
        rr = [r for r in runs if r["tag"] == tag]
        if not rr:
            continue
        out += [f"## {title}", "", "| variant | ms / V-cycle | GDOF/s | launches | exchange MB / msgs | note |",
                "|---|---|---|---|---|---|"]
        for r in rr:
            note = ""
            if "solve" in r:
                sv = r["solve"]
                note = f"solve: {sv['cycles']} cycles to {sv['final_norm']:.2e} in {sv['wall_ms']:.1f} ms wall"
            out.append(f"| {desc(r)} | {r['ms_per_vcycle']:.3f} | {r['dof_per_s'] / 1e9:.2f} | {r['launches']} | "
                       f"{r['exchange_bytes'] / 1e6:.0f} / {r['exchange_msgs']} | {note} |")
        out.append("")
    # per level x op split of the config-2 / c3_fusion default runs (instrumented cycle)
    for tag in ("c2", "c3_fusion", "c5"):
        variant = ("fusion", "ghost_mode", "smoother", "bottom_solver", "bc", "var_coef", "brick_edge",
                   "temporal_blocking", "pre", "solve")
        rr = [r for r in runs if r["tag"] == tag and not any(r.get(k) for k in variant)]
        if not rr:
            continue
        r = rr[0]
        out += [f"### Per level x op, `{tag}` {r['n']}^3 default (instrumented cycle, ms)", "",
                "| level | n | " + " | ".join(OPS) + " | total | share |", "|---" * (len(OPS) + 4) + "|"]
        tot = sum(sum(v) for v in r["level_op_ms"])
        for lvl, row in enumerate(r["level_op_ms"]):
            s = sum(row)
            out.append(f"| {lvl} | {r['n'] >> lvl} | " + " | ".join(f"{v:.3f}" if v else "" for v in row) +
                       f" | {s:.3f} | {s / tot:.1%} |")
        out.append("")
    open(sys.argv[2], "w").write("\n".join(out) + "\n")
    print("\n".join(out))


if __name__ == "__main__":
    main()
