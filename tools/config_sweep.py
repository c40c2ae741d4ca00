"""Measurement sweep over SURVEY.md §8(d) configs 1, 2, 3 and 5 on one GPU (tool; not the bench
contract).  Writes raw JSON (one object per run) for tools/model_fit.py and the profiles table.

  python tools/config_sweep.py --out gpurun_out/configs.json [--quick]

Every run: device ms per V-cycle (CUDA events over `cycles` graph-replayed cycles after 3 warm-up
cycles), then one instrumented cycle whose per-op records (level, op, ms) are kept for the
latency/throughput fits.  No oracle here (the oracle is test infrastructure).
"""
import argparse
import json
import os
import sys
import time

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import mg_inputs  # noqa: E402
from paper_conf_sc_antepara0jh24_b200 import mg  # noqa: E402
from paper_conf_sc_antepara0jh24_b200.solver import Multigrid  # noqa: E402


def run(tag, n, levels, cycles=5, solve=False, **kw):
    shape = (n, n, n)
    bsrc = mg_inputs.dirichlet_sin_rhs(shape) if kw.get("bc") == 1 else mg_inputs.sin_rhs(shape)
    b = torch.from_numpy(bsrc).cuda()
    m = Multigrid(shape, num_levels=levels, **kw)
    if kw.get("var_coef"):
        m.set_coefficients(torch.from_numpy(mg_inputs.smooth_coef(shape)).cuda())
    m.set_rhs(b)
    m.set_solution(None)
    rec = {"tag": tag, "n": n, "levels": levels, **{k: v for k, v in kw.items() if not isinstance(v, list)}}
    for k, v in kw.items():
        if isinstance(v, list):
            rec[k] = v
    if solve:
        t0 = time.perf_counter()
        _, cyc, nr = m.solve(1e-10, 20)
        torch.cuda.synchronize()
        rec["solve"] = {"cycles": cyc, "final_norm": nr, "wall_ms": (time.perf_counter() - t0) * 1e3}
        m.set_solution(None)
    for _ in range(3):
        m.vcycle()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(m.stream)
    for _ in range(cycles):
        m.vcycle()
    e1.record(m.stream)
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / cycles
    m.set_timing(True)
    m.vcycle()
    recs = m.timing_records()
    lv = m.timings()
    m.set_timing(False)
    xb, xm = m.exchange_stats()
    rec.update({"ms_per_vcycle": ms, "dof_per_s": n ** 3 / (ms / 1e3), "launches": m.launches_per_vcycle(),
                "exchange_bytes": xb, "exchange_msgs": xm, "level_op_ms": lv, "records": recs,
                "norm": m.residual_norm()})
    m.close()
    del m, b
    torch.cuda.empty_cache()
    print(json.dumps({k: v for k, v in rec.items() if k not in ("records", "level_op_ms")}), flush=True)
    return rec


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default="gpurun_out/configs.json")
    ap.add_argument("--quick", action="store_true")
    a = ap.parse_args()
    os.makedirs(os.path.dirname(a.out) or ".", exist_ok=True)

    class Out(list):  # rewritten after every run, so a late failure keeps the earlier ones
        def append(self, r):
            super().append(r)
            json.dump(self, open(a.out, "w"))

    out = Out()
    # config 1: 64^3, L = 4, solve to 1e-10; paper kernel set and fused; Chebyshev smoother variant
    for fu in (1, 3):
        out.append(run("c1", 64, 4, solve=True, fusion=[fu] * 16))
    out.append(run("c1", 64, 4, solve=True, smoother=1))
    out.append(run("c1", 64, 4, solve=True, smoother=2))
    # the N4 variants: Dirichlet / Neumann boundaries, variable coefficients, 4^3 bricks
    out.append(run("c1", 64, 4, solve=True, bc=1))
    out.append(run("c1", 64, 4, solve=True, bc=2))
    out.append(run("c1", 64, 4, solve=True, var_coef=1, bc=1))
    out.append(run("c1", 64, 4, solve=True, brick_edge=4))
    # config 2: 256^3, L = 6; paper kernel set / fused / fused + temporal blocking
    out.append(run("c2", 256, 6, fusion=[1] * 16, temporal_blocking=0))
    out.append(run("c2", 256, 6, fusion=[3] * 16, temporal_blocking=0))
    out.append(run("c2", 256, 6))
    out.append(run("c2", 256, 6, bc=1))
    out.append(run("c2", 256, 6, var_coef=1))
    out.append(run("c2", 256, 6, brick_edge=4))
    # sizes for the fits: paper kernel set (every op separate) and the default, n = 32 .. 512
    for n in (32, 64, 128, 256, 512):
        lv = max(1, min(6, n.bit_length() - 4))
        out.append(run("fit_paper", n, lv, fusion=[1] * 16, temporal_blocking=0))
        out.append(run("fit_default", n, lv))
    # config 3: 512^3 in self-exchange mode (ghost shell on every axis, local copies):
    # CA period k and smooth count s; temporal blocking off / one-brick kernel / pencils (default)
    ks = (1, 2, 4, 8)
    ss = (12,) if a.quick else (4, 8, 12, 16)
    for s in ss:
        for k in ks:
            for tb in ((3,) if s != 12 else (0, 1, 3)):
                out.append(run("c3", 512, 6, pre=s, post=s, ghost_mode=1, transport=2, ca_period=[k] * 16,
                               temporal_blocking=tb))
    # config 3: fusion variants (no ghosts)
    for fu in (1, 2, 3):
        out.append(run("c3_fusion", 512, 6, fusion=[fu] * 16, temporal_blocking=0))
    out.append(run("c3_fusion", 512, 6))
    out.append(run("c3_fusion", 512, 6, solve=True))
    out.append(run("c3_fusion", 512, 6, solve=True, smoother=1))
    out.append(run("c3_fusion", 512, 6, solve=True, smoother=2))
    out.append(run("c3_fusion", 512, 6, solve=True, bottom_solver=1))
    # config 5 at P = 1: 1024^3, L = 7 (global coarsest 16^3)
    if not a.quick:
        out.append(run("c5", 1024, 7, cycles=3))


if __name__ == "__main__":
    main()
