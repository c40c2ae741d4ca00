"""A/B timing of V-cycle variants on one GPU (tool; not the bench contract).

  python tools/ab_vcycle.py --n 512 --levels 6 --variants "tb=0" "tb=1"
Each variant: key=value pairs passed to Multigrid (tb -> temporal_blocking,
sk -> sweep_kernel, fusion, ca_period, ghost_mode).  Prints one JSON line per
variant: device ms per V-cycle (CUDA events, 10 cycles after 3 warm-up) and the
per-level ms of an instrumented cycle.
"""
import argparse
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import mg_inputs  # noqa: E402
from paper_conf_sc_antepara0jh24_b200.solver import Multigrid  # noqa: E402

ALIAS = {"tb": "temporal_blocking", "sk": "sweep_kernel"}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=512)
    ap.add_argument("--levels", type=int, default=6)
    ap.add_argument("--cycles", type=int, default=10)
    ap.add_argument("--variants", nargs="+", default=["tb=0"])
    a = ap.parse_args()
    n = a.n
    b = torch.from_numpy(mg_inputs.sin_rhs((n, n, n))).cuda()
    for v in a.variants:
        kw = {}
        for tok in v.split(","):
            if tok:
                k, val = tok.split("=")
                kw[ALIAS.get(k, k)] = int(val)
        m = Multigrid((n, n, n), num_levels=a.levels, **kw)
        m.set_rhs(b)
        m.set_solution(None)
        for _ in range(3):
            m.vcycle()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(m.stream)
        for _ in range(a.cycles):
            m.vcycle()
        e1.record(m.stream)
        torch.cuda.synchronize()
        m.set_timing(True)
        m.vcycle()
        t = m.timings()
        m.set_timing(False)
        print(json.dumps({"variant": v, "ms_per_vcycle": e0.elapsed_time(e1) / a.cycles,
                          "level_ms": [round(sum(r), 3) for r in t], "norm": m.residual_norm()}), flush=True)
        m.close()
        del m
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
