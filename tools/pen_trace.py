"""Tail of the level-0 pencil passes (measurement, MG_PEN_TRACE=1): one V-cycle of the 512^3 bench
workload without graph capture; every pencil pass prints the spread of its CTAs' start / end times
(globaltimer) to stderr.

  MG_PEN_TRACE=1 python tools/pen_trace.py [n]
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import mg_inputs  # noqa: E402
from paper_conf_sc_antepara0jh24_b200.solver import Multigrid  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 512
m = Multigrid((n, n, n), num_levels=6, use_graph=False)
m.set_rhs(torch.from_numpy(mg_inputs.sin_rhs((n, n, n))).cuda())
m.set_solution(None)
for _ in range(2):
    m.vcycle()
    torch.cuda.synchronize()
    print("---- cycle done", file=sys.stderr, flush=True)
