"""One small V-cycle through the C ABI for compute-sanitizer (tools/gpu_sanitize.sh).

python tools/sanitize_run.py N L SWEEP_KERNEL TB [GHOST_MODE] [bc=B] [vc=1] [E=4] [tr=T] [ca=K]
Runs one V-cycle (no graph: each kernel is launched and checked on its own) and the residual norm
on an N^3 grid with L levels, sweep_kernel / temporal_blocking as given (sweep_kernel 2 forces the
streaming / two-sweep kernels on every level), and checks x against the CPU oracle bit for bit.
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import mg_inputs  # noqa: E402
import oracle  # noqa: E402
from paper_conf_sc_antepara0jh24_b200.solver import Multigrid  # noqa: E402


def main():
    n, L, sk, tb = (int(v) for v in sys.argv[1:5])
    pos = [a for a in sys.argv[5:] if "=" not in a]
    kv = dict(a.split("=") for a in sys.argv[5:] if "=" in a)
    gm = int(pos[0]) if pos else 0
    bc, vc, E = int(kv.get("bc", 0)), int(kv.get("vc", 0)), int(kv.get("E", 0))
    tr, ca = int(kv.get("tr", 0)), int(kv.get("ca", 0))  # transport (3: peer kernel), CA period
    shape = (n, n, n)
    b = mg_inputs.random_rhs(shape, 0)
    c = mg_inputs.random_coef(shape, 0) if vc else None
    m = Multigrid(shape, num_levels=L, use_graph=False, sweep_kernel=sk, temporal_blocking=tb, ghost_mode=gm,
                  bc=bc, var_coef=vc, brick_edge=E, transport=tr, ca_period=ca or None)
    if vc:
        m.set_coefficients(torch.from_numpy(c).cuda())
    m.set_rhs(torch.from_numpy(b).cuda())
    m.set_solution(None)
    m.vcycle()
    nr = m.residual_norm()
    x = m.get_solution().cpu().numpy()
    m.close()
    o = oracle.OracleMG(shape, L, bc=bc, coef=c)
    o.set_b(b)
    o.set_x(None)
    o.vcycle()
    ok = np.array_equal(x, o.get_x()) and nr == o.norm()
    print(f"sanitize_run n={n} L={L} sweep_kernel={sk} tb={tb} ghost_mode={gm} bc={bc} vc={vc} E={E or 8}: "
          f"bitwise={ok}")
    sys.exit(0 if ok else 1)


if __name__ == "__main__":
    main()
