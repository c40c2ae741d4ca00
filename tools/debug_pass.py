"""Debug aid: one level-0 operator run through the C ABI vs the oracle, with the error pattern.

python tools/debug_pass.py NX NY NZ NSWEEPS TB [GHOST_MODE]
Prints, for x after NSWEEPS sweeps (mg_op_smooth, write_r = 1) and r, how many cells differ and
how the wrong cells distribute over in-brick i, j, k and over tile rows / columns (16-cell tiles).
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import mg_inputs  # noqa: E402
import oracle  # noqa: E402
from paper_conf_sc_antepara0jh24_b200 import mg  # noqa: E402
from paper_conf_sc_antepara0jh24_b200.solver import Multigrid  # noqa: E402


def pattern(name, got, want):
    bad = got != want
    n = int(bad.sum())
    print(f"{name}: {n} of {bad.size} cells differ, max err {np.abs(got - want).max():.3e}")
    if n == 0:
        return
    k, j, i = np.nonzero(bad)
    for lab, v, m in (("i%8", i, 8), ("j%8", j, 8), ("k%8", k, 8), ("i%16", i, 16), ("j%16", j, 16)):
        print(f"  {lab}: {np.bincount(v % m, minlength=m).tolist()}")
    print("  first:", list(zip(k[:8].tolist(), j[:8].tolist(), i[:8].tolist())))
    kk = int(np.bincount(k).argmax())
    print(f"  plane {kk} (rows j top to bottom, i left to right; # wrong, . right):")
    for jj in range(min(bad.shape[1], 20)):
        print("   ", "".join("#" if v else "." for v in bad[kk, jj, :min(bad.shape[2], 40)]))


def main():
    nx, ny, nz, ns, tb = (int(v) for v in sys.argv[1:6])
    gm = int(sys.argv[6]) if len(sys.argv) > 6 else 0
    shape = (nz, ny, nx)
    m = Multigrid((nx, ny, nz), num_levels=1, pre=1, post=1, bottom=1, sweep_kernel=2, temporal_blocking=tb,
                  ghost_mode=gm)
    h = mg_inputs.default_h0(shape)
    x = mg_inputs.random_field(shape, 1)
    b = mg_inputs.random_field(shape, 2)
    m.level_set(0, mg.MG_FIELD_X, torch.from_numpy(x).cuda())
    m.level_set(0, mg.MG_FIELD_B, torch.from_numpy(b).cuda())
    mg.mg_op_smooth(m.ctx, 0, ns, 1, 2)
    gx = m.level_get(0, mg.MG_FIELD_X).cpu().numpy()
    gr = m.level_get(0, mg.MG_FIELD_R).cpu().numpy()
    xo, ro = x, None
    for _ in range(ns):
        xo, ro = oracle.smooth_residual(xo, oracle.apply_op(xo, h), b, h)
    pattern("x", gx, xo)
    pattern("r", gr, ro)
    m.close()


if __name__ == "__main__":
    main()
