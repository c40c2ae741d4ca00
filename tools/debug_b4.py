import sys, numpy as np, torch
sys.path.insert(0, '.')
import mg_inputs, oracle
from paper_conf_sc_antepara0jh24_b200.solver import Multigrid
shape = (32, 32, 64)
b = mg_inputs.random_rhs(shape, 42)
orc = oracle.OracleMG(shape, 3, 5, 4, 30); orc.set_b(b); orc.set_x(None); orc.vcycle(); want = orc.get_x(); wn = orc.norm()
for E in (8, 4):
  for gm in (0, 1):
    for fus in (1, 2):
      for L in (1, 2, 3):
        try:
          o2 = oracle.OracleMG(shape, L, 5, 4, 30); o2.set_b(b); o2.set_x(None); o2.vcycle()
          m = Multigrid((64, 32, 32), num_levels=L, pre=5, post=4, bottom=30, brick_edge=E, fusion=fus, ghost_mode=gm, ca_period=1)
          m.set_rhs(torch.from_numpy(b).cuda()); m.set_solution(None); m.vcycle(); x = m.get_solution().cpu().numpy()
          print(E, gm, fus, L, 'bitwise' if np.array_equal(x, o2.get_x()) else 'DIFF %.3e' % np.abs(x - o2.get_x()).max(), flush=True)
          m.close()
        except Exception as e:
          print(E, gm, fus, L, 'ERR', e)
