import sys, time, torch
sys.path.insert(0, '.')
import mg_inputs
from paper_conf_sc_antepara0jh24_b200.solver import Multigrid
for n, L in ((512, 6), (256, 5), (128, 3)):
    b = torch.from_numpy(mg_inputs.sin_rhs((n, n, n))).cuda()
    for bs in (0, 1):
        if bs == 1 and (n // 2 ** (L - 1)) > 16:
            continue
        m = Multigrid((n, n, n), num_levels=L, bottom_solver=bs)
        m.set_rhs(b); m.set_solution(None)
        st, cyc, nr = m.solve(1e-10, 30)
        m.set_solution(None)
        for _ in range(3): m.vcycle()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(m.stream)
        for _ in range(5): m.vcycle()
        e1.record(m.stream); torch.cuda.synchronize()
        m.set_timing(True); m.vcycle(); torch.cuda.synchronize(); tm = m.timings(); m.set_timing(False)
        print(f"n={n} L={L} bottom_solver={bs}: solve {cyc} cycles to {nr:.2e}; {e0.elapsed_time(e1)/5:.3f} ms/cycle; bottom level ms {tm[L-1]}", flush=True)
        m.close()
