"""Weak-scaling rehearsal on one GPU: the 512^3-per-rank decompositions 2x1x1,
2x2x1 and 2x2x2 run as in-process loopback groups (every rank's V-cycle on the same GPU, ghost exchanges
as device copies through the same depth-limited plans the peer transport uses), timed per V-cycle and
divided by the rank count: the per-rank cost of the decomposition (redundant ghost work, the exchanges as
local copies, the replicated bottom) without the NVLink transfer.  A projection then swaps the local
copies for NVLink transfers: t_P = t_rank - sum(local exchange time) + sum(alpha_link + bytes / beta_link)
per exchange, with the exchanges and bytes from the schedule's own plan (mg_layout_exchange_plan).

  python tools/loopback_scaling.py [n] [levels] [beta_link_gbs] [alpha_link_us] > profiles/r02_scaling_rehearsal.md
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import mg_inputs  # noqa: E402
from paper_conf_sc_antepara0jh24_b200 import mg  # noqa: E402
from paper_conf_sc_antepara0jh24_b200.solver import LoopbackGroup, Multigrid  # noqa: E402

# local copy kernel fit (profiles/r02_exchange.md, depth-limited copies): alpha 3.0 us, beta ~2.5 TB/s
ALPHA_LOCAL_US, BETA_LOCAL_GBS = 3.0, 2500.0


def time_cycles(step, stream, warm=3, reps=10):
    for _ in range(warm):
        step()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for _ in range(reps):
        step()
    e1.record(stream)
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps


def main():
    n = int(sys.argv[1]) if len(sys.argv) > 1 else 512
    L = int(sys.argv[2]) if len(sys.argv) > 2 else 6
    beta_link = float(sys.argv[3]) if len(sys.argv) > 3 else 700.0  # GB/s into one GPU over NVLink (of 900)
    alpha_link = float(sys.argv[4]) if len(sys.argv) > 4 else 10.0  # us: the peer kernel's flag handshake
    rows = []
    m = Multigrid((n, n, n), num_levels=L)
    m.set_rhs(torch.from_numpy(mg_inputs.sin_rhs((n, n, n))).cuda())
    m.set_solution(None)
    t1 = time_cycles(m.vcycle, m.stream)
    m.close()
    del m
    torch.cuda.empty_cache()
    # exchanges fused into the pencil pass after them (the same schedule rules on every ghost-shell level:
    # asked of a one-rank context with a self-exchanged ghost shell on every axis)
    mf = Multigrid((n, n, n), num_levels=L, ghost_mode=mg.MG_GHOST_ALL, transport=mg.MG_TRANSPORT_LOCAL)
    fused = mf.exchange_fused()
    mf.close()
    del mf
    torch.cuda.empty_cache()
    for pg in ((2, 1, 1), (2, 2, 1), (2, 2, 2)):
        P = pg[0] * pg[1] * pg[2]
        g = LoopbackGroup((n, n, n), pg, num_levels=L)
        gshape = (n * pg[2], n * pg[1], n * pg[0])
        b = mg_inputs.sin_rhs(gshape)
        blocks = [torch.from_numpy(np.ascontiguousarray(mg_inputs.local_block(b, r, pg))).cuda() for r in range(P)]
        del b
        g.set_rhs(blocks)
        g.set_solution(None)
        tg = time_cycles(g.vcycle, g.stream)
        g.close()
        del g, blocks
        torch.cuda.empty_cache()
        # the schedule's exchanges per level and bytes per exchange (rank 0; every rank of these grids is alike)
        p = mg.params((n, n, n), pg, num_levels=L, transport=mg.MG_TRANSPORT_PEER)
        ex, by = mg.Layout(p, 0, P).exchange_plan()
        fu = [min(f, e) for f, e in zip(fused, ex)]
        # separate exchanges: a local copy in the measured group, an NVLink transfer projected; fused ones:
        # no copy in the group (the passes read the other ranks' fields), projected as the flag handshake
        # alone (transfer hidden under the pass) or with the transfer serialised onto the pass (bound)
        t_local = sum((e - f) * (ALPHA_LOCAL_US + b_ / (BETA_LOCAL_GBS * 1e3)) for e, f, b_ in zip(ex, fu, by)) / 1e3
        t_link = sum((e - f) * (alpha_link + b_ / (beta_link * 1e3)) + f * alpha_link
                     for e, f, b_ in zip(ex, fu, by)) / 1e3
        t_ser = sum(f * b_ / (beta_link * 1e3) for f, b_ in zip(fu, by)) / 1e3
        t_rank = tg / P
        t_proj = t_rank - t_local + t_link
        rows.append((pg, P, tg, t_rank, t_local, t_link, t_proj, ex, by, fu, t_ser))
    print(f"# Weak-scaling rehearsal on one B200 ({n}^3 per rank, L = {L}; `tools/loopback_scaling.py`)\n")
    print("Loopback groups: all ranks of the decomposition in one process on one GPU, exchanges as device copies "
          "through the depth-limited plans (the peer transport's plans); CUDA events around 10 graph-replayed "
          "V-cycles after 3 warm-up.  t_rank = group time / P is the per-rank cost with local copies.  Projection: "
          f"swap each exchange's modelled local copy (alpha {ALPHA_LOCAL_US} us, beta {BETA_LOCAL_GBS:.0f} GB/s, "
          f"`r02_exchange.md`) for an NVLink transfer (alpha {alpha_link} us, beta {beta_link:.0f} GB/s into one GPU); "
          "no overlap assumed for separate exchanges.  Exchanges fused into the pencil pass after them (DESIGN.md "
          "§9) cost no copy in the group; projected as the flag handshake alone (alpha: the slab transfer hidden "
          "under the pass) and, as a bound, with the transfer serialised onto the pass.\n")
    print(f"Single GPU, no decomposition: **{t1:.3f} ms** per V-cycle.\n")
    print("| proc grid | ranks | group ms / cycle | t_rank (ms) | local exchanges (model, ms) | NVLink exchanges "
          "(model, ms) | projected ms / cycle | projected efficiency t_1 / t_P | bound: fused transfers serialised |")
    print("|---|---|---|---|---|---|---|---|---|")
    for pg, P, tg, tr, tl, tk, tp, ex, by, fu, ts in rows:
        print(f"| {pg[0]}x{pg[1]}x{pg[2]} | {P} | {tg:.3f} | {tr:.3f} | {tl:.3f} | {tk:.3f} | {tp:.3f} | "
              f"{100 * t1 / tp:.1f}% | {tp + ts:.3f} ms, {100 * t1 / (tp + ts):.1f}% |")
    print("\nExchanges per cycle (fused into a pencil pass) and MB per exchange by level (rank 0):\n")
    for pg, P, tg, tr, tl, tk, tp, ex, by, fu, ts in rows:
        print(f"* {pg[0]}x{pg[1]}x{pg[2]}: " + ", ".join(f"L{l}: {e} ({f}) x {b_ / 1e6:.1f} MB" for l, (e, f, b_) in
                                                       enumerate(zip(ex, fu, by)) if e))


if __name__ == "__main__":
    main()
