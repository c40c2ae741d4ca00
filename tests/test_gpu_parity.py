"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle.

Tolerances (north_star): 1e-12 relative per operator application, 1e-10
relative on the residual norm after each V-cycle.  The design target is
BITWISE equality (same expression DAG, no FMA), so most
assertions are exact; the stated tolerances are asserted too.
"""
import os

import numpy as np
import pytest

import mg_inputs

torch = pytest.importorskip("torch")
pytestmark = [pytest.mark.gpu,
              pytest.mark.skipif(not torch.cuda.is_available(), reason="needs a CUDA device")]


def _mg():
    from paper_conf_sc_antepara0jh24_b200 import mg, solver

    return mg, solver


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def host(t):
    torch.cuda.synchronize()
    return t.cpu().numpy()


def assert_bitwise(got, want, rel=1e-12, what=""):
    scale = max(np.abs(want).max(), 1e-300)
    err = np.abs(got - want).max()
    assert err <= rel * scale, f"{what}: max err {err:.3e} (rel {err / scale:.3e})"
    assert np.array_equal(got, want), f"{what}: not bitwise (max err {err:.3e})"


def new(shape_zyx, L, **kw):
    mg, solver = _mg()
    nz, ny, nx = shape_zyx
    return solver.Multigrid((nx, ny, nz), num_levels=L, **kw)


# ------------------------------------------------------------------ per-op
@pytest.mark.parametrize("fusion", [2, 1])
@pytest.mark.parametrize("shape", [(32, 16, 48), (64, 64, 64)])
def test_smooth_residual_per_op(oracle_mod, fusion, shape):
    """applyOp + smooth+residual, fused sweep and paper kernel set."""
    mg, _ = _mg()
    m = new(shape, 1, pre=1, post=1, bottom=1)
    h = mg_inputs.default_h0(shape)
    x = mg_inputs.random_field(shape, 1)
    b = mg_inputs.random_field(shape, 2)
    m.level_set(0, mg.MG_FIELD_X, dev(x))
    m.level_set(0, mg.MG_FIELD_B, dev(b))
    mg.mg_op_smooth(m.ctx, 0, 3, 1, fusion)
    xo, ro = x, None
    for _ in range(3):
        xo, ro = oracle_mod.smooth_residual(xo, oracle_mod.apply_op(xo, h), b, h)
    assert_bitwise(host(m.level_get(0, mg.MG_FIELD_X)), xo, what="x")
    assert_bitwise(host(m.level_get(0, mg.MG_FIELD_R)), ro, what="r")
    m.close()


def test_apply_op_via_residual(oracle_mod):
    """applyOp alone: with b = 0 the residual is r = -Ax exactly."""
    mg, _ = _mg()
    shape = (16, 24, 40)
    m = new(shape, 1)
    h = mg_inputs.default_h0(shape)
    x = mg_inputs.random_field(shape, 3)
    m.level_set(0, mg.MG_FIELD_X, dev(x))
    m.level_set(0, mg.MG_FIELD_B, dev(np.zeros(shape)))
    mg.mg_op_smooth(m.ctx, 0, 1, 1, 2)
    assert_bitwise(-host(m.level_get(0, mg.MG_FIELD_R)), oracle_mod.apply_op(x, h), what="Ax")
    m.close()


def test_restriction_and_interpolation_per_op(oracle_mod):
    mg, _ = _mg()
    shape = (32, 48, 64)
    m = new(shape, 2, pre=1)
    r = mg_inputs.random_field(shape, 4)
    m.level_set(0, mg.MG_FIELD_R, dev(r))
    mg.mg_op_restrict(m.ctx, 0)
    assert_bitwise(host(m.level_get(1, mg.MG_FIELD_B)), oracle_mod.restriction(r), what="restriction")
    xf = mg_inputs.random_field(shape, 5)
    xc = mg_inputs.random_field(tuple(s // 2 for s in shape), 6)
    m.level_set(0, mg.MG_FIELD_X, dev(xf))
    m.level_set(1, mg.MG_FIELD_X, dev(xc))
    mg.mg_op_interp(m.ctx, 0)
    assert_bitwise(host(m.level_get(0, mg.MG_FIELD_X)), oracle_mod.interpolation_increment(xc, xf), what="interp")
    m.close()


@pytest.mark.parametrize("bottom_mode", [1, 2])
@pytest.mark.parametrize("shape", [(8, 8, 8), (16, 16, 16), (8, 16, 32), (8, 24, 40), (16, 32, 32), (32, 32, 32),
                                   (24, 24, 24)])
def test_bottom_solver(oracle_mod, bottom_mode, shape):
    """100 point-Jacobi sweeps: the resident kernels (one CTA for <= 8 bricks, one
    cluster of ceil(n / 8) CTAs for 9-64: 15 bricks = a part-filled second CTA, 27 and 64 = the
    replicated bottoms' sizes) and per-sweep launches."""
    mg, _ = _mg()
    m = new(shape, 1, bottom_mode=bottom_mode)
    h = mg_inputs.default_h0(shape)
    x = mg_inputs.random_field(shape, 7)
    b = mg_inputs.random_field(shape, 8)
    m.level_set(0, mg.MG_FIELD_X, dev(x))
    m.level_set(0, mg.MG_FIELD_B, dev(b))
    mg.mg_op_bottom(m.ctx, 0, 100)
    xo = x
    for _ in range(100):
        xo = oracle_mod.smooth(xo, oracle_mod.apply_op(xo, h), b, h)
    assert_bitwise(host(m.level_get(0, mg.MG_FIELD_X)), xo, what="bottom")
    m.close()


def test_residual_norm(oracle_mod):
    mg, _ = _mg()
    shape = (32, 64, 16)
    m = new(shape, 2)
    h = mg_inputs.default_h0(shape)
    x = mg_inputs.random_field(shape, 9)
    b = mg_inputs.random_field(shape, 10)
    m.set_rhs(dev(b))
    m.set_solution(dev(x))
    assert m.residual_norm() == oracle_mod.max_norm_residual(x, b, h)
    m.close()


# ------------------------------------------------------------------ V-cycle
def oracle_cycles(oracle_mod, b, L, ncyc, pre=12, post=12, bottom=100):
    orc = oracle_mod.OracleMG(b.shape, L, pre, post, bottom)
    orc.set_b(b)
    orc.set_x(None)
    xs, ns = [], []
    for _ in range(ncyc):
        orc.vcycle()
        xs.append(orc.get_x())
        ns.append(orc.norm())
    return xs, ns


def check_cycles(m, xs, ns, get=None):
    for c in range(len(xs)):
        m.vcycle()
        nr = m.residual_norm()
        assert abs(nr - ns[c]) <= 1e-10 * ns[c], (c, nr, ns[c])
        got = host(m.get_solution()) if get is None else get()
        assert_bitwise(got, xs[c], what=f"x after cycle {c + 1}")
        assert nr == ns[c]


@pytest.mark.parametrize("rhs", ["random", "sin"])
def test_vcycle_config1_bitwise(oracle_mod, rhs):
    """Config 1: 64^3, L = 4 (64 -> 8), 12/12/100; x and the residual norm after each of 3 cycles."""
    shape = (64, 64, 64)
    b = mg_inputs.random_rhs(shape, 0) if rhs == "random" else mg_inputs.sin_rhs(shape)
    xs, ns = oracle_cycles(oracle_mod, b, 4, 3)
    m = new(shape, 4)
    m.set_rhs(dev(b))
    m.set_solution(None)
    check_cycles(m, xs, ns)
    m.close()


@pytest.mark.parametrize("fusion", [1, 2, 3])
@pytest.mark.parametrize("use_graph", [True, False])
def test_vcycle_fusion_variants_bitwise(oracle_mod, fusion, use_graph):
    """Every fusion variant (paper kernel set / fused sweep / full fusion) and graph
    replay give the oracle's bits.  Non-cubic, ragged brick counts."""
    shape = (32, 48, 80)
    b = mg_inputs.random_rhs(shape, 3)
    xs, ns = oracle_cycles(oracle_mod, b, 2, 2, 4, 3, 30)
    m = new(shape, 2, pre=4, post=3, bottom=30, fusion=fusion, use_graph=use_graph)
    m.set_rhs(dev(b))
    m.set_solution(None)
    check_cycles(m, xs, ns)
    m.close()


@pytest.mark.parametrize("transport", [2, 1, 3])
@pytest.mark.parametrize("period", [0, 1, 2, 4, 8])
def test_self_exchange_ca_periods_bitwise(oracle_mod, transport, period):
    """Ghost shell on every axis with self-exchange (communication avoiding on one
    GPU): local copies, NCCL send/recv and the peer-memory kernel; any CA period (0: the
    per-level auto choice) gives the same bits."""
    shape = (64, 64, 64)
    b = mg_inputs.random_rhs(shape, 4)
    xs, ns = oracle_cycles(oracle_mod, b, 3, 2, 12, 12, 100)
    m = new(shape, 3, ghost_mode=1, transport=transport, ca_period=period)
    m.set_rhs(dev(b))
    m.set_solution(None)
    check_cycles(m, xs, ns)
    m.close()


@pytest.mark.parametrize("transport", [3, 2])
@pytest.mark.parametrize("shape,L", [((128, 128, 128), 4), ((128, 128, 256), 3)])
def test_fused_exchange_pencil_pass_bitwise(oracle_mod, transport, shape, L):
    """The exchange fused into the pencil pass: with a self-exchanged ghost shell on every
    axis, level 0's passes after an x exchange stage their ghost bricks' slabs, corners and warm-up /
    cool-down half bricks straight from the owner's field (here: this rank's own owned bricks across the
    periodic wrap) instead of running the exchange kernel -- the plan says so (exchange_fused), and x and
    the norm stay bitwise equal to the oracle's after each cycle."""
    b = mg_inputs.random_rhs(shape, 14)
    xs, ns = oracle_cycles(oracle_mod, b, L, 2, 12, 12, 100)
    m = new(shape, L, ghost_mode=1, transport=transport)
    fused = m.exchange_fused()
    counts, _ = m.exchange_plan()
    if os.environ.get("MG_NO_FUSED_EXCH"):
        assert not any(fused)
    else:
        assert fused[0] >= 5 and fused[0] <= counts[0], (fused, counts)
    m.set_rhs(dev(b))
    m.set_solution(None)
    check_cycles(m, xs, ns)
    m.close()


def test_fused_exchange_loopback_group_bitwise(oracle_mod):
    """2x2x1 loopback group of 128^3 ranks (level 0: 4096 bricks, pencil passes): every rank's fused
    level-0 passes read the neighbour ranks' fields directly (the group runs the ranks in lockstep); x of
    every rank bitwise after 2 cycles."""
    _, solver = _mg()
    pg, n_local, L = (2, 2, 1), (128, 128, 128), 4
    gshape = (n_local[2] * pg[2], n_local[1] * pg[1], n_local[0] * pg[0])
    b = mg_inputs.random_rhs(gshape, 15)
    xs, ns = oracle_cycles(oracle_mod, b, L, 2)
    g = solver.LoopbackGroup(n_local, pg, num_levels=L)
    P = pg[0] * pg[1] * pg[2]
    g.set_rhs([dev(mg_inputs.local_block(b, r, pg)) for r in range(P)])
    g.set_solution(None)
    for c in range(2):
        g.vcycle()
        nr = g.residual_norm()
        assert nr == ns[c], (c, nr, ns[c])
        for r in range(P):
            assert_bitwise(host(g.get_solution(r)), mg_inputs.local_block(xs[c], r, pg), what=f"rank {r} cycle {c}")
    g.close()


@pytest.mark.parametrize("pg,n_local,L", [((2, 1, 1), (32, 32, 32), 3), ((2, 2, 2), (32, 32, 32), 3),
                                          ((1, 2, 3), (16, 32, 16), 2), ((2, 2, 1), (16, 16, 16), 2)])
@pytest.mark.parametrize("overlap", [True, False])
def test_loopback_decomposition_bitwise(oracle_mod, pg, n_local, L, overlap):
    """A 3D decomposition run on one GPU (ranks exchange ghost bricks through the
    same plans the NCCL path uses) reproduces the undecomposed oracle bit for bit."""
    _, solver = _mg()
    gshape = (n_local[2] * pg[2], n_local[1] * pg[1], n_local[0] * pg[0])
    b = mg_inputs.random_rhs(gshape, 5)
    xs, ns = oracle_cycles(oracle_mod, b, L, 2)
    g = solver.LoopbackGroup(n_local, pg, num_levels=L, overlap=overlap)
    g.set_rhs([dev(mg_inputs.local_block(b, r, pg)) for r in range(g.world_size)])
    g.set_solution(None)
    for c in range(2):
        g.vcycle()
        nr = g.residual_norm()
        assert nr == ns[c]
        for r in range(g.world_size):
            assert_bitwise(host(g.get_solution(r)), mg_inputs.local_block(xs[c], r, pg), what=f"rank {r}")
    g.close()


def test_solve_matches_oracle(oracle_mod):
    """Alg 1 to max-norm 1e-10: same cycle count and final norm."""
    shape = (64, 64, 64)
    b = mg_inputs.sin_rhs(shape)
    orc = oracle_mod.OracleMG(shape, 4)
    orc.set_b(b)
    orc.set_x(None)
    c_o, norms = orc.solve(1e-10, 20)
    m = new(shape, 4)
    m.set_rhs(dev(b))
    m.set_solution(None)
    st, c_g, fin = m.solve(1e-10, 20)
    assert st == 0 and c_g == c_o and fin == norms[-1] and fin < 1e-10
    m.close()


@pytest.mark.parametrize("where", ["nan", "inf"])
def test_solve_reports_nonfinite_norm(oracle_mod, where):
    """A non-finite residual never looks converged (Alg 1 loops while norm > tol; a NaN fails
    both norm > tol and norm <= tol): mg_solve stops and returns MG_NOT_CONVERGED with the non-finite
    norm, as the oracle's NaN-propagating max does.  Cases: a NaN in b (norm NaN before any cycle);
    an inf in b (norm inf, the V-cycle turns x into inf - inf = NaN, the loop stops on the NaN)."""
    mg, _ = _mg()
    shape = (32, 32, 32)
    b = mg_inputs.random_rhs(shape, 1)
    b[3, 4, 5] = np.nan if where == "nan" else np.inf
    orc = oracle_mod.OracleMG(shape, 3)
    orc.set_b(b)
    orc.set_x(None)
    assert not np.isfinite(orc.norm())
    m = new(shape, 3)
    m.set_rhs(dev(b))
    m.set_solution(None)
    st, cyc, fin = m.solve(1e-10, 20)
    assert st == mg.MG_NOT_CONVERGED and not np.isfinite(fin), (st, cyc, fin)
    assert cyc < 20
    if where == "nan":
        assert cyc == 0 and np.isnan(fin)
    m.close()


@pytest.mark.parametrize("bottom_mode", [0, 1, 2, 3, 4])
@pytest.mark.parametrize("shape,L,pre,post,bottom", [
    ((64, 64, 64), 4, 12, 12, 100),   # config 1: levels 1-3 (64, 8, 1 bricks) in the cluster
    ((32, 96, 64), 3, 3, 2, 20),      # non-cubic, ragged brick counts per CTA (48 -> 6 bricks)
    ((64, 32, 96), 3, 2, 0, 5),       # post = 0
    ((32, 32, 32), 3, 1, 1, 0),       # bottom = 0
    ((64, 64, 64), 2, 2, 2, 7),       # coarsest level alone (64 bricks) in the cluster
    ((128, 64, 64), 3, 1, 2, 3),      # pre = 1 (the first sweep is the restriction sweep)
    ((128, 128, 128), 5, 12, 12, 100),  # grid solve: levels 1-4 (512 .. 1 bricks)
    ((96, 128, 64), 2, 3, 3, 9),      # coarsest level of 48 bricks: the bottom as grid sweeps
])
def test_coarse_cluster_solver_bitwise(oracle_mod, bottom_mode, shape, L, pre, post, bottom):
    """The cluster-resident coarse solve (coarse.cu, bottom_mode cluster: the deepest ghost-free
    levels in one launch, neighbours through DSMEM) and the grid-resident one (coarse_grid.cu,
    bottom_mode grid: one CTA per SM, grid barriers) against per-level launches (auto / sweeps /
    resident) and the oracle, bit for bit, 2 cycles."""
    b = mg_inputs.random_rhs(shape, 31)
    xs, ns = oracle_cycles(oracle_mod, b, L, 2, pre, post, bottom)
    m = new(shape, L, pre=pre, post=post, bottom=bottom, bottom_mode=bottom_mode)
    m.set_rhs(dev(b))
    m.set_solution(None)
    check_cycles(m, xs, ns)
    m.close()


def test_edge_cases_single_level_and_minimal_sweeps(oracle_mod):
    """L = 1 (bottom only), pre = 1, post = 0, bottom = 0."""
    for shape, L, pre, post, bottom in [((16, 8, 24), 1, 1, 1, 7), ((32, 32, 32), 3, 1, 0, 0),
                                        ((32, 32, 32), 2, 1, 1, 1)]:
        b = mg_inputs.random_rhs(shape, 6)
        xs, ns = oracle_cycles(oracle_mod, b, L, 2, pre, post, bottom)
        m = new(shape, L, pre=pre, post=post, bottom=bottom)
        m.set_rhs(dev(b))
        m.set_solution(None)
        check_cycles(m, xs, ns)
        m.close()


def test_host_api_e2e(oracle_mod):
    """mg_set_rhs_host / mg_get_solution_host (the e2e path bench.py times)."""
    shape = (32, 32, 32)
    b = mg_inputs.random_rhs(shape, 8)
    xs, ns = oracle_cycles(oracle_mod, b, 3, 1)
    m = new(shape, 3)
    bh = torch.from_numpy(b).pin_memory()
    m.set_rhs_host(bh)
    m.set_solution(None)
    m.vcycle()
    out = torch.empty(shape, dtype=torch.float64).pin_memory()
    m.get_solution_host(out)
    assert np.array_equal(out.numpy(), xs[0])
    assert m.residual_norm() == ns[0]
    m.close()


@pytest.mark.parametrize("ghost_mode", [0, 1])
def test_host_api_pipelined(oracle_mod, ghost_mode):
    """The pipelined e2e pattern bench.py times: a different b per step, uploaded on the copy
    stream (double-buffered staging) while the previous V-cycle runs, async norm + wait.  Each
    step's norm and the final x must equal the oracle driven step by step."""
    mg, _ = _mg()
    shape = (32, 32, 64)
    bs = [mg_inputs.random_rhs(shape, 20 + s) for s in range(4)]
    orc = oracle_mod.OracleMG(shape, 3, 12, 12, 100)
    orc.set_x(None)
    want = []
    for b in bs:
        orc.set_b(b)
        orc.vcycle()
        want.append(orc.norm())
    m = new(shape, 3, ghost_mode=ghost_mode)
    m.set_solution(None)
    bh = [torch.from_numpy(b).pin_memory() for b in bs]
    got = []
    m.set_rhs_host(bh[0])
    for s in range(len(bs)):
        m.vcycle()
        m.residual_norm_async()
        if s + 1 < len(bs):
            m.set_rhs_host(bh[s + 1])
        got.append(m.residual_norm_wait())
    assert got == want
    out = torch.empty(shape, dtype=torch.float64).pin_memory()
    m.get_solution_host(out)
    assert np.array_equal(out.numpy(), orc.get_x())
    with pytest.raises(RuntimeError):
        m.residual_norm_wait()  # nothing pending
    m.residual_norm_async()
    with pytest.raises(RuntimeError):
        m.residual_norm_async()  # one pending at most
    assert m.residual_norm_wait() == orc.norm()
    m.close()
    orc.close()


# ------------------------------------------------------------- full sizes
def test_full_size_512_sweep_sampled(oracle_mod):
    """512^3 (the bench workload), level-0 fused sweep: 20k sampled points vs the
    oracle's point evaluation, plus r."""
    mg, _ = _mg()
    shape = (512, 512, 512)
    m = new(shape, 6)
    h = mg_inputs.default_h0(shape)
    x = mg_inputs.random_field(shape, 12)
    b = mg_inputs.sin_rhs(shape)
    m.level_set(0, mg.MG_FIELD_X, dev(x))
    m.level_set(0, mg.MG_FIELD_B, dev(b))
    mg.mg_op_smooth(m.ctx, 0, 1, 1, 2)
    rng = np.random.default_rng(0)
    pts = rng.integers(0, x.size, 20000)
    pts = np.concatenate([pts, [0, x.size - 1, 511, 512 * 512 - 1]])  # corners (periodic wrap)
    xn, r = oracle_mod.sweep_points(x, b, h, pts)
    gx = host(m.level_get(0, mg.MG_FIELD_X)).ravel()[pts]
    gr = host(m.level_get(0, mg.MG_FIELD_R)).ravel()[pts]
    assert np.array_equal(gx, xn) and np.array_equal(gr, r)
    m.close()


def test_full_size_512_pencil_pass_bitwise(oracle_mod):
    """512^3 (the bench workload, launch configuration of bench.py: the 2x2-brick pencil pass over
    888 CTAs, 6 per SM): one two-sweep pass with r, every point against the oracle's two sweeps."""
    mg, _ = _mg()
    shape = (512, 512, 512)
    m = new(shape, 6)
    h = mg_inputs.default_h0(shape)
    x = mg_inputs.random_field(shape, 26)
    b = mg_inputs.sin_rhs(shape)
    m.level_set(0, mg.MG_FIELD_X, dev(x))
    m.level_set(0, mg.MG_FIELD_B, dev(b))
    mg.mg_op_smooth(m.ctx, 0, 2, 1, 2)
    gx = host(m.level_get(0, mg.MG_FIELD_X))
    gr = host(m.level_get(0, mg.MG_FIELD_R))
    m.close()
    xo, ro = x, None
    for _ in range(2):
        xo, ro = oracle_mod.smooth_residual(xo, oracle_mod.apply_op(xo, h), b, h)
    assert_bitwise(gx, xo, what="x")
    assert_bitwise(gr, ro, what="r")


@pytest.mark.slow
def test_full_size_512_vcycle_bitwise(oracle_mod):
    """512^3, L = 6, 12/12/100 (bench configuration): one full V-cycle bitwise + norm."""
    shape = (512, 512, 512)
    b = mg_inputs.sin_rhs(shape)
    xs, ns = oracle_cycles(oracle_mod, b, 6, 1)
    m = new(shape, 6)
    m.set_rhs(dev(b))
    m.set_solution(None)
    check_cycles(m, xs, ns)
    m.close()


@pytest.mark.slow
def test_full_size_decomposed_2x1x1_vs_oracle(oracle_mod):
    """Config 4's per-rank size in a decomposition, against the oracle itself: 1024 x 512 x 512 global
    as a 2x1x1 loopback (512^3 per rank, L = 6: ghost shells on x, exchanges through the NCCL plans,
    pencil passes over the stored box, the replicated bottom), one V-cycle: x of every rank and the
    residual norm bit for bit equal to the undecomposed oracle (about 5 s of oracle time)."""
    import torch

    _, solver = _mg()
    torch.cuda.empty_cache()
    pg, L = (2, 1, 1), 6
    nl = (512, 512, 512)
    G = (512, 512, 1024)  # (nz, ny, nx)
    b = mg_inputs.sin_rhs(G)
    xs, ns = oracle_cycles(oracle_mod, b, L, 1)
    g = solver.LoopbackGroup(nl, pg, num_levels=L)
    try:
        g.set_rhs([dev(mg_inputs.local_block(b, r, pg)) for r in range(2)])
        g.set_solution(None)
        g.vcycle()
        assert g.residual_norm() == ns[0]
        for r in range(2):
            assert_bitwise(host(g.get_solution(r)), mg_inputs.local_block(xs[0], r, pg), what=f"rank {r}")
    finally:
        g.close()
        del g
        torch.cuda.empty_cache()


@pytest.mark.parametrize("pg", [(2, 1, 1), (2, 2, 1), (2, 2, 2)])
def test_config5_1024_decomposition_invariant(pg):
    """Config 5 at its full size (1024^3 total, L = 7, global coarsest 16^3 for every P): one V-cycle on
    one rank and on the P = 2 / 4 / 8 loopback decompositions (down to 512^3 per rank: ghost shells,
    local exchanges
    through the NCCL plans, pencil passes over the stored box, the replicated bottom) give bit-identical
    x and the same residual norm (decomposition invariance; the oracle's own cycle at this
    size is checked by the 512^3 tests and the invariance chain)."""
    import torch

    _, solver = _mg()
    torch.cuda.empty_cache()  # (the previous case's cached blocks)
    G = (1024, 1024, 1024)
    P = pg[0] * pg[1] * pg[2]
    nl = (1024 // pg[0], 1024 // pg[1], 1024 // pg[2])  # (nx, ny, nz) per rank
    blocks = [torch.from_numpy(mg_inputs.local_sin_rhs(G, r, pg)) for r in range(P)]

    def sl(r):
        cx, cy, cz = mg_inputs.rank_coords(r, pg)
        return (slice(cz * nl[2], (cz + 1) * nl[2]), slice(cy * nl[1], (cy + 1) * nl[1]),
                slice(cx * nl[0], (cx + 1) * nl[0]))

    b = torch.empty(G, dtype=torch.float64, device="cuda")
    for r, blk in enumerate(blocks):
        b[sl(r)] = blk.cuda()
    m = new(G, 7)
    m.set_rhs(b)
    m.set_solution(None)
    m.vcycle()
    n1 = m.residual_norm()
    x1 = m.get_solution()
    m.close()
    del b
    torch.cuda.empty_cache()
    g = solver.LoopbackGroup(nl, pg, num_levels=7)
    g.set_rhs([blk.cuda() for blk in blocks])
    g.set_solution(None)
    g.vcycle()
    assert g.residual_norm() == n1
    try:
        for r in range(P):
            assert torch.equal(g.get_solution(r), x1[sl(r)]), f"rank {r}"
    finally:
        g.close()
        del g, x1
        torch.cuda.empty_cache()


# ------------------------------------------------- streaming (column) kernel
@pytest.mark.parametrize("tb", [0, 1, 3])
@pytest.mark.parametrize("fusion", [2, 3])
@pytest.mark.parametrize("ghost_mode,period", [(0, 0), (1, 1), (1, 3), (1, 8)])
def test_streaming_kernel_forced_bitwise(oracle_mod, fusion, ghost_mode, period, tb):
    """sweep_kernel = 2 forces the TMA-streamed column kernel (tb = 0) or a two-sweep
    kernel (tb = 1: CTA streams, tb = 3: 2x2-brick pencils) on every level (plain, +r and +restriction variants; owned,
    owned+ghost, interior and surface ranges)."""
    shape = (64, 32, 96)
    b = mg_inputs.random_rhs(shape, 13)
    xs, ns = oracle_cycles(oracle_mod, b, 3, 2, 5, 4, 20)
    m = new(shape, 3, pre=5, post=4, bottom=20, fusion=fusion, ghost_mode=ghost_mode, ca_period=period,
            sweep_kernel=2, temporal_blocking=tb)
    m.set_rhs(dev(b))
    m.set_solution(None)
    check_cycles(m, xs, ns)
    m.close()


@pytest.mark.parametrize("tb", [0, 1, 3])
@pytest.mark.parametrize("pg", [(2, 2, 2), (2, 1, 1)])
def test_streaming_kernel_loopback_bitwise(oracle_mod, pg, tb):
    _, solver = _mg()
    n_local = (32, 32, 32)
    gshape = (32 * pg[2], 32 * pg[1], 32 * pg[0])
    b = mg_inputs.random_rhs(gshape, 14)
    xs, ns = oracle_cycles(oracle_mod, b, 3, 1)
    g = solver.LoopbackGroup(n_local, pg, num_levels=3, sweep_kernel=2, temporal_blocking=tb)
    g.set_rhs([dev(mg_inputs.local_block(b, r, pg)) for r in range(g.world_size)])
    g.set_solution(None)
    g.vcycle()
    assert g.residual_norm() == ns[0]
    for r in range(g.world_size):
        assert_bitwise(host(g.get_solution(r)), mg_inputs.local_block(xs[0], r, pg), what=f"rank {r}")
    g.close()


def test_vcycle_config2_256_bitwise(oracle_mod):
    """Config 2: 256^3 on one GPU, L = 6 (256 -> 8), 12/12/100: the auto kernel choice
    (streaming on levels 0-1) gives the oracle's bits for 2 cycles."""
    shape = (256, 256, 256)
    b = mg_inputs.sin_rhs(shape)
    xs, ns = oracle_cycles(oracle_mod, b, 6, 2)
    m = new(shape, 6)
    m.set_rhs(dev(b))
    m.set_solution(None)
    check_cycles(m, xs, ns)
    m.close()


# ------------------------------------------------- two sweeps per pass (temporal blocking)
@pytest.mark.parametrize("tb", [1, 3])
@pytest.mark.parametrize("n", [2, 3, 5])
@pytest.mark.parametrize("shape,ghost_mode", [((64, 32, 96), 0), ((32, 48, 64), 1), ((40, 24, 56), 0)])
def test_two_sweep_pass_per_op(oracle_mod, n, shape, ghost_mode, tb):
    """OP_SWEEP2 (x0 -> x1 -> x2 in one pass, redundant x1 on the side faces) equals
    n separate sweeps of the oracle bit for bit, including r of the last sweep."""
    mg, _ = _mg()
    m = new(shape, 1, pre=1, post=1, bottom=1, sweep_kernel=2, ghost_mode=ghost_mode, temporal_blocking=tb)
    h = mg_inputs.default_h0(shape)
    x = mg_inputs.random_field(shape, 21)
    b = mg_inputs.random_field(shape, 22)
    m.level_set(0, mg.MG_FIELD_X, dev(x))
    m.level_set(0, mg.MG_FIELD_B, dev(b))
    mg.mg_op_smooth(m.ctx, 0, n, 1, 2)
    xo, ro = x, None
    for _ in range(n):
        xo, ro = oracle_mod.smooth_residual(xo, oracle_mod.apply_op(xo, h), b, h)
    assert_bitwise(host(m.level_get(0, mg.MG_FIELD_X)), xo, what="x")
    assert_bitwise(host(m.level_get(0, mg.MG_FIELD_R)), ro, what="r")
    m.close()


@pytest.mark.parametrize("n", [2, 3, 4])
@pytest.mark.parametrize("shape,ghost_mode", [((16, 64, 64), 0), ((24, 64, 96), 0), ((96, 64, 128), 0),
                                              ((32, 64, 64), 0), ((64, 48, 32), 1), ((8, 16, 16), 0)])
@pytest.mark.parametrize("tb", [3])
def test_pencil_pass_work_splits(oracle_mod, n, shape, ghost_mode, tb):
    """tb = 3 (2x2-brick pencil chunk streams): whole tile columns per CTA, several columns per CTA,
    columns cut into pieces across CTAs, a ghost-shell level and a single-layer level all give the
    oracle's bits for x and r (n sweeps: n // 2 pencil passes plus a single sweep if n is odd)."""
    mg, _ = _mg()
    m = new(shape, 1, pre=1, post=1, bottom=1, sweep_kernel=2, ghost_mode=ghost_mode, temporal_blocking=tb)
    h = mg_inputs.default_h0(shape)
    x = mg_inputs.random_field(shape, 24)
    b = mg_inputs.random_field(shape, 25)
    m.level_set(0, mg.MG_FIELD_X, dev(x))
    m.level_set(0, mg.MG_FIELD_B, dev(b))
    mg.mg_op_smooth(m.ctx, 0, n, 1, 2)
    xo, ro = x, None
    for _ in range(n):
        xo, ro = oracle_mod.smooth_residual(xo, oracle_mod.apply_op(xo, h), b, h)
    assert_bitwise(host(m.level_get(0, mg.MG_FIELD_X)), xo, what="x")
    assert_bitwise(host(m.level_get(0, mg.MG_FIELD_R)), ro, what="r")
    m.close()


def test_vcycle_512_grid_coarse_bitwise(oracle_mod):
    """At the bench size (512^3, L = 6) the grid-resident coarse solve (levels 2-5) and the
    per-level launches give identical x after one V-cycle (bitwise over the whole field) and the
    same residual norm."""
    import torch

    shape = (512, 512, 512)
    b = mg_inputs.sin_rhs(shape)
    out = []
    for bm in (0, 4):
        m = new(shape, 6, bottom_mode=bm)
        m.set_rhs(dev(b))
        m.set_solution(None)
        m.vcycle()
        out.append((m.get_solution(), m.residual_norm()))
        m.close()
        torch.cuda.empty_cache()
    assert torch.equal(out[0][0], out[1][0])
    assert out[0][1] == out[1][1]


@pytest.mark.parametrize("tb", [0, 1, 3])
def test_temporal_blocking_on_off_bitwise(oracle_mod, tb):
    """The V-cycle with and without temporal blocking gives the oracle's bits (256^3, L = 6,
    where levels 0 and 1 stream; 12/12/100)."""
    shape = (256, 256, 256)
    b = mg_inputs.random_rhs(shape, 23)
    xs, ns = oracle_cycles(oracle_mod, b, 6, 1)
    m = new(shape, 6, temporal_blocking=tb)
    m.set_rhs(dev(b))
    m.set_solution(None)
    check_cycles(m, xs, ns)
    m.close()


@pytest.mark.parametrize("shape,L,pre,post,bottom", [
    ((64, 64, 64), 4, 12, 12, 100),   # coarsest 8^3: one brick
    ((128, 128, 128), 4, 12, 12, 100),  # coarsest 16^3: 8 bricks, the paper's bottom size
    ((24, 16, 8), 1, 0, 0, 37),       # bottom only, 6 bricks: a non-power-of-two dot-product length
    ((64, 32, 16), 2, 3, 2, 60),      # non-cubic, 8 bricks
])
def test_cg_bottom_vcycle_bitwise(oracle_mod, shape, L, pre, post, bottom):
    """bottom_solver = 1: CG bottom (reading A21) from x = 0 with the fixed-order dot product, bit for
    bit with the oracle's CG V-cycle (2 cycles)."""
    b = mg_inputs.random_rhs(shape, 43)
    orc = oracle_mod.OracleMG(shape, L, pre, post, bottom, bottom_solver=1)
    orc.set_b(b)
    orc.set_x(None)
    xs, ns = [], []
    for _ in range(2):
        orc.vcycle()
        xs.append(orc.get_x())
        ns.append(orc.norm())
    m = new(shape, L, pre=pre, post=post, bottom=bottom, bottom_solver=1)
    m.set_rhs(dev(b))
    m.set_solution(None)
    check_cycles(m, xs, ns)
    m.close()


def test_cg_bottom_replicated_loopback_bitwise(oracle_mod):
    """CG bottom on the replicated global coarsest grid of a 2x2x2 loopback decomposition (8^3 per
    rank: 16^3 globally, 8 bricks), bit for bit with the undecomposed oracle."""
    _, solver = _mg()
    pg, n_local, L = (2, 2, 2), (32, 32, 32), 3
    gshape = (n_local[2] * pg[2], n_local[1] * pg[1], n_local[0] * pg[0])
    b = mg_inputs.random_rhs(gshape, 44)
    orc = oracle_mod.OracleMG(gshape, L, bottom_solver=1)
    orc.set_b(b)
    orc.set_x(None)
    g = solver.LoopbackGroup(n_local, pg, num_levels=L, bottom_solver=1)
    g.set_rhs([dev(mg_inputs.local_block(b, r, pg)) for r in range(g.world_size)])
    g.set_solution(None)
    for c in range(2):
        orc.vcycle()
        g.vcycle()
        assert g.residual_norm() == orc.norm()
        for r in range(g.world_size):
            assert_bitwise(host(g.get_solution(r)), mg_inputs.local_block(orc.get_x(), r, pg), what=f"rank {r}")
    g.close()


@pytest.mark.parametrize("mode", ["loopback", "self-local", "self-nccl"])
def test_pencil_exchange_overlap_bitwise(oracle_mod, mode, monkeypatch):
    """Pencil passes on ghost-shell levels with the exchange overlapped (MG_PENCIL_OVERLAP=1: the
    units that read no ghost brick run while the exchange fills the ghosts, the rest after it):
    oracle bits for a 2x2x2 loopback decomposition and for the self-exchanged ghost shell over local
    copies and over NCCL (send/recv on the comm stream inside the captured graph; the replicated
    bottom's ncclAllGather)."""
    monkeypatch.setenv("MG_PENCIL_OVERLAP", "1")
    mg, solver = _mg()
    if mode.startswith("self"):
        shape = (128, 128, 128)
        b = mg_inputs.random_rhs(shape, 37)
        xs, ns = oracle_cycles(oracle_mod, b, 4, 2)
        m = new(shape, 4, ghost_mode=1, ca_period=8, transport=1 if mode == "self-nccl" else 2)
        m.set_rhs(dev(b))
        m.set_solution(None)
        check_cycles(m, xs, ns)
        m.close()
        return
    pg, n_local = (2, 2, 2), (64, 64, 64)
    gshape = (n_local[2] * pg[2], n_local[1] * pg[1], n_local[0] * pg[0])
    b = mg_inputs.random_rhs(gshape, 38)
    xs, ns = oracle_cycles(oracle_mod, b, 3, 2)
    g = solver.LoopbackGroup(n_local, pg, num_levels=3)
    g.set_rhs([dev(mg_inputs.local_block(b, r, pg)) for r in range(g.world_size)])
    g.set_solution(None)
    for c in range(2):
        g.vcycle()
        assert g.residual_norm() == ns[c]
        for r in range(g.world_size):
            assert_bitwise(host(g.get_solution(r)), mg_inputs.local_block(xs[c], r, pg), what=f"rank {r}")
    g.close()


@pytest.mark.parametrize("launch_pdl", [1, 2])
@pytest.mark.parametrize("use_graph", [True, False])
def test_programmatic_dependent_launch_on_off_bitwise(oracle_mod, launch_pdl, use_graph):
    """Programmatic dependent launch on (1) and off (2), captured in the V-cycle graph or launched
    op by op, gives the oracle's bits: 128^3, L = 5 (pencil passes on levels 0-1, one-brick kernels,
    the resident bottom), 12/12/100, two cycles."""
    shape = (128, 128, 128)
    b = mg_inputs.random_rhs(shape, 29)
    xs, ns = oracle_cycles(oracle_mod, b, 5, 2)
    m = new(shape, 5, launch_pdl=launch_pdl, use_graph=use_graph)
    m.set_rhs(dev(b))
    m.set_solution(None)
    check_cycles(m, xs, ns)
    m.close()


# ------------------------------------------------- Chebyshev smoother variant (N4, reading A19)
@pytest.mark.parametrize("kw", [dict(), dict(temporal_blocking=0), dict(fusion=1), dict(temporal_blocking=1),
                                dict(bottom_mode=1), dict(bottom_mode=3), dict(bottom_mode=4),
                                dict(ghost_mode=1, ca_period=4),
                                dict(sweep_kernel=2), dict(cheby_ratio=10), dict(temporal_blocking=3),
                                dict(temporal_blocking=3, sweep_kernel=2), dict(temporal_blocking=1, sweep_kernel=2)])
def test_chebyshev_smoother_vcycle_bitwise(oracle_mod, kw):
    """smoother = 1: per-sweep Chebyshev steps in every kernel that sweeps (single, two-sweep
    passes, paper kernel set, cluster coarse solve, ghost sweeps), bit for bit with the oracle's
    Chebyshev V-cycle; the bottom stays damped Jacobi."""
    shape = (64, 64, 64)
    rho = kw.get("cheby_ratio", 6)
    b = mg_inputs.random_rhs(shape, 41)
    orc = oracle_mod.OracleMG(shape, 4, 12, 12, 100, smoother=1, cheby_ratio=rho)
    orc.set_b(b)
    orc.set_x(None)
    xs, ns = [], []
    for _ in range(2):
        orc.vcycle()
        xs.append(orc.get_x())
        ns.append(orc.norm())
    m = new(shape, 4, smoother=1, **kw)
    m.set_rhs(dev(b))
    m.set_solution(None)
    check_cycles(m, xs, ns)
    m.close()
    orc.close()


def test_chebyshev_smoother_loopback_bitwise(oracle_mod):
    _, solver = _mg()
    pg, n_local = (2, 2, 1), (32, 32, 32)
    gshape = (32, 64, 64)
    b = mg_inputs.random_rhs(gshape, 42)
    orc = oracle_mod.OracleMG(gshape, 3, 12, 12, 100, smoother=1, cheby_ratio=6)
    orc.set_b(b)
    orc.set_x(None)
    orc.vcycle()
    g = solver.LoopbackGroup(n_local, pg, num_levels=3, smoother=1)
    g.set_rhs([dev(mg_inputs.local_block(b, r, pg)) for r in range(g.world_size)])
    g.set_solution(None)
    g.vcycle()
    assert g.residual_norm() == orc.norm()
    for r in range(g.world_size):
        assert_bitwise(host(g.get_solution(r)), mg_inputs.local_block(orc.get_x(), r, pg), what=f"rank {r}")
    g.close()
    orc.close()


# ------------------------------------------------- red-black Gauss-Seidel variant (N4, reading A20)
@pytest.mark.parametrize("kw", [dict(), dict(temporal_blocking=0), dict(fusion=1), dict(fusion=2),
                                dict(temporal_blocking=1), dict(bottom_mode=1), dict(ghost_mode=1, ca_period=3),
                                dict(ghost_mode=1, ca_period=8), dict(sweep_kernel=2), dict(temporal_blocking=3),
                                dict(temporal_blocking=3, sweep_kernel=2), dict(temporal_blocking=1, sweep_kernel=2)])
def test_gsrb_smoother_vcycle_bitwise(oracle_mod, kw):
    """smoother = 2: every pre / post sweep is a red then a black half-sweep (step h^2/6) in the
    single-sweep, two-sweep (red + black in one pass), paper-set and ghost-shell schedules; bit
    for bit with the oracle's GSRB V-cycle."""
    shape = (64, 64, 64)
    b = mg_inputs.random_rhs(shape, 43)
    orc = oracle_mod.OracleMG(shape, 4, 12, 12, 100, smoother=2)
    orc.set_b(b)
    orc.set_x(None)
    xs, ns = [], []
    for _ in range(2):
        orc.vcycle()
        xs.append(orc.get_x())
        ns.append(orc.norm())
    m = new(shape, 4, smoother=2, **kw)
    m.set_rhs(dev(b))
    m.set_solution(None)
    check_cycles(m, xs, ns)
    m.close()
    orc.close()


def test_gsrb_fused_exchange_bitwise(oracle_mod):
    """Red-black Gauss-Seidel with a self-exchanged ghost shell at 128^3 (level 0: pencil passes of a red
    and a black half-sweep): the passes after an x exchange stage their ghost bricks from the owner's
    field (the fused exchange, colour-masked variant); bit for bit with the oracle's GSRB V-cycle."""
    shape = (128, 128, 128)
    b = mg_inputs.random_rhs(shape, 45)
    orc = oracle_mod.OracleMG(shape, 4, 12, 12, 100, smoother=2)
    orc.set_b(b)
    orc.set_x(None)
    xs, ns = [], []
    for _ in range(2):
        orc.vcycle()
        xs.append(orc.get_x())
        ns.append(orc.norm())
    m = new(shape, 4, smoother=2, ghost_mode=1, transport=3)
    if not os.environ.get("MG_NO_FUSED_EXCH"):
        assert m.exchange_fused()[0] >= 5, m.exchange_fused()
    m.set_rhs(dev(b))
    m.set_solution(None)
    check_cycles(m, xs, ns)
    m.close()
    orc.close()


def test_gsrb_smoother_loopback_bitwise(oracle_mod):
    _, solver = _mg()
    pg, n_local = (2, 1, 2), (32, 32, 32)
    gshape = (64, 32, 64)
    b = mg_inputs.random_rhs(gshape, 44)
    orc = oracle_mod.OracleMG(gshape, 3, 12, 12, 100, smoother=2)
    orc.set_b(b)
    orc.set_x(None)
    orc.vcycle()
    g = solver.LoopbackGroup(n_local, pg, num_levels=3, smoother=2)
    g.set_rhs([dev(mg_inputs.local_block(b, r, pg)) for r in range(g.world_size)])
    g.set_solution(None)
    g.vcycle()
    assert g.residual_norm() == orc.norm()
    for r in range(g.world_size):
        assert_bitwise(host(g.get_solution(r)), mg_inputs.local_block(orc.get_x(), r, pg), what=f"rank {r}")
    g.close()
    orc.close()


@pytest.mark.parametrize("transport", [2, 1, 3])
def test_exchange_plan_and_timing_keep_the_bits(oracle_mod, transport):
    """mg_exchange_plan / mg_exchange_time (the bench's exchange block): a self-exchanged ghost shell
    on every axis has exchanges on every level, the timing runs the V-cycle's own transport (local
    copies / NCCL), and refreshing the ghosts in between leaves the V-cycle bitwise on the oracle."""
    mg, _ = _mg()
    shape = (64, 64, 64)
    b = mg_inputs.random_rhs(shape, 41)
    xs, ns = oracle_cycles(oracle_mod, b, 3, 2)
    m = new(shape, 3, ghost_mode=1, transport=transport)
    m.set_rhs(dev(b))
    m.set_solution(None)
    counts, nbytes = m.exchange_plan()
    # (the coarsest level runs the replicated bottom: its b is all-gathered, no ghost exchange)
    assert all(c > 0 for c in counts[:-1]) and counts[-1] == 0 and all(v > 0 for v in nbytes)
    # NCCL: one exchange of level 0 fills the whole one-brick ghost shell, 10^3 - 8^3 bricks of 4 KiB
    # (a surface brick goes to every face / edge / corner direction it borders); the copy transports
    # (local, peer) at level 0's period 2 copy only the ghost cells within 2 of the owned box
    if transport == 1:
        assert nbytes[0] == (10**3 - 8**3) * 4096
    else:
        assert nbytes[0] == (68**3 - 64**3) * 8
    # level 1 (period 8 = the brick edge): whole bricks on every transport
    assert nbytes[1] == (6**3 - 4**3) * 4096
    m.vcycle()
    for l in range(3):
        assert m.exchange_time(l, 3) > 0
    nr = m.residual_norm()
    assert nr == ns[0]
    assert_bitwise(host(m.get_solution()), xs[0], what="x after cycle 1")
    m.vcycle()
    assert m.residual_norm() == ns[1]
    assert_bitwise(host(m.get_solution()), xs[1], what="x after cycle 2")
    m.close()


@pytest.mark.parametrize("args", ["32 32 32 2 1 1 3 2 0", "16 16 16 2 2 1 2 2 0", "32 32 32 2 1 1 3 1 1",
                                  "16 16 16 2 2 2 2 2 0", "32 32 32 2 1 1 3 2 0 1", "16 16 32 2 2 2 2 2 1 2",
                                  "128 128 128 2 1 1 3 2 0 0 pencil-overlap", "128 128 128 2 2 1 3 2 0 0 pencil-overlap",
                                  "128 128 128 2 2 1 3 2 0", "128 128 128 2 2 2 3 2 0"])
def test_peer_transport_multiprocess_bitwise(args):
    """The peer-memory transport between PROCESSES (CUDA IPC mappings, device-side ready/done flags, the
    norm's max and the replicated bottom's gather over peer memory): torchrun starts one process per
    rank -- on one GPU they share the device, which CUDA IPC allows -- and every rank's x and the global
    norm equal the oracle bit for bit (tools/peer_check.py)."""
    import os
    import socket
    import subprocess
    import sys

    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    a = args.split()
    env = dict(os.environ)
    if a[-1] == "pencil-overlap":  # the pencil passes' exchange overlap (units without ghosts first)
        a = a[:-1]
        env["MG_PENCIL_OVERLAP"] = "1"
    nproc = int(a[3]) * int(a[4]) * int(a[5])
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={nproc}",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.join(root, "tools", "peer_check.py"), *a]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=600, cwd=root, env=env)
    assert r.returncode == 0 and "peer_check ok" in r.stdout, (r.stdout[-2000:], r.stderr[-3000:])
    if "MG_PENCIL_OVERLAP" not in env and not env.get("MG_NO_FUSED_EXCH") and int(a[0]) >= 128:
        # level 0's passes take the fused exchange: a handshake kernel, then slabs from the peers' fields
        assert "fused exchanges per level [0, " not in r.stdout and "fused exchanges per level [" in r.stdout, r.stdout
