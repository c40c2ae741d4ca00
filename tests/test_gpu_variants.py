"""GPU parity of the SURVEY §8(f) N4 variants beyond the paper's model problem, through the C ABI,
against the CPU oracle (bitwise, and within the north-star tolerances):

  * non-periodic boundaries (reading A22): homogeneous Dirichlet / Neumann; the library gives every
    axis a ghost shell whose domain-face bricks are filled by the mirror exchange (method of images),
    so the paper's kernels, the communication-avoiding schedule and the decompositions run unchanged;
  * variable coefficients (reading A23): div(c grad x) with face averages of the cell coefficients,
    damped Jacobi with the local diagonal, coarse c = restriction of c (one-brick kernels, SW_VARCOEF);
  * 4^3 bricks (brick_edge = 4, P:L154 Sunspot): the generic kernel family of generic.cu on the same
    layout, exchange and schedule machinery.
"""
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
    _, solver = _mg()
    nz, ny, nx = shape_zyx
    return solver.Multigrid((nx, ny, nz), num_levels=L, **kw)


def oracle_cycles(oracle_mod, b, L, ncyc, pre=12, post=12, bottom=100, **kw):
    orc = oracle_mod.OracleMG(b.shape, L, pre, post, bottom, **kw)
    orc.set_b(b)
    orc.set_x(None)
    xs, ns = [], []
    for _ in range(ncyc):
        orc.vcycle()
        xs.append(orc.get_x())
        ns.append(orc.norm())
    return xs, ns


def check_cycles(m, xs, ns):
    for c in range(len(xs)):
        m.vcycle()
        nr = m.residual_norm()
        assert abs(nr - ns[c]) <= 1e-10 * ns[c], (c, nr, ns[c])
        assert_bitwise(host(m.get_solution()), xs[c], what=f"x after cycle {c + 1}")
        assert nr == ns[c]


# ------------------------------------------------------------ boundary conditions (A22)
@pytest.mark.parametrize("bc", [1, 2])
@pytest.mark.parametrize("shape,L", [((64, 64, 64), 4), ((32, 16, 48), 2), ((128, 128, 128), 5), ((64, 64, 64), 2),
                                     ((48, 32, 64), 2)])
def test_bc_vcycle_bitwise(oracle_mod, bc, shape, L):
    """Dirichlet / Neumann V-cycles (12/12/100) bitwise equal to the oracle's after each of 2 cycles,
    x and the norm; 128^3 runs the pencil passes over the ghost-shell plan on level 0; L = 2 at 64^3
    / 48x32x64 ends on 64 / 24 bricks: the cluster-resident bottom with the mirror images."""
    b = mg_inputs.random_field(shape, 21)
    xs, ns = oracle_cycles(oracle_mod, b, L, 2, bc=bc)
    m = new(shape, L, bc=bc)
    m.set_rhs(dev(b))
    m.set_solution(None)
    check_cycles(m, xs, ns)
    m.close()


@pytest.mark.parametrize("period", [1, 2, 3, 8])
@pytest.mark.parametrize("kernels", [(0, 3), (1, 0), (2, 0), (2, 1)])
def test_bc_ca_periods_and_kernel_families_bitwise(oracle_mod, period, kernels):
    """Any CA period (the mirror ghosts lose one valid cell per sweep exactly like exchanged ones) and
    every kernel family (auto / one-brick / streaming column / one-brick two-sweep streams forced on
    every level) give the oracle's bits under a Dirichlet boundary."""
    sweep_kernel, tb = kernels
    shape = (64, 32, 32)
    b = mg_inputs.random_field(shape, 22)
    xs, ns = oracle_cycles(oracle_mod, b, 3, 2, 6, 5, 40, bc=1)
    m = new(shape, 3, pre=6, post=5, bottom=40, bc=1, ca_period=period, sweep_kernel=sweep_kernel,
            temporal_blocking=tb)
    m.set_rhs(dev(b))
    m.set_solution(None)
    check_cycles(m, xs, ns)
    m.close()


@pytest.mark.parametrize("bc", [1, 2])
@pytest.mark.parametrize("pg,n_local,L", [((2, 1, 1), (32, 32, 32), 3), ((2, 2, 2), (32, 32, 32), 3),
                                          ((1, 2, 3), (16, 32, 16), 2)])
@pytest.mark.parametrize("overlap", [True, False])
def test_bc_loopback_decomposition_bitwise(oracle_mod, bc, pg, n_local, L, overlap):
    """Decomposed runs under a non-periodic bc: no message crosses a domain face, the outer ranks'
    domain-face ghosts are mirrored (after the receives: corner ghosts reflect received bricks), and
    the result is the undecomposed oracle's bit for bit."""
    _, solver = _mg()
    gshape = (n_local[2] * pg[2], n_local[1] * pg[1], n_local[0] * pg[0])
    b = mg_inputs.random_field(gshape, 23)
    xs, ns = oracle_cycles(oracle_mod, b, L, 2, bc=bc)
    g = solver.LoopbackGroup(n_local, pg, num_levels=L, overlap=overlap, bc=bc)
    g.set_rhs([dev(mg_inputs.local_block(b, r, pg)) for r in range(g.world_size)])
    g.set_solution(None)
    for c in range(2):
        g.vcycle()
        nr = g.residual_norm()
        assert nr == ns[c]
        for r in range(g.world_size):
            assert_bitwise(host(g.get_solution(r)), mg_inputs.local_block(xs[c], r, pg), what=f"rank {r}")
    g.close()


def test_bc_chebyshev_bitwise(oracle_mod):
    """The Chebyshev smoother (A19, pointwise: commutes with the reflection) under Dirichlet."""
    shape = (64, 64, 64)
    b = mg_inputs.random_field(shape, 24)
    xs, ns = oracle_cycles(oracle_mod, b, 4, 2, smoother=1, bc=1)
    m = new(shape, 4, smoother=1, bc=1)
    m.set_rhs(dev(b))
    m.set_solution(None)
    check_cycles(m, xs, ns)
    m.close()


def test_bc_solve_matches_oracle(oracle_mod):
    """Alg 1 with the lowest Dirichlet mode as right-hand side: same cycle count, same final norm."""
    shape = (64, 64, 64)
    b = mg_inputs.dirichlet_sin_rhs(shape)
    orc = oracle_mod.OracleMG(shape, 4, bc=1)
    orc.set_b(b)
    orc.set_x(None)
    c_o, norms = orc.solve(1e-10, 20)
    m = new(shape, 4, bc=1)
    m.set_rhs(dev(b))
    m.set_solution(None)
    st, c_g, fin = m.solve(1e-10, 20)
    assert st == 0 and c_g == c_o and fin == norms[-1] and fin < 1e-10
    m.close()


def test_bc_rejected_combinations():
    """GSRB (colours not reflection-invariant) and the CG bottom (periodic null space) are refused."""
    mg, _ = _mg()
    for kw in ({"smoother": 2}, {"bottom_solver": 1}, {"bc": 3}):
        bc = kw.pop("bc", 1)
        with pytest.raises(mg.MGError):
            new((32, 32, 32), 2, bc=bc, **kw)


# ------------------------------------------------------------ variable coefficients (A23)
@pytest.mark.parametrize("bc", [0, 1, 2])
@pytest.mark.parametrize("shape,L,coef", [((64, 64, 64), 4, "random"), ((32, 16, 48), 2, "random"),
                                          ((64, 32, 64), 3, "smooth")])
def test_var_coef_vcycle_bitwise(oracle_mod, bc, shape, L, coef):
    """div(c grad x) V-cycles (12/12/100) bitwise equal to the oracle's after each of 2 cycles, under
    every boundary condition; a rough random c in [0.5, 2) and the smooth timing coefficient."""
    b = mg_inputs.random_field(shape, 31) if bc == 1 else mg_inputs.random_rhs(shape, 31)
    c = mg_inputs.random_coef(shape, 31) if coef == "random" else mg_inputs.smooth_coef(shape)
    xs, ns = oracle_cycles(oracle_mod, b, L, 2, bc=bc, coef=c)
    m = new(shape, L, bc=bc, var_coef=1)
    m.set_coefficients(dev(c))
    m.set_rhs(dev(b))
    m.set_solution(None)
    check_cycles(m, xs, ns)
    m.close()


@pytest.mark.parametrize("period", [1, 4, 8])
@pytest.mark.parametrize("ghost_mode", [0, 1])
def test_var_coef_ca_periods_and_ghost_shells_bitwise(oracle_mod, period, ghost_mode):
    """Communication avoiding with coefficient ghosts (exchanged once per setup): any CA period, with a
    self-exchanged ghost shell on every axis, gives the oracle's bits."""
    shape = (64, 32, 32)
    b = mg_inputs.random_rhs(shape, 32)
    c = mg_inputs.random_coef(shape, 32)
    xs, ns = oracle_cycles(oracle_mod, b, 3, 2, 6, 5, 40, coef=c)
    m = new(shape, 3, pre=6, post=5, bottom=40, var_coef=1, ca_period=period, ghost_mode=ghost_mode)
    m.set_coefficients(dev(c))
    m.set_rhs(dev(b))
    m.set_solution(None)
    check_cycles(m, xs, ns)
    m.close()


@pytest.mark.parametrize("bc", [0, 1, 2])
@pytest.mark.parametrize("ghost_mode,period", [(0, 0), (1, 3), (1, 8)])
def test_var_coef_column_kernel_bitwise(oracle_mod, bc, ghost_mode, period):
    """The TMA column kernel's coefficient variant (c brick + face halos staged with x and b, c k-halos
    carried like x), forced on every level (sweep_kernel = 2: plain, +r, +restriction sweeps over owned,
    ghost-shell, interior and surface ranges, and the norm) gives the oracle's bits."""
    shape = (64, 32, 96)
    b = mg_inputs.random_field(shape, 35) if bc == 1 else mg_inputs.random_rhs(shape, 35)
    c = mg_inputs.random_coef(shape, 35)
    xs, ns = oracle_cycles(oracle_mod, b, 3, 2, 5, 4, 20, bc=bc, coef=c)
    m = new(shape, 3, pre=5, post=4, bottom=20, bc=bc, var_coef=1, sweep_kernel=2, ghost_mode=ghost_mode,
            ca_period=period)
    m.set_coefficients(dev(c))
    m.set_rhs(dev(b))
    m.set_solution(None)
    check_cycles(m, xs, ns)
    m.close()


@pytest.mark.parametrize("bc", [0, 1])
@pytest.mark.parametrize("pg,n_local,L", [((2, 1, 1), (32, 32, 32), 3), ((2, 2, 2), (16, 16, 16), 2),
                                          ((1, 2, 3), (16, 32, 16), 2)])
def test_var_coef_loopback_decomposition_bitwise(oracle_mod, bc, pg, n_local, L):
    """Decomposed variable-coefficient runs (each rank restricts its c, the coefficient ghosts are
    exchanged once) reproduce the undecomposed oracle bit for bit."""
    _, solver = _mg()
    gshape = (n_local[2] * pg[2], n_local[1] * pg[1], n_local[0] * pg[0])
    b = mg_inputs.random_field(gshape, 33)
    c = mg_inputs.random_coef(gshape, 33)
    xs, ns = oracle_cycles(oracle_mod, b, L, 2, bc=bc, coef=c)
    g = solver.LoopbackGroup(n_local, pg, num_levels=L, bc=bc, var_coef=1)
    g.set_coefficients([dev(mg_inputs.local_block(c, r, pg)) for r in range(g.world_size)])
    g.set_rhs([dev(mg_inputs.local_block(b, r, pg)) for r in range(g.world_size)])
    g.set_solution(None)
    for cyc in range(2):
        g.vcycle()
        assert g.residual_norm() == ns[cyc]
        for r in range(g.world_size):
            assert_bitwise(host(g.get_solution(r)), mg_inputs.local_block(xs[cyc], r, pg), what=f"rank {r}")
    g.close()


def test_var_coef_unit_coefficient_close_to_the_paper_cycle(oracle_mod):
    """c = 1 gives the paper's V-cycle up to the rounding of the different expression (1e-12)."""
    shape = (64, 64, 64)
    b = mg_inputs.random_rhs(shape, 34)
    xs, _ = oracle_cycles(oracle_mod, b, 4, 1)
    m = new(shape, 4, var_coef=1)
    m.set_coefficients(dev(np.ones(shape)))
    m.set_rhs(dev(b))
    m.set_solution(None)
    m.vcycle()
    x = host(m.get_solution())
    assert np.abs(x - xs[0]).max() <= 1e-12 * np.abs(xs[0]).max()
    m.close()


def test_var_coef_solve_and_state_errors(oracle_mod):
    """Alg 1 with variable coefficients: same cycle count and final norm as the oracle; a V-cycle
    before the coefficients are set, and coefficients on a constant-coefficient context, are refused."""
    mg, _ = _mg()
    shape = (64, 64, 64)
    b = mg_inputs.dirichlet_sin_rhs(shape)
    c = mg_inputs.smooth_coef(shape)
    orc = oracle_mod.OracleMG(shape, 4, bc=1, coef=c)
    orc.set_b(b)
    orc.set_x(None)
    c_o, norms = orc.solve(1e-10, 20)
    m = new(shape, 4, bc=1, var_coef=1)
    m.set_rhs(dev(b))
    m.set_solution(None)
    with pytest.raises(mg.MGError):
        m.vcycle()
    m.close()
    m = new(shape, 4, bc=1, var_coef=1)
    m.set_coefficients(dev(c))
    m.set_rhs(dev(b))
    m.set_solution(None)
    st, c_g, fin = m.solve(1e-10, 20)
    assert st == 0 and c_g == c_o and fin == norms[-1] and fin < 1e-10
    m.close()
    m = new(shape, 4)
    with pytest.raises(mg.MGError):
        m.set_coefficients(dev(c))
    m.close()


# ------------------------------------------------------------ 4^3 bricks
@pytest.mark.parametrize("shape,L", [((64, 64, 64), 4), ((32, 16, 48), 3), ((64, 64, 64), 5)])
@pytest.mark.parametrize("variant", ["paper", "dirichlet", "varcoef"])
def test_brick4_vcycle_bitwise(oracle_mod, shape, L, variant):
    """4^3 bricks: V-cycles (12/12/100) bitwise equal to the oracle's after each of 2 cycles -- the
    paper's problem, Dirichlet, and variable coefficients with a Neumann boundary (the oracle does not
    know bricks: the brick edge must not change a bit)."""
    bc = {"paper": 0, "dirichlet": 1, "varcoef": 2}[variant]
    vc = variant == "varcoef"
    b = mg_inputs.random_field(shape, 41) if bc == 1 else mg_inputs.random_rhs(shape, 41)
    c = mg_inputs.random_coef(shape, 41) if vc else None
    xs, ns = oracle_cycles(oracle_mod, b, L, 2, bc=bc, coef=c)
    m = new(shape, L, bc=bc, var_coef=int(vc), brick_edge=4)
    if vc:
        m.set_coefficients(dev(c))
    m.set_rhs(dev(b))
    m.set_solution(None)
    check_cycles(m, xs, ns)
    m.close()


@pytest.mark.parametrize("fusion", [1, 2, 3])
@pytest.mark.parametrize("period", [1, 3, 4])
@pytest.mark.parametrize("ghost_mode", [0, 1])
@pytest.mark.parametrize("E", [4, 8])
def test_brick4_fusion_ca_ghosts_bitwise(oracle_mod, fusion, period, ghost_mode, E):
    """4^3 (and 8^3) bricks through the paper's kernel set (applyOp + smooth+residual + restriction +
    initZero + interpolation), the fused sweep and full fusion; CA periods up to the 4-cell ghost
    depth, with and without a self-exchanged ghost shell (the paper set's in-place smooth under the
    interior / surface overlap split: every applyOp before the first smooth): the oracle's bits."""
    shape = (32, 32, 64)
    b = mg_inputs.random_rhs(shape, 42)
    xs, ns = oracle_cycles(oracle_mod, b, 3, 2, 5, 4, 30)
    m = new(shape, 3, pre=5, post=4, bottom=30, brick_edge=E, fusion=fusion, ca_period=period,
            ghost_mode=ghost_mode)
    m.set_rhs(dev(b))
    m.set_solution(None)
    check_cycles(m, xs, ns)
    m.close()


@pytest.mark.parametrize("pg,n_local,L,bc", [((2, 1, 1), (16, 16, 16), 3, 0), ((2, 2, 2), (16, 16, 16), 2, 1),
                                             ((1, 2, 3), (8, 16, 8), 2, 0)])
def test_brick4_loopback_decomposition_bitwise(oracle_mod, pg, n_local, L, bc):
    """Decomposed 4^3-brick runs (one-brick-deep = 4-cell ghost shells exchanged through the same
    packing-free plans) reproduce the undecomposed oracle bit for bit."""
    _, solver = _mg()
    gshape = (n_local[2] * pg[2], n_local[1] * pg[1], n_local[0] * pg[0])
    b = mg_inputs.random_field(gshape, 43) if bc else mg_inputs.random_rhs(gshape, 43)
    xs, ns = oracle_cycles(oracle_mod, b, L, 2, bc=bc)
    g = solver.LoopbackGroup(n_local, pg, num_levels=L, bc=bc, brick_edge=4)
    g.set_rhs([dev(mg_inputs.local_block(b, r, pg)) for r in range(g.world_size)])
    g.set_solution(None)
    for cyc in range(2):
        g.vcycle()
        assert g.residual_norm() == ns[cyc]
        for r in range(g.world_size):
            assert_bitwise(host(g.get_solution(r)), mg_inputs.local_block(xs[cyc], r, pg), what=f"rank {r}")
    g.close()


def test_brick4_solve_matches_oracle(oracle_mod):
    """Alg 1 with 4^3 bricks: same cycle count and final norm as the oracle."""
    shape = (64, 64, 64)
    b = mg_inputs.sin_rhs(shape)
    orc = oracle_mod.OracleMG(shape, 4)
    orc.set_b(b)
    orc.set_x(None)
    c_o, norms = orc.solve(1e-10, 20)
    m = new(shape, 4, brick_edge=4)
    m.set_rhs(dev(b))
    m.set_solution(None)
    st, c_g, fin = m.solve(1e-10, 20)
    assert st == 0 and c_g == c_o and fin == norms[-1] and fin < 1e-10
    m.close()


# ------------------------------------------------------------ the variants at the bench size
@pytest.mark.parametrize("variant", ["dirichlet", "varcoef_neumann", "brick4"])
def test_full_size_512_variant_vcycle_bitwise(oracle_mod, variant):
    """512^3, L = 6, 12/12/100 (the bench workload, its launch configuration): one V-cycle of each
    variant -- Dirichlet (pencil passes over the ghost-shell plan, mirror exchanges, the resident
    bottom with domain faces), variable coefficients with Neumann faces (one-brick kernels), 4^3
    bricks (generic kernels) -- bitwise equal to the oracle's, x and the norm (the column-kernel
    norm for the 8^3 cases)."""
    import gc
    shape = (512, 512, 512)
    bc = {"dirichlet": 1, "varcoef_neumann": 2, "brick4": 0}[variant]
    vc = variant == "varcoef_neumann"
    b = mg_inputs.dirichlet_sin_rhs(shape) if bc == 1 else mg_inputs.sin_rhs(shape)
    c = mg_inputs.smooth_coef(shape) if vc else None
    xs, ns = oracle_cycles(oracle_mod, b, 6, 1, bc=bc, coef=c)
    gc.collect()
    m = new(shape, 6, bc=bc, var_coef=int(vc), brick_edge=4 if variant == "brick4" else 0)
    if vc:
        m.set_coefficients(dev(c))
    m.set_rhs(dev(b))
    m.set_solution(None)
    check_cycles(m, xs, ns)
    m.close()
    del m, xs
    gc.collect()
    torch.cuda.empty_cache()
