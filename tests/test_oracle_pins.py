"""Pins for the CPU oracle against things OTHER than itself (-m "not gpu").

Each test names the paper passage the pinned function follows and what fixes
the expected value: a closed form, an invariant, exact arithmetic, or an
independent SciPy sparse-matrix formulation of the same algorithm.  Chosen so
that a plausible slip (dropped neighbour, wrong sign of gamma, transposed
axis, wrong parent index, missing initZero, wrong h per level) fails one.
"""
import json
import os

import numpy as np
import pytest
import scipy.sparse as sp

import mg_inputs

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "paper_constants.json")


def centres(shape, h):
    nz, ny, nx = shape
    z = (np.arange(nz) + 0.5) * h
    y = (np.arange(ny) + 0.5) * h
    x = (np.arange(nx) + 0.5) * h
    return np.meshgrid(z, y, x, indexing="ij")  # Z, Y, X each (nz, ny, nx)


def mode(shape, h, k=(1, 2, 3)):
    """Periodic Fourier mode s = sin(w_x x) cos(w_y y) sin(w_z z), w_d = 2 pi k_d / L_d."""
    nz, ny, nx = shape
    Z, Y, X = centres(shape, h)
    kx, ky, kz = k
    wx, wy, wz = (2 * np.pi * kx / (nx * h), 2 * np.pi * ky / (ny * h), 2 * np.pi * kz / (nz * h))
    lam = -(4.0 / h**2) * (np.sin(wx * h / 2) ** 2 + np.sin(wy * h / 2) ** 2 + np.sin(wz * h / 2) ** 2)
    return np.sin(wx * X) * np.cos(wy * Y) * np.sin(wz * Z), lam, (wx, wy, wz)


# ---------------------------------------------------------------- golden
def test_golden_constants_match_table_iv_bytes():
    """Table IV AI = flops / algorithmic bytes; the byte counts the
    bench's roofline uses must reproduce the paper's AI."""
    g = json.load(open(GOLDEN))
    ai = g["table_iv_theoretical_ai_flop_per_byte"]
    # (flops, bytes) per point, DESIGN.md "Algorithmic bytes"
    per_pt = {"applyOp": (8, 16), "smooth": (4, 32), "smooth+residual": (6, 40),
              "restriction": (8, 72), "interpolation+increment": (8, 136)}
    for op, (fl, by) in per_pt.items():
        assert abs(fl / by - ai[op]) <= 0.006, op
    assert g["operator"]["alpha_times_h2"] == -6.0 and g["smoother"]["gamma_over_h2"] == 1.0 / 12.0


# --------------------------------------------------------------- applyOp
@pytest.mark.parametrize("q_kind", ["harmonic", "six"])
def test_apply_op_exact_on_quadratics(oracle_mod, q_kind):
    """applyOp is exact on quadratics: away from the periodic seam
    A q == Laplacian(q) exactly (dyadic h, exact arithmetic)."""
    shape = (16, 16, 16)
    h = 1.0 / 16
    Z, Y, X = centres(shape, h)
    if q_kind == "harmonic":
        q, lap = X**2 + 2 * Y**2 - 3 * Z**2 + X * Y, 0.0
    else:
        q, lap = X**2 + Y**2 + Z**2, 6.0
    Aq = oracle_mod.apply_op(q, h)
    inner = Aq[1:-1, 1:-1, 1:-1]
    assert np.all(inner == lap), np.abs(inner - lap).max()


def test_apply_op_fourier_eigenvalue(oracle_mod):
    """Periodic modes are eigenvectors: A s = lambda s, lambda = -(4/h^2) sum sin^2(w_d h/2).
    Non-cubic grid + distinct wave numbers catch transposed axes / wrong wrap."""
    shape = (16, 8, 32)  # nz, ny, nx
    h = 1.0 / 32
    s, lam, _ = mode(shape, h, k=(3, 1, 2))
    As = oracle_mod.apply_op(s, h)
    assert np.abs(As - lam * s).max() <= 1e-12 * abs(lam)


def test_apply_op_matches_kronecker_matrix_and_norm(oracle_mod):
    """Brute force: A as a Kronecker sum of 1D periodic Laplacians (SciPy);
    maxNormRes = max |b - A x| computed from that matrix."""
    shape = (6, 4, 10)
    h = 0.1
    x = mg_inputs.random_field(shape, 3)
    b = mg_inputs.random_field(shape, 4)
    A = kron_laplacian(shape, h)
    Ax_ref = (A @ x.ravel()).reshape(shape)
    Ax = oracle_mod.apply_op(x, h)
    assert np.abs(Ax - Ax_ref).max() <= 1e-13 * np.abs(Ax_ref).max()
    n_ref = np.abs(b.ravel() - A @ x.ravel()).max()
    assert abs(oracle_mod.max_norm_residual(x, b, h) - n_ref) <= 1e-13 * n_ref


# ------------------------------------------------------ smooth / residual
def test_smooth_closed_form_on_mode(oracle_mod):
    """Jacobi x := x + gamma(Ax-b), gamma=h^2/12.  With b = s (an
    eigenmode) and x0 = 0: c_{k+1} = c_k(1+gamma*lam) - gamma, so
    c_k = (1 - (1+gamma*lam)^k)/lam.  A wrong sign of gamma diverges."""
    shape = (8, 8, 8)
    h = 1.0 / 8
    s, lam, _ = mode(shape, h, k=(1, 1, 1))
    x = np.zeros(shape)
    g = h * h / 12.0
    for _ in range(100):  # the paper's 100 bottom sweeps
        x = oracle_mod.smooth(x, oracle_mod.apply_op(x, h), s, h)
    c = (1.0 - (1.0 + g * lam) ** 100) / lam
    assert np.abs(x - c * s).max() <= 1e-13 * abs(c)


def test_smooth_residual_zero_at_discrete_solution(oracle_mod):
    """r = b - Ax vanishes (to rounding) at x = b/lambda, and the x
    that smooth+residual writes equals the x smooth writes (same Ax)."""
    shape = (16, 8, 32)
    h = 1.0 / 32
    s, lam, _ = mode(shape, h, k=(2, 1, 1))
    x = s / lam
    Ax = oracle_mod.apply_op(x, h)
    xs, r = oracle_mod.smooth_residual(x, Ax, s, h)
    assert np.abs(r).max() <= 1e-13
    assert np.array_equal(xs, oracle_mod.smooth(x, Ax, s, h))
    # residual sign: b - Ax, not Ax - b
    x2 = np.zeros(shape)
    _, r2 = oracle_mod.smooth_residual(x2, oracle_mod.apply_op(x2, h), s, h)
    assert np.array_equal(r2, s)


# ---------------------------------------------------- restriction / interp
def test_restriction_constants_and_mode(oracle_mod):
    """Restriction = volume average of 8 fine cells: R 1 = 1 exactly;
    on a cell-centred mode R s_h = prod_d cos(w_d h/2) s_2h."""
    shape = (16, 8, 32)
    ones = np.ones(shape)
    assert np.array_equal(oracle_mod.restriction(ones), np.ones((8, 4, 16)))
    h = 1.0 / 32
    s, _, (wx, wy, wz) = mode(shape, h, k=(3, 1, 2))
    sc, _, _ = mode((8, 4, 16), 2 * h, k=(3, 1, 2))
    fac = np.cos(wx * h / 2) * np.cos(wy * h / 2) * np.cos(wz * h / 2)
    assert np.abs(oracle_mod.restriction(s) - fac * sc).max() <= 1e-14


def test_interpolation_constants(oracle_mod):
    """Piecewise-constant interpolation + increment: P 1 = 1, and
    the increment adds onto x."""
    xc = np.ones((4, 2, 8))
    assert np.array_equal(oracle_mod.interpolation_increment(xc, np.zeros((8, 4, 16))), np.ones((8, 4, 16)))
    x = mg_inputs.random_field((8, 4, 16), 1)
    xc = mg_inputs.random_field((4, 2, 8), 2)
    out = oracle_mod.interpolation_increment(xc, x)
    # parent of (k,j,i) is (k//2, j//2, i//2): check by explicit repeat
    up = np.repeat(np.repeat(np.repeat(xc, 2, axis=0), 2, axis=1), 2, axis=2)
    assert np.array_equal(out, x + up)


def test_restriction_interpolation_adjoint(oracle_mod):
    """Volume-weighted adjointness 8 <R r, e>_2h = <r, P e>_h (R = P^T/8), random
    non-cubic data: catches a wrong parent index or a transposed axis."""
    shape = (8, 12, 16)
    r = mg_inputs.random_field(shape, 10)
    e = mg_inputs.random_field((4, 6, 8), 11)
    Pe = oracle_mod.interpolation_increment(e, np.zeros(shape))
    lhs = 8.0 * np.sum(oracle_mod.restriction(r) * e)
    rhs = np.sum(r * Pe)
    assert abs(lhs - rhs) <= 1e-13 * np.sum(np.abs(r * Pe))


def test_restriction_of_interpolation_is_identity_bitwise(oracle_mod):
    """R(P(e)) == e bitwise with the pairwise summation order (reading A8)."""
    e = mg_inputs.random_field((4, 6, 8), 12)
    Pe = oracle_mod.interpolation_increment(e, np.zeros((8, 12, 16)))
    assert np.array_equal(oracle_mod.restriction(Pe), e)


# ------------------------------------------------------------ V-cycle
def periodic_T(n):
    T = sp.lil_matrix((n, n))
    for i in range(n):
        T[i, i] = -2.0
        T[i, (i + 1) % n] += 1.0
        T[i, (i - 1) % n] += 1.0
    return T.tocsr()


def kron_laplacian(shape, h):
    nz, ny, nx = shape
    Ix, Iy, Iz = sp.identity(nx), sp.identity(ny), sp.identity(nz)
    A = (sp.kron(Iz, sp.kron(Iy, periodic_T(nx))) + sp.kron(Iz, sp.kron(periodic_T(ny), Ix))
         + sp.kron(periodic_T(nz), sp.kron(Iy, Ix)))
    return (A / (h * h)).tocsr()


def prolong_1d(nf):
    P = sp.lil_matrix((nf, nf // 2))
    for i in range(nf):
        P[i, i // 2] = 1.0
    return P.tocsr()


def chebyshev_steps(h, s, rho):
    """The s steps of the Chebyshev smoother (reading A19) built from the textbook nodes, not from
    the oracle's index formula: the reciprocals of the Chebyshev nodes of [mu_max/rho, mu_max]
    (mu_max = 12/h^2), sorted ascending, then taken smallest, largest, second smallest, second
    largest, ... (small and large steps interleaved)."""
    mu_max = 12.0 / h**2
    lo = mu_max / rho
    nodes = [0.5 * (mu_max + lo) + 0.5 * (mu_max - lo) * np.cos(np.pi * (2 * j + 1) / (2 * s)) for j in range(s)]
    asc = sorted(1.0 / mu for mu in nodes)
    out, i, j = [], 0, s - 1
    while i <= j:
        out.append(asc[i])
        i += 1
        if i <= j:
            out.append(asc[j])
            j -= 1
    return out


def red_black_gs(A, shape):
    """One Gauss-Seidel step in red-black ordering ((i+j+k) mod 2 = 0 first) as sparse matrices:
    returns step(x, b) -> (x after the red half, x after both halves), the red half being the
    exact solve of the red rows for the red unknowns with black fixed (the 7-point stencil couples
    red only to black), the full step a sparse lower-triangular solve (D + L) x' = b - U x."""
    import scipy.sparse.linalg as spla
    nz, ny, nx = shape
    K, J, I = np.meshgrid(np.arange(nz), np.arange(ny), np.arange(nx), indexing="ij")
    colour = ((I + J + K) & 1).ravel()
    perm = np.concatenate([np.flatnonzero(colour == 0), np.flatnonzero(colour == 1)])
    nred = int(np.count_nonzero(colour == 0))
    Ap = A.tocsr()[perm][:, perm]
    lower = sp.tril(Ap, 0, format="csr")
    upper = sp.triu(Ap, 1, format="csr")

    def step(x, b):
        y = spla.spsolve_triangular(lower, b[perm] - upper @ x[perm], lower=True)
        full = np.empty_like(x)
        full[perm] = y
        half = x.copy()
        half[perm[:nred]] = y[:nred]
        return half, full

    return step


def matrix_vcycle(b0, x0, L, h0, pre, post, bottom, smoother=0, rho=6, bottom_solver=0):
    """Alg 2 written with SciPy sparse matrices: A_l Kronecker sum at h_l = 2^l h0,
    P_l = piecewise-constant prolongation, R_l = P_l^T / 8.  An independent
    formulation (different summation order) of the same algorithm.

    Variants, each in its own matrix form:
      smoother 1 (Chebyshev, reading A19): the pre / post sweeps of a level take the steps of
        `chebyshev_steps(h_l, pre|post, rho)` in order; the restricted residual is the lagged one of
        the last sweep (A5);
      smoother 2 (GSRB, reading A20): each sweep is one red-black ordered Gauss-Seidel step (sparse
        triangular solve); the restricted residual is b - A x of the x after the last red half;
      bottom_solver 1 (CG, reading A21): the coarsest problem solved exactly, x = A^+ (b - mean b)
        (dense pseudo-inverse; CG from x = 0 converges to it on the tiny coarsest grids used here).
    The bottom of the smoother variants stays damped Jacobi."""
    shapes = [tuple(s >> l for s in b0.shape) for l in range(L)]
    hs = [h0 * 2**l for l in range(L)]
    A = [kron_laplacian(shapes[l], hs[l]) for l in range(L)]
    P = [sp.kron(prolong_1d(shapes[l][0]), sp.kron(prolong_1d(shapes[l][1]), prolong_1d(shapes[l][2]))).tocsr()
         for l in range(L - 1)]
    g = [hs[l] ** 2 / 12.0 for l in range(L)]
    gs = [red_black_gs(A[l], shapes[l]) for l in range(L - 1)] if smoother == 2 else None

    def smooth(l, n):
        """n sweeps at level l; returns the residual the last one writes."""
        steps = chebyshev_steps(hs[l], n, rho) if smoother == 1 else [g[l]] * n
        r = None
        for it in range(n):
            if smoother == 2:
                half, x[l] = gs[l](x[l], b[l])
                r = b[l] - A[l] @ half
                continue
            Ax = A[l] @ x[l]
            r = b[l] - Ax
            x[l] = x[l] + steps[it] * (Ax - b[l])
        return r

    x = [None] * L
    b = [None] * L
    x[0], b[0] = x0.ravel().copy(), b0.ravel().copy()
    for l in range(L - 1):
        r = smooth(l, pre)
        b[l + 1] = (P[l].T @ r) / 8.0
        x[l + 1] = np.zeros_like(b[l + 1])
    if bottom_solver == 1:
        bb = b[L - 1] - b[L - 1].mean()
        x[L - 1] = np.linalg.pinv(A[L - 1].toarray()) @ bb
    else:
        for _ in range(bottom):
            Ax = A[L - 1] @ x[L - 1]
            x[L - 1] = x[L - 1] + g[L - 1] * (Ax - b[L - 1])
    for l in range(L - 2, -1, -1):
        x[l] = x[l] + P[l] @ x[l + 1]
        smooth(l, post)
    return x[0].reshape(b0.shape)


@pytest.mark.parametrize("shape,L,sweeps", [((16, 16, 16), 2, (3, 3, 10)), ((16, 32, 24), 3, (4, 2, 20)),
                                             ((32, 32, 32), 3, (12, 12, 100))])
def test_vcycle_matches_sparse_matrix_vcycle(oracle_mod, shape, L, sweeps):
    """The stencil V-cycle (Alg 2) equals the sparse-matrix V-cycle to
    rounding after 1 and 2 cycles (non-cubic grids, 2-3 levels)."""
    pre, post, bottom = sweeps
    h0 = mg_inputs.default_h0(shape)
    b = mg_inputs.random_rhs(shape, 0)
    mg = oracle_mod.OracleMG(shape, L, pre, post, bottom, h0)
    mg.set_b(b)
    mg.set_x(None)
    xm = np.zeros(shape)
    for _ in range(2):
        mg.vcycle()
        xm = matrix_vcycle(b, xm, L, h0, pre, post, bottom)
        xo = mg.get_x()
        assert np.abs(xo - xm).max() <= 1e-12 * np.abs(xm).max()


@pytest.mark.parametrize("smoother,shape,L,sweeps", [
    (1, (16, 32, 24), 3, (5, 3, 20)),   # Chebyshev, pre != post
    (1, (16, 16, 32), 2, (2, 7, 10)),
    (2, (16, 32, 24), 3, (3, 2, 20)),   # red-black Gauss-Seidel, pre != post
    (2, (8, 16, 16), 2, (1, 4, 10)),
])
def test_variant_vcycle_matches_sparse_matrix_vcycle(oracle_mod, smoother, shape, L, sweeps):
    """The smoother variants' V-cycles (readings A19, A20) equal the sparse-matrix V-cycle written
    with the textbook Chebyshev nodes resp. a red-black ordered Gauss-Seidel triangular solve, after 1
    and 2 cycles, on non-cubic grids with pre != post: a swapped colour order, a reversed or
    mis-counted step list, or the wrong lagged residual fails."""
    pre, post, bottom = sweeps
    h0 = mg_inputs.default_h0(shape)
    b = mg_inputs.random_rhs(shape, 1)
    mg = oracle_mod.OracleMG(shape, L, pre, post, bottom, h0, smoother=smoother, cheby_ratio=6)
    mg.set_b(b)
    mg.set_x(None)
    xm = np.zeros(shape)
    for _ in range(2):
        mg.vcycle()
        xm = matrix_vcycle(b, xm, L, h0, pre, post, bottom, smoother=smoother, rho=6)
        xo = mg.get_x()
        assert np.abs(xo - xm).max() <= 1e-11 * np.abs(xm).max()


@pytest.mark.parametrize("shape,L", [((16, 32, 24), 3), ((16, 16, 16), 3)])
def test_cg_bottom_vcycle_matches_matrix_vcycle_with_exact_bottom(oracle_mod, shape, L):
    """The CG-bottom V-cycle (reading A21) equals the matrix V-cycle whose coarsest problem is solved
    exactly (pseudo-inverse of the consistent system): 100 CG iterations from x = 0 on a <= 4x8x6
    coarsest grid reach the discrete solution (finite termination), so a wrong start, a skipped mean
    removal or a bottom that is not the CG solve fails."""
    pre, post, bottom = 3, 4, 100
    h0 = mg_inputs.default_h0(shape)
    b = mg_inputs.random_rhs(shape, 2)
    mg = oracle_mod.OracleMG(shape, L, pre, post, bottom, h0, bottom_solver=1)
    mg.set_b(b)
    mg.set_x(None)
    xm = np.zeros(shape)
    for _ in range(2):
        mg.vcycle()
        xm = matrix_vcycle(b, xm, L, h0, pre, post, bottom, bottom_solver=1)
        xo = mg.get_x()
        assert np.abs(xo - xm).max() <= 1e-9 * np.abs(xm).max()


def test_max_norm_propagates_nan(oracle_mod):
    """maxNormRes of a residual with a NaN is NaN (a diverged solve must not look
    converged: max over a set containing NaN is taken as NaN, as the GPU's bit-pattern max does),
    wherever the NaN sits (first / last cell, any thread's chunk); finite values are unaffected."""
    shape = (8, 8, 16)
    h = 1.0 / 16
    x = np.zeros(shape)
    for p in (0, 5, x.size // 2, x.size - 1):
        b = mg_inputs.random_field(shape, 7)
        b.ravel()[p] = np.nan
        assert np.isnan(oracle_mod.max_norm_residual(x, b, h)), p
    b = mg_inputs.random_field(shape, 7)
    assert oracle_mod.max_norm_residual(x, b, h) == np.abs(b).max()


def _rho(oracle_mod, N, L, b):
    mg = oracle_mod.OracleMG((N, N, N), L)
    mg.set_b(b)
    mg.set_x(None)
    norms = [mg.norm()]
    for _ in range(6):
        mg.vcycle()
        norms.append(mg.norm())
    ratios = [norms[c] / norms[c - 1] for c in range(2, 7)]
    return float(np.exp(np.mean(np.log(ratios))))


def test_vcycle_convergence_level_independent(oracle_mod):
    """V-cycle convergence factor is level independent (north_star check 4):
    fixed 8^3 coarsest grid, 12/12/100, random zero-mean b, rho(L) for
    L = 2..5 (N = 16..128) all in [0.01, 0.04] with max/min <= 1.5."""
    rhos = []
    for L in range(2, 6):
        N = 8 * 2 ** (L - 1)
        rhos.append(_rho(oracle_mod, N, L, mg_inputs.random_rhs((N, N, N), 0)))
    assert all(0.01 <= r <= 0.04 for r in rhos), rhos
    assert max(rhos) / min(rhos) <= 1.5, rhos


def test_second_order_convergence_to_continuum(oracle_mod):
    """Manufactured solution (north_star check 3): for b = sin sin sin
    the exact solution is u = -b/(12 pi^2); the converged discrete x (mean
    removed, reading A12) converges at second order: error ratios -> 4.
    Also: converged x equals the discrete solution b/lambda_h."""
    errs = []
    for N, L in ((16, 2), (32, 3), (64, 4)):
        b = mg_inputs.sin_rhs((N, N, N))
        mg = oracle_mod.OracleMG((N, N, N), L)
        mg.set_b(b)
        mg.set_x(None)
        cycles, norms = mg.solve(1e-10, 20)
        assert norms[-1] < 1e-10 and cycles <= 12
        x = mg.get_x()
        x = x - x.mean()
        h = 1.0 / N
        lam = -(4.0 / h**2) * 3 * np.sin(np.pi * h) ** 2
        assert np.abs(x - b / lam).max() <= 1e-9 * np.abs(b / lam).max()
        errs.append(np.abs(x + b / (12 * np.pi**2)).max())
    r1, r2 = errs[0] / errs[1], errs[1] / errs[2]
    assert 3.6 <= r1 <= 4.4 and 3.8 <= r2 <= 4.2, (errs, r1, r2)


def test_solve_reaches_paper_tolerance(oracle_mod):
    """Alg 1: loop until max-norm residual < 1e-10."""
    b = mg_inputs.random_rhs((32, 32, 32), 1)
    mg = oracle_mod.OracleMG((32, 32, 32), 3)
    mg.set_b(b)
    mg.set_x(None)
    cycles, norms = mg.solve(1e-10, 20)
    assert norms[-1] < 1e-10 and 1 <= cycles <= 12
    assert np.all(np.diff(norms) < 0)


def test_oracle_thread_count_invariant(oracle_mod):
    """Per-point expressions + exact max: identical bits for 1 and N threads."""
    b = mg_inputs.random_rhs((32, 32, 32), 2)
    outs = []
    nthreads = oracle_mod.get_threads()
    for t in (1, max(2, nthreads)):
        oracle_mod.set_threads(t)
        mg = oracle_mod.OracleMG((32, 32, 32), 3)
        mg.set_b(b)
        mg.set_x(None)
        mg.vcycle()
        outs.append((mg.get_x(), mg.norm()))
    oracle_mod.set_threads(nthreads)
    assert np.array_equal(outs[0][0], outs[1][0]) and outs[0][1] == outs[1][1]


def test_sweep_points_matches_full_sweep(oracle_mod):
    """The point-sampled smooth+residual used for full-size sampled parity agrees
    bitwise with applyOp + smooth+residual on the whole grid."""
    shape = (8, 12, 16)
    h = 1.0 / 16
    x = mg_inputs.random_field(shape, 5)
    b = mg_inputs.random_field(shape, 6)
    xs, r = oracle_mod.smooth_residual(x, oracle_mod.apply_op(x, h), b, h)
    pts = np.arange(x.size)
    xn_p, r_p = oracle_mod.sweep_points(x, b, h, pts)
    assert np.array_equal(xn_p, xs.ravel()) and np.array_equal(r_p, r.ravel())


# ------------------------------------------------ Chebyshev smoother (N4 variant, reading A19)
def cheb_T(s, t):
    """Chebyshev polynomial of the first kind T_s(t) for any real t (textbook closed forms)."""
    if abs(t) <= 1.0:
        return np.cos(s * np.arccos(t))
    v = np.cosh(s * np.arccosh(abs(t)))
    return v if t > 0 or s % 2 == 0 else -v


@pytest.mark.parametrize("s,rho", [(12, 6), (4, 4), (7, 10)])
def test_chebyshev_error_factor_on_modes(oracle_mod, s, rho):
    """s Chebyshev sweeps multiply the error of an eigenmode (A u = -mu u) by
    P(mu) = T_s((theta - mu/mu_max)/delta) / T_s(theta/delta), mu_max = 12/h^2,
    theta = (1+1/rho)/2, delta = (1-1/rho)/2 -- the polynomial whose roots are the
    Chebyshev nodes of [mu_max/rho, mu_max].  Computed here from the closed form of T_s,
    not from the oracle's step formula; a wrong node, scaling or missing sweep fails."""
    shape = (16, 16, 16)
    h = 1.0 / 16
    mu_max = 12.0 / h**2
    th, de = 0.5 * (1 + 1 / rho), 0.5 * (1 - 1 / rho)
    for k in [(1, 0, 0), (2, 3, 1), (4, 4, 4), (8, 8, 7)]:
        u, lam, _ = mode(shape, h, k=k)
        mu = -lam
        b = lam * u  # x* = u
        x = np.zeros(shape)
        for it in range(s):
            g = oracle_mod.chebyshev_gamma(h, s, it, rho)
            x = oracle_mod.smooth_gamma(x, oracle_mod.apply_op(x, h), b, g)
        P = cheb_T(s, (th - mu / mu_max) / de) / cheb_T(s, th / de)
        err = x - u  # = P(mu) * (x0 - u) = -P u
        assert np.abs(err + P * u).max() <= 1e-11 * max(1.0, abs(P)), (k, P)
        if mu >= mu_max / rho:  # inside the smoothing interval: damped by 1/T_s(theta/delta)
            assert abs(P) <= 1.0 / cheb_T(s, th / de) * (1 + 1e-9), (k, P)


def test_chebyshev_steps_are_node_reciprocals(oracle_mod):
    """The s steps are exactly the reciprocals of the s Chebyshev nodes (each used once),
    interleaved small/large; s = 1 with rho -> 1 is the damped-Jacobi step h^2/12."""
    h, s, rho = 1.0 / 32, 12, 6
    mu_max = 12.0 / h**2
    th, de = 0.5 * (1 + 1 / rho), 0.5 * (1 - 1 / rho)
    nodes = sorted(mu_max * (th + de * np.cos(np.pi * (2 * j + 1) / (2 * s))) for j in range(s))
    steps = [oracle_mod.chebyshev_gamma(h, s, k, rho) for k in range(s)]
    assert np.allclose(sorted(1.0 / g for g in steps), nodes, rtol=1e-14)
    assert steps[0] < steps[1] and steps[2] < steps[1]  # interleaved order
    assert oracle_mod.chebyshev_gamma(h, 1, 0, 1) == h * h / 12.0


def test_chebyshev_vcycle_converges_faster(oracle_mod):
    """With the same sweep counts the Chebyshev-smoothed V-cycle contracts faster than the
    paper's damped Jacobi (a property, not a value: the variant must not break the cycle),
    and smoother = 0 is the paper's cycle bit for bit."""
    N, L = 32, 3
    b = mg_inputs.random_rhs((N, N, N), 0)
    rj = _rho(oracle_mod, N, L, b)
    mg = oracle_mod.OracleMG((N, N, N), L, smoother=1, cheby_ratio=6)
    mg.set_b(b)
    mg.set_x(None)
    norms = [mg.norm()]
    for _ in range(6):
        mg.vcycle()
        norms.append(mg.norm())
    rc = float(np.exp(np.mean(np.log([norms[c] / norms[c - 1] for c in range(2, 7)]))))
    assert rc < rj, (rc, rj)
    a = oracle_mod.OracleMG((N, N, N), L, smoother=0)
    c = oracle_mod.OracleMG((N, N, N), L)
    for m in (a, c):
        m.set_b(b)
        m.set_x(None)
        m.vcycle()
    assert np.array_equal(a.get_x(), c.get_x())


# ------------------------------------------------ GSRB smoother (N4 variant, reading A20)
@pytest.mark.parametrize("shape", [(8, 8, 8), (4, 6, 8)])
def test_gsrb_sweep_is_red_black_ordered_gauss_seidel(oracle_mod, shape):
    """A red half-sweep then a black half-sweep (oracle_gsrb_half, colour (i+j+k) mod 2) is one
    Gauss-Seidel step in red-black ordering: (D + L) x_new = b - U x_old with the Kronecker-sum
    matrix permuted reds-first, solved by a sparse triangular solve (not the point formula)."""
    import scipy.sparse.linalg as spla
    h = 1.0 / max(shape)
    A = kron_laplacian(shape, h).tocsr()
    nz, ny, nx = shape
    K, J, I = np.meshgrid(np.arange(nz), np.arange(ny), np.arange(nx), indexing="ij")
    colour = ((I + J + K) & 1).ravel()
    perm = np.concatenate([np.flatnonzero(colour == 0), np.flatnonzero(colour == 1)])
    Ap = A[perm][:, perm]
    rng = np.random.default_rng(5)
    x0 = rng.uniform(-1, 1, shape)
    b = rng.uniform(-1, 1, shape)
    lower = sp.tril(Ap, 0, format="csr")
    upper = sp.triu(Ap, 1, format="csr")
    rhs = b.ravel()[perm] - upper @ x0.ravel()[perm]
    y = spla.spsolve_triangular(lower, rhs, lower=True)
    want = np.empty(x0.size)
    want[perm] = y
    x = x0
    for c in (0, 1):
        x, r = oracle_mod.gsrb_half(x, oracle_mod.apply_op(x, h), b, h, c)
    assert np.abs(x.ravel() - want).max() <= 1e-12 * np.abs(want).max()
    # the residual of the last half-sweep is b - A x of the x it read (after the red half)
    xr, _ = oracle_mod.gsrb_half(x0, oracle_mod.apply_op(x0, h), b, h, 0)
    assert np.array_equal(r, b - oracle_mod.apply_op(xr, h))


def test_gsrb_vcycle_converges_faster(oracle_mod):
    """GSRB-smoothed V-cycle contracts faster than the paper's damped Jacobi (property)."""
    N, L = 32, 3
    b = mg_inputs.random_rhs((N, N, N), 0)
    rj = _rho(oracle_mod, N, L, b)
    mg = oracle_mod.OracleMG((N, N, N), L, smoother=2)
    mg.set_b(b)
    mg.set_x(None)
    norms = [mg.norm()]
    for _ in range(6):
        mg.vcycle()
        norms.append(mg.norm())
    rg = float(np.exp(np.mean(np.log([norms[c] / norms[c - 1] for c in range(2, 7)]))))
    assert rg < rj, (rg, rj)


# ------------------------------------------------ CG bottom solver (N4 variant, reading A21)
def test_dot_tree_order_and_accuracy(oracle_mod):
    """The fixed-order dot product: exact on integer-valued data (any n, powers of two or not), within
    the pairwise-summation bound of the exactly rounded sum (math.fsum) on random data, and
    dependent on the order it states: a value whose sum cancels only in the pairwise pairing."""
    import math
    rng = np.random.default_rng(3)
    for n in (1, 2, 3, 7, 8, 100, 512, 4096, 4097):
        a = rng.integers(-50, 50, n).astype(np.float64)
        b = rng.integers(-50, 50, n).astype(np.float64)
        assert oracle_mod.dot_tree(a, b) == float(np.dot(a.astype(np.int64), b.astype(np.int64)))
        a, b = rng.standard_normal(n), rng.standard_normal(n)
        exact = math.fsum(a * b)
        bound = (math.ceil(math.log2(max(n, 2))) + 1) * 2.0**-53 * float(np.sum(np.abs(a * b)))
        assert abs(oracle_mod.dot_tree(a, b) - exact) <= bound
    # the tree pairs (v0 + v1) + (v2 + v3) = (1e16 + 1) + (-1e16 + 1) = 1e16 + (-1e16) = 0 (each
    # inner sum rounds the 1 away); left to right gives 1.0
    v = np.array([1e16, 1.0, -1e16, 1.0])
    assert oracle_mod.dot_tree(v, np.ones(4)) == 0.0
    assert ((1e16 + 1.0) + -1e16) + 1.0 == 1.0


def _fft_solution(b, h):
    """Exact solution of the periodic discrete Poisson problem A x = b (zero-mean x) by the FFT."""
    nz, ny, nx = b.shape
    s = [np.sin(np.pi * np.arange(n) / n) ** 2 for n in (nz, ny, nx)]
    lam = -(4.0 / h**2) * (s[0][:, None, None] + s[1][None, :, None] + s[2][None, None, :])
    bh = np.fft.fftn(b)
    lam[0, 0, 0] = 1.0
    xh = bh / lam
    xh[0, 0, 0] = 0.0
    return np.real(np.fft.ifftn(xh))


def test_cg_is_krylov_optimal(oracle_mod):
    """CG's k-th iterate is the A-orthogonal (Galerkin) projection of the solution onto the Krylov
    space span{b, Ab, ..., A^(k-1) b}: computed independently with the Kronecker-sum matrix and a QR
    basis of the Krylov vectors, for k = 1..5 on a non-cubic grid."""
    shape, h = (8, 16, 8), 1.0 / 16
    b = mg_inputs.random_rhs(shape, 11)
    A = kron_laplacian(shape, h).toarray()
    K = [b.ravel()]
    for k in range(1, 6):
        V, _ = np.linalg.qr(np.stack(K, axis=1))
        y = np.linalg.solve(V.T @ A @ V, V.T @ b.ravel())
        want = V @ y
        got = oracle_mod.cg(b, h, k).ravel()
        assert np.abs(got - want).max() <= 1e-9 * np.abs(want).max(), k
        K.append(A @ K[-1])


def test_cg_converges_to_the_discrete_solution(oracle_mod):
    """The A-norm error of the CG iterates decreases monotonically and 100 iterations reach the
    exact discrete solution (FFT) on an 8x16x16 grid to 1e-7 relative (the coarsest grids the CG
    bottom is built for have <= 4096 cells)."""
    shape, h = (8, 16, 16), 1.0 / 16
    b = mg_inputs.random_rhs(shape, 12)
    xs = _fft_solution(b, h)
    A = kron_laplacian(shape, h)
    errs = []
    for k in (2, 5, 10, 20, 40):
        e = (oracle_mod.cg(b, h, k) - xs).ravel()
        errs.append(float(-(e @ (A @ e))))  # -A is positive semi-definite
    assert all(errs[i + 1] < errs[i] for i in range(len(errs) - 1)), errs
    x = oracle_mod.cg(b, h, 100)
    assert np.abs((x - x.mean()) - xs).max() <= 1e-7 * np.abs(xs).max()


def test_cg_bottom_vcycle_contracts_faster_with_a_large_coarsest_grid(oracle_mod):
    """With a 32^3 coarsest grid, 100 Jacobi smooths barely reduce the coarse error (survey: rho ~
    0.36 per V-cycle), 100 CG iterations solve it: the CG-bottom V-cycle contracts much faster.
    bottom_solver = 0 is the paper's cycle bit for bit."""
    N, L = 64, 2
    b = mg_inputs.sin_rhs((N, N, N))

    def rho(**kw):
        m = oracle_mod.OracleMG((N, N, N), L, **kw)
        m.set_b(b)
        m.set_x(None)
        norms = [m.norm()]
        for _ in range(4):
            m.vcycle()
            norms.append(m.norm())
        return float(np.exp(np.mean(np.log([norms[c] / norms[c - 1] for c in range(2, 5)])))), m

    rj, mj = rho()
    rc, _ = rho(bottom_solver=1)
    assert rj > 0.2 and rc < 0.1, (rj, rc)
    r0, m0 = rho(bottom_solver=0)
    assert np.array_equal(m0.get_x(), mj.get_x())


def test_cg_solves_the_consistent_system(oracle_mod):
    """The periodic operator annihilates constants (reading A12), so CG runs on b - mean(b) (reading
    A21): a constant added to b changes nothing beyond rounding, and the converged residual is b's
    mean (b - A x = mean(b) to 1e-10 relative)."""
    shape, h = (16, 16, 8), 1.0 / 16
    b = mg_inputs.random_rhs(shape, 13)
    x0 = oracle_mod.cg(b, h, 100)
    x1 = oracle_mod.cg(b + 0.25, h, 100)
    assert np.abs(x1 - x0).max() <= 1e-10 * np.abs(x0).max()
    r = (b + 0.25) - oracle_mod.apply_op(x1, h)
    assert np.abs(r - 0.25).max() <= 1e-10 * np.abs(b).max()


def test_cg_bottom_vcycle_converges_with_a_16_cube_bottom(oracle_mod):
    """128^3, L = 4 (the paper's 16^3 coarsest): the CG-bottom V-cycle contracts every cycle down to
    the paper's tolerance (with b's rounding-level mean left in CG, this cycle diverged)."""
    N = 128
    m = oracle_mod.OracleMG((N, N, N), 4, bottom_solver=1)
    m.set_b(mg_inputs.sin_rhs((N, N, N)))
    m.set_x(None)
    norms = [m.norm()]
    for _ in range(7):
        m.vcycle()
        norms.append(m.norm())
    assert all(norms[c + 1] < 0.2 * norms[c] for c in range(len(norms) - 1)), norms
    assert norms[-1] < 1e-10
