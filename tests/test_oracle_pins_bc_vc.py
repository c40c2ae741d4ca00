"""Pins for the oracle's boundary-condition and variable-coefficient variants (-m "not gpu").

SURVEY §8(f) N4 "non-periodic BCs and variable coefficients" ("nonconstant coefficients ...
domain boundary conditions", P:L148 the model problem they generalise).  DESIGN.md readings:
  A22  homogeneous Dirichlet (bc = 1) / Neumann (bc = 2) on the faces of the cell-centred grid: the
       neighbour across a domain face is -x_p / +x_p, on every level;
  A23  A x = div(c grad x): (A x)_p = (1/h^2) sum_n ((c_p + c_n)/2) (x_n - x_p), damped Jacobi with
       the local diagonal, gamma_p = (h^2/2) / sum_n (c_p + c_n)/2, coarse c = restriction of c.
Each pin checks the oracle against something other than itself: closed-form eigenpairs, the
method of images (Dirichlet / Neumann on N^3 IS the periodic problem on the odd / even extension
to (2N)^3, whose oracle is pinned in test_oracle_pins.py), an independent sparse-matrix assembly
from face fluxes, exact invariants and second-order convergence to continuum solutions.
"""
import numpy as np
import pytest
import scipy.sparse as sp

import mg_inputs


def centres(shape, h):
    nz, ny, nx = shape
    return np.meshgrid((np.arange(nz) + 0.5) * h, (np.arange(ny) + 0.5) * h, (np.arange(nx) + 0.5) * h,
                       indexing="ij")


def extend(a, odd):
    """The (2nz, 2ny, 2nx) extension of a by reflection across every domain face: a(-1-i) = -a(i)
    (odd, Dirichlet's image) or +a(i) (even, Neumann's image), periodic with period 2N."""
    s = -1.0 if odd else 1.0
    for ax in range(3):
        a = np.concatenate([a, s * np.flip(a, axis=ax)], axis=ax)
    return np.ascontiguousarray(a)


# ------------------------------------------------------------- eigenpairs
@pytest.mark.parametrize("bc", [1, 2])
def test_bc_operator_eigenpairs(oracle_mod, bc):
    """Cell-centred Dirichlet (ghost -x) has eigenvectors prod sin(pi k_d (i_d + 1/2) / N_d), Neumann
    (ghost +x) prod cos(...), both with lambda = -(4/h^2) sum_d sin^2(pi k_d / (2 N_d)); non-cubic grid,
    distinct wave numbers, so a transposed axis, a wrong boundary sign or a wrapped neighbour fails."""
    shape = (12, 16, 20)
    h = 1.0 / 20
    nz, ny, nx = shape
    kz, ky, kx = 3, 2, 5
    f = np.sin if bc == 1 else np.cos
    K, J, I = np.meshgrid(np.arange(nz), np.arange(ny), np.arange(nx), indexing="ij")
    s = f(np.pi * kx * (I + 0.5) / nx) * f(np.pi * ky * (J + 0.5) / ny) * f(np.pi * kz * (K + 0.5) / nz)
    lam = -(4.0 / h**2) * sum(np.sin(np.pi * k / (2 * n)) ** 2 for k, n in ((kx, nx), (ky, ny), (kz, nz)))
    As = oracle_mod.apply_op(s, h, bc=bc)
    assert np.abs(As - lam * s).max() <= 1e-12 * abs(lam)
    # the variable-coefficient operator with c = 1 has the same eigenpairs
    As2 = oracle_mod.apply_op_vc(s, np.ones(shape), h, bc=bc)
    assert np.abs(As2 - lam * s).max() <= 1e-12 * abs(lam)


# --------------------------------------------------------- method of images
@pytest.mark.parametrize("bc,kw", [
    (1, {}),                             # Dirichlet, the paper's smoother
    (2, {}),                             # Neumann
    (1, {"smoother": 1}),                # Dirichlet, Chebyshev steps (pointwise: commute with reflection)
    (1, {"coef": True}),                 # Dirichlet, variable coefficients
    (2, {"coef": True}),
])
def test_bc_vcycle_equals_periodic_vcycle_on_the_reflected_domain(oracle_mod, bc, kw):
    """Method of images: every step of the V-cycle (stencil with boundary images, restriction of
    brick-aligned pairs, piecewise-constant interpolation, pointwise smoothing) commutes with the
    reflection across a domain face, and IEEE arithmetic is symmetric under negation, so the
    Dirichlet (Neumann) V-cycle on N^3 equals BIT FOR BIT the paper's periodic V-cycle on the odd
    (even) extension to (2N)^3 (same h0), restricted to the first octant -- x after each of 2
    cycles and the max-norm residual.  With variable coefficients c is extended evenly."""
    shape = (16, 8, 24)
    L = 3
    h0 = mg_inputs.default_h0(shape)
    b = mg_inputs.random_field(shape, 3)
    coef = mg_inputs.random_coef(shape, 3) if kw.get("coef") else None
    extra = {k: v for k, v in kw.items() if k != "coef"}
    m = oracle_mod.OracleMG(shape, L, 5, 4, 30, h0, bc=bc, coef=coef, **extra)
    m.set_b(b)
    m.set_x(None)
    odd = bc == 1
    ecoef = None if coef is None else extend(coef, False)
    e = oracle_mod.OracleMG(tuple(2 * s for s in shape), L, 5, 4, 30, h0, coef=ecoef, **extra)
    e.set_b(extend(b, odd))
    e.set_x(None)
    nz, ny, nx = shape
    for _ in range(2):
        m.vcycle()
        e.vcycle()
        assert np.array_equal(m.get_x(), e.get_x()[:nz, :ny, :nx])
        assert m.norm() == e.norm()
    assert np.array_equal(extend(m.get_x(), odd), e.get_x())


# ------------------------------------------------- sparse assembly from fluxes
def axis_difference(n, bc, boundary_weight=None):
    """Face-difference matrix G (faces x cells) of one axis and the boundary-face weights.
    Face f sits between cells f-1 and f.  Periodic: n faces, face 0 between n-1 and 0.  Dirichlet:
    n+1 faces, the boundary faces 0 and n carry g = x_0 and g = -x_{n-1} (x_ghost - x_p = -2 x_p: a
    weight of 2 makes w g^2 = 2 c x_p^2); Neumann: the boundary faces carry no flux (weight 0)."""
    if bc == 0:
        G = sp.lil_matrix((n, n))
        for f in range(n):
            G[f, f] += 1.0
            G[f, (f - 1) % n] -= 1.0
        return G.tocsr(), np.ones(n)
    G = sp.lil_matrix((n + 1, n))
    for f in range(1, n):
        G[f, f] = 1.0
        G[f, f - 1] = -1.0
    G[0, 0] = 1.0
    G[n, n - 1] = -1.0
    wb = boundary_weight if boundary_weight is not None else (2.0 if bc == 1 else 0.0)
    w = np.ones(n + 1)
    w[0] = w[n] = wb
    return G.tocsr(), w


def face_coefficients(c_axis_major, bc):
    """(c_left + c_right)/2 on the faces of the last axis (c at a boundary face: the cell's own)."""
    c = c_axis_major
    if bc == 0:
        return 0.5 * (np.roll(c, 1, axis=-1) + c)
    n = c.shape[-1]
    out = np.empty(c.shape[:-1] + (n + 1,))
    out[..., 1:n] = 0.5 * (c[..., :-1] + c[..., 1:])
    out[..., 0] = c[..., 0]
    out[..., n] = c[..., -1]
    return out


def flux_matrix(shape, h, bc, c=None, boundary_weight=None):
    """A = -(1/h^2) sum_d G_d^T W_d G_d assembled from face fluxes (numpy order (z, y, x) ->
    lexicographic i + nx (j + ny k)): an independent formulation of the oracle's stencil.
    boundary_weight = 1 gives the matrix whose diagonal is -(1/h^2) x (sum of the six face
    coefficients), the diagonal reading A23's Jacobi step uses (a domain face counts c_p once, as in
    the reflected periodic problem, so c = 1 keeps the paper's h^2/12 on every cell)."""
    nz, ny, nx = shape
    c = np.ones(shape) if c is None else c
    A = None
    for axis, n in ((2, nx), (1, ny), (0, nz)):
        G1, wb = axis_difference(n, bc, boundary_weight)
        eye = [sp.identity(nz), sp.identity(ny), sp.identity(nx)]
        mats = list(eye)
        mats[axis] = G1
        G = sp.kron(mats[0], sp.kron(mats[1], mats[2])).tocsr()
        cm = np.moveaxis(c, axis, -1)
        fc = face_coefficients(cm, bc) * wb  # boundary weights folded in
        fc = np.moveaxis(fc, -1, axis)
        term = G.T @ sp.diags(fc.ravel()) @ G
        A = term if A is None else A + term
    return (-A / (h * h)).tocsr()


@pytest.mark.parametrize("bc", [0, 1, 2])
@pytest.mark.parametrize("variable", [False, True])
def test_operator_matches_flux_assembly(oracle_mod, bc, variable):
    """The stencil (paper operator under bc, or the variable-coefficient one) equals the matrix
    assembled from face fluxes, on a non-cubic grid with a rough random coefficient."""
    shape = (8, 12, 16)
    h = 1.0 / 16
    x = mg_inputs.random_field(shape, 5)
    c = mg_inputs.random_coef(shape, 5) if variable else None
    A = flux_matrix(shape, h, bc, c)
    want = (A @ x.ravel()).reshape(shape)
    got = oracle_mod.apply_op_vc(x, c, h, bc=bc) if variable else oracle_mod.apply_op(x, h, bc=bc)
    assert np.abs(got - want).max() <= 1e-12 * np.abs(want).max()
    if variable:  # the Jacobi step is (1/2) / (face-sum diagonal)
        gam = oracle_mod.vc_gamma(c, h, bc=bc)
        D = np.abs(flux_matrix(shape, h, bc, c, boundary_weight=1.0).diagonal()).reshape(shape)
        assert np.abs(gam - 0.5 / D).max() <= 1e-14 * gam.max()


def matrix_vcycle(b0, x0, L, h0, pre, post, bottom, bc, c0=None):
    """Alg 2 with matrices: A_l from face fluxes at h_l = 2^l h0 (coarse c_{l+1} = P^T c_l / 8), Jacobi
    steps 0.5 / (face-sum diagonal) (= h_l^2/12 for the paper's operator), P piecewise constant,
    R = P^T/8."""
    from tests.test_oracle_pins import prolong_1d
    shapes = [tuple(s >> l for s in b0.shape) for l in range(L)]
    hs = [h0 * 2**l for l in range(L)]
    P = [sp.kron(prolong_1d(shapes[l][0]), sp.kron(prolong_1d(shapes[l][1]), prolong_1d(shapes[l][2]))).tocsr()
         for l in range(L - 1)]
    cs = [None] * L
    if c0 is not None:
        cs[0] = c0.ravel().copy()
        for l in range(L - 1):
            cs[l + 1] = (P[l].T @ cs[l]) / 8.0
    A = [flux_matrix(shapes[l], hs[l], bc, None if cs[l] is None else cs[l].reshape(shapes[l])) for l in range(L)]
    g = [0.5 / np.abs(flux_matrix(shapes[l], hs[l], bc, cs[l].reshape(shapes[l]), 1.0).diagonal())
         if c0 is not None else np.full(A[l].shape[0], hs[l] ** 2 / 12.0) for l in range(L)]
    x, b = [None] * L, [None] * L
    x[0], b[0] = x0.ravel().copy(), b0.ravel().copy()

    def smooth(l, n):
        r = None
        for _ in range(n):
            Ax = A[l] @ x[l]
            r = b[l] - Ax
            x[l] = x[l] + g[l] * (Ax - b[l])
        return r

    for l in range(L - 1):
        r = smooth(l, pre)
        b[l + 1] = (P[l].T @ r) / 8.0
        x[l + 1] = np.zeros_like(b[l + 1])
    smooth(L - 1, bottom)
    for l in range(L - 2, -1, -1):
        x[l] = x[l] + P[l] @ x[l + 1]
        smooth(l, post)
    return x[0].reshape(b0.shape)


@pytest.mark.parametrize("bc,variable,shape,L", [(1, False, (16, 32, 24), 3), (2, False, (16, 16, 32), 2),
                                                 (0, True, (16, 32, 24), 3), (1, True, (16, 16, 16), 3),
                                                 (2, True, (8, 16, 24), 2)])
def test_variant_vcycle_matches_flux_matrix_vcycle(oracle_mod, bc, variable, shape, L):
    """The V-cycle under bc / with variable coefficients equals the flux-assembled matrix V-cycle to
    rounding after 1 and 2 cycles (pre != post): a wrong boundary image, face average, diagonal, or
    coarse coefficient fails."""
    pre, post, bottom = 4, 3, 30
    h0 = mg_inputs.default_h0(shape)
    b = mg_inputs.random_field(shape, 7)
    c = mg_inputs.random_coef(shape, 7) if variable else None
    m = oracle_mod.OracleMG(shape, L, pre, post, bottom, h0, bc=bc, coef=c)
    m.set_b(b)
    m.set_x(None)
    xm = np.zeros(shape)
    for _ in range(2):
        m.vcycle()
        xm = matrix_vcycle(b, xm, L, h0, pre, post, bottom, bc, c)
        assert np.abs(m.get_x() - xm).max() <= 1e-11 * np.abs(xm).max()


# ------------------------------------------------------------- invariants
@pytest.mark.parametrize("bc", [0, 1, 2])
def test_variable_operator_symmetric_and_constants(oracle_mod, bc):
    """div(c grad .) with arithmetic face averages is symmetric for any c (a one-sided face value,
    c_p or c_n alone, is not); it annihilates constants exactly without a Dirichlet face; c = 1 gives
    the paper's operator to rounding and the paper's step h^2/12 exactly."""
    shape = (8, 16, 24)
    h = 1.0 / 24
    c = mg_inputs.random_coef(shape, 1)
    x, y = mg_inputs.random_field(shape, 1), mg_inputs.random_field(shape, 2)
    Ax, Ay = oracle_mod.apply_op_vc(x, c, h, bc), oracle_mod.apply_op_vc(y, c, h, bc)
    lhs, rhs = float(np.sum(Ax * y)), float(np.sum(x * Ay))
    assert abs(lhs - rhs) <= 1e-12 * np.sum(np.abs(Ax * y))
    if bc != 1:
        assert np.all(oracle_mod.apply_op_vc(np.full(shape, 3.25), c, h, bc) == 0.0)
    one = np.ones(shape)
    ref = oracle_mod.apply_op(x, h, bc)
    assert np.abs(oracle_mod.apply_op_vc(x, one, h, bc) - ref).max() <= 1e-13 * np.abs(ref).max()
    assert np.all(oracle_mod.vc_gamma(one, h, bc) == (h * h) / 12.0)
    # c scaled by 4 (a power of two: exact) scales A by 4 and gamma by 1/4 exactly
    assert np.array_equal(oracle_mod.apply_op_vc(x, 4.0 * c, h, bc), 4.0 * oracle_mod.apply_op_vc(x, c, h, bc))
    assert np.array_equal(oracle_mod.vc_gamma(4.0 * c, h, bc), 0.25 * oracle_mod.vc_gamma(c, h, bc))


def test_variable_vcycle_with_unit_coefficient_is_the_paper_cycle(oracle_mod):
    """c = 1 reproduces the paper's V-cycle up to the rounding of the different expression."""
    shape = (16, 16, 32)
    b = mg_inputs.random_rhs(shape, 8)
    m1 = oracle_mod.OracleMG(shape, 3, 6, 6, 50)
    m2 = oracle_mod.OracleMG(shape, 3, 6, 6, 50, coef=np.ones(shape))
    for m in (m1, m2):
        m.set_b(b)
        m.set_x(None)
        m.vcycle()
    x1, x2 = m1.get_x(), m2.get_x()
    assert np.abs(x1 - x2).max() <= 1e-12 * np.abs(x1).max()


# ------------------------------------------------------- second order
def test_dirichlet_second_order_convergence(oracle_mod):
    """Solving A x = f with u = sin(pi x) sin(pi y) sin(pi z) on the unit cube (u = 0 on the faces),
    f = -3 pi^2 u: the max error of the converged discrete solution falls ~4x per refinement."""
    errs = []
    for n in (16, 32, 64):
        shape = (n, n, n)
        h = 1.0 / n
        Z, Y, X = centres(shape, h)
        u = np.sin(np.pi * X) * np.sin(np.pi * Y) * np.sin(np.pi * Z)
        m = oracle_mod.OracleMG(shape, int(np.log2(n)) - 2, bc=1)
        m.set_b(-3.0 * np.pi**2 * u)
        m.set_x(None)
        cycles, norms = m.solve(1e-10, 20)
        assert norms[-1] <= 1e-10
        errs.append(np.abs(m.get_x() - u).max())
    r1, r2 = errs[0] / errs[1], errs[1] / errs[2]
    assert 3.5 < r1 < 4.5 and 3.7 < r2 < 4.3, errs


def test_variable_coefficient_second_order_convergence(oracle_mod):
    """div(c grad u) = f with u = sin(pi x) sin(pi y) sin(pi z), c = 1 + x y z / 2 (Dirichlet):
    f = c lap u + grad c . grad u; the converged discrete solution converges at second order."""
    errs = []
    for n in (16, 32, 64):
        shape = (n, n, n)
        h = 1.0 / n
        Z, Y, X = centres(shape, h)
        sx, sy, sz = np.sin(np.pi * X), np.sin(np.pi * Y), np.sin(np.pi * Z)
        cx, cy, cz = np.cos(np.pi * X), np.cos(np.pi * Y), np.cos(np.pi * Z)
        u = sx * sy * sz
        c = 1.0 + 0.5 * X * Y * Z
        grad_c = (0.5 * Y * Z, 0.5 * X * Z, 0.5 * X * Y)
        grad_u = (np.pi * cx * sy * sz, np.pi * sx * cy * sz, np.pi * sx * sy * cz)
        f = c * (-3.0 * np.pi**2 * u) + sum(a * b for a, b in zip(grad_c, grad_u))
        m = oracle_mod.OracleMG(shape, int(np.log2(n)) - 2, bc=1, coef=c)
        m.set_b(f)
        m.set_x(None)
        cycles, norms = m.solve(1e-10, 30)
        assert norms[-1] <= 1e-10
        errs.append(np.abs(m.get_x() - u).max())
    r1, r2 = errs[0] / errs[1], errs[1] / errs[2]
    assert 3.3 < r1 < 4.7 and 3.6 < r2 < 4.4, errs


@pytest.mark.parametrize("bc", [1, 2])
def test_bc_vcycle_convergence_level_independent(oracle_mod, bc):
    """With a non-periodic boundary the V-cycle still contracts the max-norm residual by a factor
    that does not grow with the number of levels (random zero-mean b, 12/12/100, coarsest 8^3).
    Dirichlet: rho < 0.06 like the periodic cycle.  Neumann: the 100-sweep bottom limits the rate --
    its slowest non-constant mode on 8^3 has 4 sin^2(pi/16) = 0.15 of h^-2 (periodic: 4 sin^2(pi/8) =
    0.59), so it contracts only to (1 - 0.15/12)^100 = 0.28 per cycle; measured 0.12-0.23."""
    rhos = []
    for L in (2, 3, 4):
        n = 8 << (L - 1)
        shape = (n, n, n)
        b = mg_inputs.random_rhs(shape, 0)
        m = oracle_mod.OracleMG(shape, L, bc=bc)
        m.set_b(b)
        m.set_x(None)
        norms = [m.norm()]
        for _ in range(5):
            m.vcycle()
            norms.append(m.norm())
        rhos.append((norms[5] / norms[1]) ** 0.25)
    if bc == 1:
        assert max(rhos) < 0.06 and max(rhos) / min(rhos) < 1.8, rhos
    else:
        assert max(rhos) < 0.3 and rhos[-1] <= rhos[0], rhos


def test_cg_bottom_needs_the_periodic_operator(oracle_mod):
    """The CG bottom (reading A21) removes the periodic null space; with a boundary or variable
    coefficients the oracle refuses it instead of solving the wrong system."""
    with pytest.raises(ValueError):
        oracle_mod.OracleMG((16, 16, 16), 2, bc=1, bottom_solver=1)
    with pytest.raises(ValueError):
        oracle_mod.OracleMG((16, 16, 16), 2, coef=np.ones((16, 16, 16)), bottom_solver=1)
