/*
 * mg_oracle.c -- CPU ORACLE for the brick-GMG V-cycle.  TEST INFRASTRUCTURE ONLY.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
 * reference legs may load this file's library.  The product path
 * (paper_conf_sc_antepara0jh24_b200/) never links, imports or calls it and
 * shares no code, header, table or helper with it.
 *
 * What it is: a plain, slow, obviously-correct multigrid on a GLOBAL
 * lexicographic periodic cell-centred grid (never decomposed, never
 * bricked), index p = i + nx*(j + ny*k), i fastest.  Every function follows
 * one passage of PAPER.md (Antepara et al., SC'24), cited as P:Lnn:
 *
 *   applyOp               P:L117, L133, L148 (7-point stencil, alpha=-6/h^2,
 *                         beta=1/h^2, h = spacing of the level), Fig 1 DSL P:L44-55
 *   smooth                P:L118, L148   x := x + gamma*(Ax - b), gamma = h^2/12
 *   smooth+residual       P:L119, L133, L148  r = b - Ax computed from the same Ax
 *   restriction           P:L69, L120    average of the 8 fine cells of a coarse cell
 *   initZero              P:L146 (Alg 2 step 8)
 *   interpolation+incr.   P:L69, L123, L135  x^h = x^h + I(x^2h), piecewise constant
 *   V-cycle               P:L144-146 (Alg 2), readings A1-A3 of DESIGN.md
 *   maxNormRes            P:L139-141 (Alg 1), P:L148 (max residual, 1e-10)
 *   GSRB smoother         variant (N4, reading A20): red then black Gauss-Seidel half-sweeps,
 *                         oracle_gsrb_half; pinned against a sparse triangular solve
 *   Chebyshev smoother    variant (N4, reading A19): per-sweep steps gamma_k, see
 *                         oracle_chebyshev_gamma; pinned by the Chebyshev-polynomial
 *                         error factor on eigenmodes (tests/test_oracle_pins.py)
 *   boundary conditions   variant (N4 "non-periodic BCs", reading A22): homogeneous Dirichlet
 *                         (bc = 1) or Neumann (bc = 2) on the domain faces of the cell-centred
 *                         grid: the neighbour across a domain face is -x_p (Dirichlet: the linear
 *                         extrapolation through 0 on the face) or +x_p (Neumann), on every level
 *                         (rediscretised); oracle_apply_op_bc
 *   variable coefficients variant (N4, reading A23): A x = div(c grad x) with a cell coefficient
 *                         c > 0 and face values (c_p + c_n)/2, damped Jacobi with the local
 *                         diagonal, coarse c = restriction of c; oracle_apply_op_vc,
 *                         oracle_vc_gamma
 *   CG bottom solver      variant (N4 "other bottom solvers", reading A21): `bottom`
 *                         iterations of conjugate gradients on A x = b from x = 0 with a
 *                         fixed-order (stride-doubling pairwise tree, lexicographic) dot
 *                         product, oracle_cg / oracle_dot_tree; pinned by Krylov optimality
 *                         against a dense projection and by finite termination
 *
 * Readings of garbled / silent passages:
 *   - expression order (A8): neighbour sum pairwise by axis
 *       ((xW+xE)+(xS+xN))+(xB+xT); restriction pairwise i -> j -> k;
 *     every + - * separately rounded binary64, NO FMA (-ffp-contract=off).
 *   - residual restricted is the one smooth+residual writes, i.e. b - A x
 *     with x the iterate BEFORE that sweep (A5, lagged; Table IV
 *     0.15 FLOP/B = 6 flop / 40 B).
 *   - exactly `pre`, `post`, `bottom` sweeps (A1, A3); levels 0..L-1,
 *     bottom at L-1 (A2).
 *   - the exchange() of Alg 2 is the periodic wrap of the global grid.
 *
 * Threads: OpenMP over k-planes; every output point is computed by one fixed
 * expression, and max is exact, so results do not depend on the thread count.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#define IDX(i, j, k, nx, ny) ((size_t)(i) + (size_t)(nx) * ((size_t)(j) + (size_t)(ny) * (size_t)(k)))

void oracle_set_threads(int n) {
#ifdef _OPENMP
  if (n > 0) omp_set_num_threads(n);
#else
  (void)n;
#endif
}

int oracle_get_threads(void) {
#ifdef _OPENMP
  return omp_get_max_threads();
#else
  return 1;
#endif
}

/* Neighbour of cell i on an axis of n cells (reading A22): the periodic wrap (bc 0, the paper,
 * P:L148), or -1 when the neighbour lies outside a non-periodic domain (the caller then uses the
 * boundary value: -x_p for homogeneous Dirichlet, +x_p for homogeneous Neumann). */
static int nbr(int i, int d, int n, int bc) {
  const int j = i + d;
  if (j >= 0 && j < n) return j;
  if (bc == 0) return (j + n) % n;
  return -1;
}

/* value of x at neighbour (a, b, c) of cell p: inside, or the boundary image of x_p (reading A22) */
static double nbv(const double *x, int a, int b, int c, int nx, int ny, int bc, double xp) {
  if (a < 0 || b < 0 || c < 0) return bc == 1 ? -xp : xp;
  return x[IDX(a, b, c, nx, ny)];
}

/* applyOp (Fig 1): Ax = alpha*x + beta*(6 neighbours),
 * alpha = -6/h^2, beta = 1/h^2; periodic wrap stands for exchange() (bc = 0, the paper), or the
 * homogeneous Dirichlet / Neumann boundary image of reading A22 (bc = 1 / 2). */
void oracle_apply_op_bc(int nx, int ny, int nz, double h, int bc, const double *x, double *Ax) {
  const double inv = 1.0 / (h * h);
  const double alpha = -6.0 * inv;
  const double beta = inv;
#pragma omp parallel for schedule(static)
  for (int k = 0; k < nz; ++k) {
    const int kb = nbr(k, -1, nz, bc), kt = nbr(k, 1, nz, bc);
    for (int j = 0; j < ny; ++j) {
      const int js = nbr(j, -1, ny, bc), jn = nbr(j, 1, ny, bc);
      for (int i = 0; i < nx; ++i) {
        const int iw = nbr(i, -1, nx, bc), ie = nbr(i, 1, nx, bc);
        const double xp = x[IDX(i, j, k, nx, ny)];
        const double xw = nbv(x, iw, j, k, nx, ny, bc, xp), xe = nbv(x, ie, j, k, nx, ny, bc, xp);
        const double xs = nbv(x, i, js, k, nx, ny, bc, xp), xn = nbv(x, i, jn, k, nx, ny, bc, xp);
        const double xb = nbv(x, i, j, kb, nx, ny, bc, xp), xt = nbv(x, i, j, kt, nx, ny, bc, xp);
        const double sum = ((xw + xe) + (xs + xn)) + (xb + xt);
        Ax[IDX(i, j, k, nx, ny)] = alpha * xp + beta * sum;
      }
    }
  }
}

/* the paper's operator (periodic) */
void oracle_apply_op(int nx, int ny, int nz, double h, const double *x, double *Ax) {
  oracle_apply_op_bc(nx, ny, nz, h, 0, x, Ax);
}

/* Variable-coefficient operator (variant N4, reading A23; the paper's BrickLib "nonconstant
 * coefficients"): (A x)_p = inv * sum_n beta_n (x_n - x_p), beta_n = (c_p + c_n) * 0.5 the
 * face coefficient between p and neighbour n (arithmetic mean of the cell coefficients), inv = 1/h^2,
 * terms t_n = beta_n * (x_n - x_p) summed ((tW+tE)+(tS+tN))+(tB+tT).  Across a non-periodic
 * domain face (reading A22) the neighbour's x is the boundary image of x_p and its c is c_p (the
 * face coefficient is then c_p).  With c = 1 this is the paper's operator up to rounding. */
void oracle_apply_op_vc(int nx, int ny, int nz, double h, int bc, const double *c, const double *x, double *Ax) {
  const double inv = 1.0 / (h * h);
#pragma omp parallel for schedule(static)
  for (int k = 0; k < nz; ++k) {
    const int kb = nbr(k, -1, nz, bc), kt = nbr(k, 1, nz, bc);
    for (int j = 0; j < ny; ++j) {
      const int js = nbr(j, -1, ny, bc), jn = nbr(j, 1, ny, bc);
      for (int i = 0; i < nx; ++i) {
        const int iw = nbr(i, -1, nx, bc), ie = nbr(i, 1, nx, bc);
        const size_t p = IDX(i, j, k, nx, ny);
        const double xp = x[p], cp = c[p];
        const int na[6][3] = {{iw, j, k}, {ie, j, k}, {i, js, k}, {i, jn, k}, {i, j, kb}, {i, j, kt}};
        double t[6];
        for (int q = 0; q < 6; ++q) {
          const int a = na[q][0], b = na[q][1], cc = na[q][2];
          const double xn = nbv(x, a, b, cc, nx, ny, bc, xp);
          const double cn = (a < 0 || b < 0 || cc < 0) ? cp : c[IDX(a, b, cc, nx, ny)];
          t[q] = ((cp + cn) * 0.5) * (xn - xp);
        }
        Ax[p] = inv * (((t[0] + t[1]) + (t[2] + t[3])) + (t[4] + t[5]));
      }
    }
  }
}

/* Damped-Jacobi step of the variable-coefficient operator (reading A23): gamma_p = omega / |diag_p|
 * with omega = 1/2 and diag_p = -inv * S_p, S_p = ((bW+bE)+(bS+bN))+(bB+bT) the sum of the six face
 * coefficients, i.e. gamma_p = (0.5*h*h) / S_p (c = 1: S_p = 6, gamma = h^2/12, the paper's step,
 * P:L148). */
void oracle_vc_gamma(int nx, int ny, int nz, double h, int bc, const double *c, double *gam) {
  const double g = 0.5 * (h * h);
#pragma omp parallel for schedule(static)
  for (int k = 0; k < nz; ++k) {
    const int kb = nbr(k, -1, nz, bc), kt = nbr(k, 1, nz, bc);
    for (int j = 0; j < ny; ++j) {
      const int js = nbr(j, -1, ny, bc), jn = nbr(j, 1, ny, bc);
      for (int i = 0; i < nx; ++i) {
        const int iw = nbr(i, -1, nx, bc), ie = nbr(i, 1, nx, bc);
        const size_t p = IDX(i, j, k, nx, ny);
        const double cp = c[p];
        const int na[6][3] = {{iw, j, k}, {ie, j, k}, {i, js, k}, {i, jn, k}, {i, j, kb}, {i, j, kt}};
        double f[6];
        for (int q = 0; q < 6; ++q) {
          const int a = na[q][0], b = na[q][1], cc = na[q][2];
          const double cn = (a < 0 || b < 0 || cc < 0) ? cp : c[IDX(a, b, cc, nx, ny)];
          f[q] = (cp + cn) * 0.5;
        }
        gam[p] = g / (((f[0] + f[1]) + (f[2] + f[3])) + (f[4] + f[5]));
      }
    }
  }
}

/* smooth(+residual) with a step per cell (variable coefficients, reading A23):
 * r = b - Ax (if r != NULL), x := x + gamma_p (Ax - b). */
void oracle_smooth_residual_field(size_t n, const double *gam, double *x, const double *Ax, const double *b,
                                  double *r) {
#pragma omp parallel for schedule(static)
  for (size_t p = 0; p < n; ++p) {
    if (r) r[p] = b[p] - Ax[p];
    x[p] = x[p] + gam[p] * (Ax[p] - b[p]);
  }
}

/* smooth with an explicit step: x := x + gamma*(Ax - b) (P:L118, L148 with gamma given). */
void oracle_smooth_gamma(size_t n, double gamma, double *x, const double *Ax, const double *b) {
#pragma omp parallel for schedule(static)
  for (size_t p = 0; p < n; ++p) x[p] = x[p] + gamma * (Ax[p] - b[p]);
}

/* smooth+residual with an explicit step; r = b - Ax from the SAME Ax. */
void oracle_smooth_residual_gamma(size_t n, double gamma, double *x, const double *Ax, const double *b, double *r) {
#pragma omp parallel for schedule(static)
  for (size_t p = 0; p < n; ++p) {
    r[p] = b[p] - Ax[p];
    x[p] = x[p] + gamma * (Ax[p] - b[p]);
  }
}

/* smooth: point Jacobi x := x + gamma*(Ax - b), gamma = h^2/12. */
void oracle_smooth(size_t n, double h, double *x, const double *Ax, const double *b) {
  oracle_smooth_gamma(n, (h * h) / 12.0, x, Ax, b);
}

/* smooth+residual: the smooth above and r = b - Ax from the
 * SAME Ax ("simultaneously calculates the residual"). */
void oracle_smooth_residual(size_t n, double h, double *x, const double *Ax, const double *b, double *r) {
  oracle_smooth_residual_gamma(n, (h * h) / 12.0, x, Ax, b, r);
}

/* Red-black Gauss-Seidel half-sweep (GSRB smoother variant, reading A20): from
 * the same Ax of the whole grid, cells of colour c = (i+j+k) mod 2 (global indices) take the
 * Gauss-Seidel update x := x + (h^2/6)(Ax - b) (1/|diag| of P:L148's operator); the other colour
 * keeps x.  If r != NULL, r = b - Ax on every cell (the residual of the x the half-sweep read). */
void oracle_gsrb_half(int nx, int ny, int nz, double h, int colour, double *x, const double *Ax, const double *b,
                      double *r) {
  const double g = (h * h) / 6.0;
#pragma omp parallel for schedule(static)
  for (int k = 0; k < nz; ++k)
    for (int j = 0; j < ny; ++j)
      for (int i = 0; i < nx; ++i) {
        const size_t p = IDX(i, j, k, nx, ny);
        if (r) r[p] = b[p] - Ax[p];
        if (((i + j + k) & 1) == colour) x[p] = x[p] + g * (Ax[p] - b[p]);
      }
}

/* Chebyshev smoother variant (the paper names other smoothers as
 * future work; not in its method).  Reading A19: s sweeps of
 * non-stationary Richardson x := x + gamma_k (Ax - b) whose steps are the reciprocals of
 * the Chebyshev nodes of the smoothing interval mu in [mu_max/rho, mu_max], mu = -lambda,
 * mu_max = 12/h^2 (the damped-Jacobi bound):
 *   nu_j = theta + delta*cos(pi*(2j+1)/(2s)), theta = (1+1/rho)/2, delta = (1-1/rho)/2,
 *   gamma_k = h^2 / (12*nu_j(k)),  j(k) = k/2 for even k, s-1-(k-1)/2 for odd k
 * (small and large steps interleaved).  After the s sweeps the error of every mode is
 * multiplied by T_s((theta - mu/mu_max)/delta) / T_s(theta/delta). */
double oracle_chebyshev_gamma(double h, int s, int k, int rho) {
  const int j = (k % 2 == 0) ? k / 2 : s - 1 - (k - 1) / 2;
  const double th = 0.5 * (1.0 + 1.0 / (double)rho), de = 0.5 * (1.0 - 1.0 / (double)rho);
  const double nu = th + de * cos(3.14159265358979323846 * (double)(2 * j + 1) / (double)(2 * s));
  return (h * h) / (12.0 * nu);
}

/* restriction: b^{2h} = average of the 8 fine cells of each coarse
 * cell (finite-volume volume average).  nx,ny,nz are FINE dims (even). */
void oracle_restriction(int nx, int ny, int nz, const double *r, double *bc) {
  const int cx = nx / 2, cy = ny / 2, cz = nz / 2;
#pragma omp parallel for schedule(static)
  for (int K = 0; K < cz; ++K)
    for (int J = 0; J < cy; ++J)
      for (int I = 0; I < cx; ++I) {
        const int i = 2 * I, j = 2 * J, k = 2 * K;
        const double r000 = r[IDX(i, j, k, nx, ny)], r100 = r[IDX(i + 1, j, k, nx, ny)];
        const double r010 = r[IDX(i, j + 1, k, nx, ny)], r110 = r[IDX(i + 1, j + 1, k, nx, ny)];
        const double r001 = r[IDX(i, j, k + 1, nx, ny)], r101 = r[IDX(i + 1, j, k + 1, nx, ny)];
        const double r011 = r[IDX(i, j + 1, k + 1, nx, ny)], r111 = r[IDX(i + 1, j + 1, k + 1, nx, ny)];
        bc[IDX(I, J, K, cx, cy)] = 0.125 * (((r000 + r100) + (r010 + r110)) + ((r001 + r101) + (r011 + r111)));
      }
}

/* initZero (Alg 2 step 8): coarse initial guess x^{2h} = 0. */
void oracle_init_zero(size_t n, double *x) {
#pragma omp parallel for schedule(static)
  for (size_t p = 0; p < n; ++p) x[p] = 0.0;
}

/* interpolation+increment: x^h = x^h + I(x^{2h}), each coarse
 * value increments its 8 fine cells.  nx,ny,nz are FINE dims. */
void oracle_interpolation_increment(int nx, int ny, int nz, const double *xc, double *x) {
  const int cx = nx / 2, cy = ny / 2;
#pragma omp parallel for schedule(static)
  for (int k = 0; k < nz; ++k)
    for (int j = 0; j < ny; ++j)
      for (int i = 0; i < nx; ++i)
        x[IDX(i, j, k, nx, ny)] = x[IDX(i, j, k, nx, ny)] + xc[IDX(i / 2, j / 2, k / 2, cx, cy)];
}

/* maxNormRes (Alg 1): max over the domain of |b - Ax|, with a
 * fresh applyOp on the current x (reading A6).  A NaN anywhere makes the max NaN (a diverged
 * iterate must not pass the 1e-10 test): each thread keeps a NaN once it saw one, and so does the
 * combination of the threads' maxima.  _ex: under the boundary condition bc (reading A22) and,
 * with c != NULL, the variable-coefficient operator (reading A23). */
double oracle_max_norm_residual_ex(int nx, int ny, int nz, double h, int bc, const double *c, const double *x,
                                   const double *b) {
  const size_t n = (size_t)nx * ny * nz;
  double *Ax = (double *)malloc(n * sizeof(double));
  if (!Ax) return NAN;
  if (c)
    oracle_apply_op_vc(nx, ny, nz, h, bc, c, x, Ax);
  else
    oracle_apply_op_bc(nx, ny, nz, h, bc, x, Ax);
  double m = 0.0;
#pragma omp parallel
  {
    double mt = 0.0;
#pragma omp for schedule(static)
    for (size_t p = 0; p < n; ++p) {
      const double a = fabs(b[p] - Ax[p]);
      if (a > mt || a != a) mt = a;
    }
#pragma omp critical
    {
      if (mt > m || mt != mt) m = mt;
    }
  }
  free(Ax);
  return m;
}

/* the paper's norm (periodic, constant coefficients) */
double oracle_max_norm_residual(int nx, int ny, int nz, double h, const double *x, const double *b) {
  return oracle_max_norm_residual_ex(nx, ny, nz, h, 0, NULL, x, b);
}

/* Fixed-order dot product (reading A21): v_i = a_i * b_i over the lexicographic index, then for
 * s = 1, 2, 4, ...: v_i = v_i + v_{i+s} for every i that is a multiple of 2s with i + s < n; the
 * result is v_0 (a pairwise tree; every operation separately rounded).  Sequential (test oracle). */
double oracle_dot_tree(size_t n, const double *a, const double *b) {
  if (n == 0) return 0.0;
  double *v = (double *)malloc(n * sizeof(double));
  if (!v) return NAN;
  for (size_t i = 0; i < n; ++i) v[i] = a[i] * b[i];
  for (size_t s = 1; s < n; s *= 2)
    for (size_t i = 0; i + s < n; i += 2 * s) v[i] = v[i] + v[i + s];
  const double d = v[0];
  free(v);
  return d;
}

/* CG bottom solver (variant, reading A21; SURVEY §8(f) N4 "other bottom solvers"; the paper's
 * bottom is `bottom` smooths): at most `iters` iterations of unpreconditioned
 * conjugate gradients on A x = b - m from x = 0.  A = the level's applyOp is symmetric negative
 * semi-definite on the periodic grid with the constants as null space (reading A12), so CG runs on
 * the consistent system: m = <b, 1> / N removes b's mean (rounding leaves a tiny one after the
 * restrictions; left in, CG divides by p.Ap ~ 0 once the rest has converged and blows x up):
 *   r = b - m;  p = r;  rr0 = rr = <r, r>
 *   repeat:  q = A p;  d = <p, q>;  if not d < 0: stop            (breakdown / converged)
 *            alpha = rr / d;  x = x + alpha p;  r = r - alpha q;  rr' = <r, r>
 *            if rr' <= 1e-24 rr0: stop                               (relative residual 1e-12)
 *            beta = rr' / rr;  p = r + beta p;  rr = rr'
 * <.,.> = oracle_dot_tree (<b, 1> sums b itself); every operation separately rounded (CG's
 * formulas hold for a definite operator of either sign: alpha < 0 here). */
void oracle_cg(int nx, int ny, int nz, double h, int iters, double *x, const double *b) {
  const size_t n = (size_t)nx * ny * nz;
  double *r = (double *)malloc(n * sizeof(double)), *p = (double *)malloc(n * sizeof(double));
  double *q = (double *)malloc(n * sizeof(double));
  if (!r || !p || !q) {
    free(r), free(p), free(q);
    return;
  }
  for (size_t i = 0; i < n; ++i) q[i] = 1.0;
  const double m = oracle_dot_tree(n, b, q) / (double)n;
  for (size_t i = 0; i < n; ++i) {
    x[i] = 0.0;
    r[i] = b[i] - m;
    p[i] = r[i];
  }
  double rr = oracle_dot_tree(n, r, r);
  const double rr0 = rr;
  for (int it = 0; it < iters; ++it) {
    oracle_apply_op(nx, ny, nz, h, p, q);
    const double d = oracle_dot_tree(n, p, q);
    if (!(d < 0.0)) break;
    const double alpha = rr / d;
    for (size_t i = 0; i < n; ++i) {
      x[i] = x[i] + alpha * p[i];
      r[i] = r[i] - alpha * q[i];
    }
    const double rr2 = oracle_dot_tree(n, r, r);
    if (rr2 <= 1e-24 * rr0) break;
    const double beta = rr2 / rr;
    for (size_t i = 0; i < n; ++i) p[i] = r[i] + beta * p[i];
    rr = rr2;
  }
  free(r), free(p), free(q);
}

/* ---------------------------------------------------------------------------
 * V-cycle hierarchy (Alg 2)
 * ------------------------------------------------------------------------- */
#define ORACLE_MAX_LEVELS 16
typedef struct {
  int L, pre, post, bottom;
  int smoother, rho; /* 0 = damped Jacobi (the paper); 1 = Chebyshev (oracle_chebyshev_gamma) on pre/post;
                        2 = red-black Gauss-Seidel on pre/post (oracle_gsrb_half: red then black) */
  int bottom_solver;  /* 0 = `bottom` damped Jacobi smooths (the paper); 1 = `bottom` CG iterations (oracle_cg) */
  int bc;             /* 0 = periodic (the paper); 1 = homogeneous Dirichlet; 2 = homogeneous Neumann (A22) */
  double *c[ORACLE_MAX_LEVELS], *gam[ORACLE_MAX_LEVELS]; /* variable coefficients (A23): NULL = constant */
  int n[ORACLE_MAX_LEVELS][3];
  double h[ORACLE_MAX_LEVELS];
  double *x[ORACLE_MAX_LEVELS], *b[ORACLE_MAX_LEVELS], *Ax[ORACLE_MAX_LEVELS], *r[ORACLE_MAX_LEVELS];
} oracle_mg;

static size_t lvl_n(const oracle_mg *m, int l) { return (size_t)m->n[l][0] * m->n[l][1] * m->n[l][2]; }

void oracle_mg_destroy(oracle_mg *m) {
  if (!m) return;
  for (int l = 0; l < m->L; ++l) {
    free(m->x[l]);
    free(m->b[l]);
    free(m->Ax[l]);
    free(m->r[l]);
    free(m->c[l]);
    free(m->gam[l]);
  }
  free(m);
}

/* Level l has spacing h_l = h0 * 2^l ("on each coarser level the grid
 * size is multiplied by two"; h is the spacing of the given level). */
oracle_mg *oracle_mg_create(int nx, int ny, int nz, int L, double h0, int pre, int post, int bottom) {
  if (L < 1 || L > ORACLE_MAX_LEVELS) return NULL;
  oracle_mg *m = (oracle_mg *)calloc(1, sizeof(oracle_mg));
  if (!m) return NULL;
  m->L = L;
  m->pre = pre;
  m->post = post;
  m->bottom = bottom;
  for (int l = 0; l < L; ++l) {
    const int s = 1 << l;
    if (nx % s || ny % s || nz % s) {
      oracle_mg_destroy(m);
      return NULL;
    }
    m->n[l][0] = nx / s;
    m->n[l][1] = ny / s;
    m->n[l][2] = nz / s;
    m->h[l] = h0 * (double)s;
    const size_t n = lvl_n(m, l);
    m->x[l] = (double *)calloc(n, sizeof(double));
    m->b[l] = (double *)calloc(n, sizeof(double));
    m->Ax[l] = (double *)calloc(n, sizeof(double));
    m->r[l] = (double *)calloc(n, sizeof(double));
    if (!m->x[l] || !m->b[l] || !m->Ax[l] || !m->r[l]) {
      oracle_mg_destroy(m);
      return NULL;
    }
  }
  return m;
}

void oracle_mg_set_smoother(oracle_mg *m, int smoother, int rho) {
  m->smoother = smoother;
  m->rho = rho;
}
/* CG bottom (A21) only for the periodic constant-coefficient operator: -1 otherwise */
int oracle_mg_set_bottom_solver(oracle_mg *m, int solver) {
  if (solver == 1 && (m->bc != 0 || m->c[0])) return -1;
  m->bottom_solver = solver;
  return 0;
}

/* boundary condition of every level (reading A22) */
int oracle_mg_set_bc(oracle_mg *m, int bc) {
  if (bc < 0 || bc > 2 || (bc != 0 && m->bottom_solver == 1)) return -1;
  m->bc = bc;
  for (int l = 0; l < m->L && m->c[l]; ++l)
    oracle_vc_gamma(m->n[l][0], m->n[l][1], m->n[l][2], m->h[l], m->bc, m->c[l], m->gam[l]);
  return 0;
}

/* Variable coefficients (reading A23): c of level 0 (lexicographic, c > 0); coarse levels take the
 * restriction (volume average) of the level above; the Jacobi steps gamma_p of every
 * level follow (oracle_vc_gamma).  c0 == NULL restores the paper's constant operator. */
int oracle_mg_set_coef(oracle_mg *m, const double *c0) {
  for (int l = 0; l < m->L; ++l) {
    free(m->c[l]);
    free(m->gam[l]);
    m->c[l] = m->gam[l] = NULL;
  }
  if (!c0) return 0;
  if (m->bottom_solver == 1) return -1;
  for (int l = 0; l < m->L; ++l) {
    m->c[l] = (double *)malloc(lvl_n(m, l) * sizeof(double));
    m->gam[l] = (double *)malloc(lvl_n(m, l) * sizeof(double));
    if (!m->c[l] || !m->gam[l]) return -1;
    if (l == 0)
      memcpy(m->c[0], c0, lvl_n(m, 0) * sizeof(double));
    else
      oracle_restriction(m->n[l - 1][0], m->n[l - 1][1], m->n[l - 1][2], m->c[l - 1], m->c[l]);
    oracle_vc_gamma(m->n[l][0], m->n[l][1], m->n[l][2], m->h[l], m->bc, m->c[l], m->gam[l]);
  }
  return 0;
}

/* the level's operator: the paper's (under bc) or the variable-coefficient one */
static void level_apply(const oracle_mg *m, int l, const double *x, double *Ax) {
  const int *n = m->n[l];
  if (m->c[l])
    oracle_apply_op_vc(n[0], n[1], n[2], m->h[l], m->bc, m->c[l], x, Ax);
  else
    oracle_apply_op_bc(n[0], n[1], n[2], m->h[l], m->bc, x, Ax);
}

/* one smooth(+residual) of level l with the step of sweep it of n (pre / post), or the bottom's */
static void level_smooth(oracle_mg *m, int l, int n, int it, int write_r) {
  if (m->c[l]) {
    oracle_smooth_residual_field(lvl_n(m, l), m->gam[l], m->x[l], m->Ax[l], m->b[l], write_r ? m->r[l] : NULL);
    return;
  }
  const double g = n > 0 ? (m->smoother ? oracle_chebyshev_gamma(m->h[l], n, it, m->rho) : (m->h[l] * m->h[l]) / 12.0)
                         : (m->h[l] * m->h[l]) / 12.0;
  if (write_r)
    oracle_smooth_residual_gamma(lvl_n(m, l), g, m->x[l], m->Ax[l], m->b[l], m->r[l]);
  else
    oracle_smooth_gamma(lvl_n(m, l), g, m->x[l], m->Ax[l], m->b[l]);
}

void oracle_mg_set_b(oracle_mg *m, const double *b) { memcpy(m->b[0], b, lvl_n(m, 0) * sizeof(double)); }
void oracle_mg_set_x(oracle_mg *m, const double *x) {
  if (x)
    memcpy(m->x[0], x, lvl_n(m, 0) * sizeof(double));
  else
    memset(m->x[0], 0, lvl_n(m, 0) * sizeof(double));
}
void oracle_mg_get_x(const oracle_mg *m, double *x) { memcpy(x, m->x[0], lvl_n(m, 0) * sizeof(double)); }
/* debug/test access to any level's fields: which = 0 x, 1 b, 2 r, 3 Ax */
int oracle_mg_get_level(const oracle_mg *m, int l, int which, double *out) {
  if (l < 0 || l >= m->L) return -1;
  const double *src = which == 0 ? m->x[l] : which == 1 ? m->b[l] : which == 2 ? m->r[l] : m->Ax[l];
  memcpy(out, src, lvl_n(m, l) * sizeof(double));
  return 0;
}

/* `n` pre / post sweeps of level l (Alg 2 steps 2-6, 18-21): exchange() + applyOp, then
 * smooth+residual; the GSRB variant (A20) a red then a black half-sweep per sweep. */
static void level_sweeps(oracle_mg *m, int l, int n) {
  const int *d = m->n[l];
  for (int it = 0; it < n; ++it) {
    if (m->smoother == 2 && !m->c[l]) { /* GSRB: red half, then black half */
      for (int c = 0; c < 2; ++c) {
        level_apply(m, l, m->x[l], m->Ax[l]);
        oracle_gsrb_half(d[0], d[1], d[2], m->h[l], c, m->x[l], m->Ax[l], m->b[l], m->r[l]);
      }
      continue;
    }
    level_apply(m, l, m->x[l], m->Ax[l]); /* exchange()+applyOp */
    level_smooth(m, l, n, it, 1);
  }
}

/* Alg 2, levels 0..L-1 with the bottom solver at L-1 (readings A1-A3). */
void oracle_mg_vcycle(oracle_mg *m) {
  const int L = m->L;
  for (int l = 0; l + 1 < L; ++l) {
    const int *n = m->n[l];
    level_sweeps(m, l, m->pre);                                 /* steps 2-6 */
    oracle_restriction(n[0], n[1], n[2], m->r[l], m->b[l + 1]); /* step 7 */
    oracle_init_zero(lvl_n(m, l + 1), m->x[l + 1]);             /* step 8 */
  }
  {                                                             /* steps 10-15: bottom */
    const int l = L - 1;
    const int *n = m->n[l];
    if (m->bottom_solver == 1) /* reading A21: x = 0 (initZero) and `bottom` CG iterations */
      oracle_cg(n[0], n[1], n[2], m->h[l], m->bottom, m->x[l], m->b[l]);
    else
      for (int it = 0; it < m->bottom; ++it) {
        level_apply(m, l, m->x[l], m->Ax[l]);
        level_smooth(m, l, 0, it, 0); /* smooth (damped Jacobi) */
      }
  }
  for (int l = L - 2; l >= 0; --l) {                            /* steps 16-23 */
    const int *n = m->n[l];
    oracle_interpolation_increment(n[0], n[1], n[2], m->x[l + 1], m->x[l]);
    level_sweeps(m, l, m->post);
  }
}

double oracle_mg_norm(const oracle_mg *m) {
  return oracle_max_norm_residual_ex(m->n[0][0], m->n[0][1], m->n[0][2], m->h[0], m->bc, m->c[0], m->x[0], m->b[0]);
}

/* Alg 1: while maxNormRes > tol: V-cycle; maxNormRes.  The cycle
 * cap (20, "-n 20") is a parameter.  norms[0..cycles] are recorded if
 * norms != NULL (norms[0] = initial). Returns cycles done. */
int oracle_mg_solve(oracle_mg *m, double tol, int max_cycles, double *norms) {
  double nr = oracle_mg_norm(m);
  if (norms) norms[0] = nr;
  int c = 0;
  while (nr > tol && c < max_cycles) {
    oracle_mg_vcycle(m);
    nr = oracle_mg_norm(m);
    ++c;
    if (norms) norms[c] = nr;
  }
  return c;
}

/* Point evaluation of one smooth+residual sweep for sampled parity checks at
 * full size: for each listed point p (lexicographic index), the value x' and
 * r that smooth+residual produces from x, b at level spacing h. */
void oracle_sweep_points(int nx, int ny, int nz, double h, const double *x, const double *b, const int64_t *pts,
                         int64_t npts, double *xn_out, double *r_out) {
  const double inv = 1.0 / (h * h);
  const double alpha = -6.0 * inv, beta = inv, gamma = (h * h) / 12.0;
#pragma omp parallel for schedule(static)
  for (int64_t q = 0; q < npts; ++q) {
    const int64_t p = pts[q];
    const int i = (int)(p % nx), j = (int)((p / nx) % ny), k = (int)(p / ((int64_t)nx * ny));
    const int iw = (i + nx - 1) % nx, ie = (i + 1) % nx, js = (j + ny - 1) % ny, jn = (j + 1) % ny;
    const int kb = (k + nz - 1) % nz, kt = (k + 1) % nz;
    const double sum = ((x[IDX(iw, j, k, nx, ny)] + x[IDX(ie, j, k, nx, ny)]) +
                        (x[IDX(i, js, k, nx, ny)] + x[IDX(i, jn, k, nx, ny)])) +
                       (x[IDX(i, j, kb, nx, ny)] + x[IDX(i, j, kt, nx, ny)]);
    const double a = alpha * x[p] + beta * sum;
    r_out[q] = b[p] - a;
    xn_out[q] = x[p] + gamma * (a - b[p]);
  }
}
