"""Mutation check for the oracle pins (run by hand: python tools/oracle_mutations.py).

Applies one plausible slip at a time to oracle/mg_oracle.c, rebuilds, runs
tests/test_oracle_pins.py + tests/test_oracle_pins_bc_vc.py and reports whether some pin catches it.
The source is restored afterwards.  Last run: every mutation below CAUGHT (22 of 22).
"""
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SRC = os.path.join(ROOT, "oracle", "mg_oracle.c")

MUTATIONS = {
    "gamma_sign_smooth_residual": ("    x[p] = x[p] + gamma * (Ax[p] - b[p]);\n  }", "    x[p] = x[p] - gamma * (Ax[p] - b[p]);\n  }"),
    "restriction_index": ("r010 = r[IDX(i, j + 1, k, nx, ny)]", "r010 = r[IDX(i + 1, j, k, nx, ny)]"),
    "interp_parent_axes": ("xc[IDX(i / 2, j / 2, k / 2, cx, cy)]", "xc[IDX(i / 2, k / 2 % cy, j / 2 % (nz/2), cx, cy)]"),
    "missing_initZero": ("    oracle_init_zero(lvl_n(m, l + 1), m->x[l + 1]);", ""),
    "h_not_doubled_per_level": ("m->h[l] = h0 * (double)s;", "m->h[l] = h0;"),
    "dropped_neighbour": ("(xb + xt)", "(xb + xb)"),
    "residual_sign": ("r[p] = b[p] - Ax[p];", "r[p] = Ax[p] - b[p];"),
    "bottom_without_smooth": ("        level_smooth(m, l, 0, it, 0); /* smooth (damped Jacobi) */", ""),
    # CG bottom variant (reading A21)
    "cg_beta_inverted": ("const double beta = rr2 / rr;", "const double beta = rr / rr2;"),
    "cg_residual_sign": ("r[i] = r[i] - alpha * q[i];", "r[i] = r[i] + alpha * q[i];"),
    "cg_mean_not_removed": ("r[i] = b[i] - m;", "r[i] = b[i];"),
    "dot_tree_left_to_right": ("for (size_t i = 0; i + s < n; i += 2 * s) v[i] = v[i] + v[i + s];",
                               "for (size_t i = 0; i + s < n; i += 2 * s) v[i] = v[i] + v[i + s];\n"
                               "  if (n > 1) { double t = v[0]; v[0] = a[0] * b[0];"
                               " for (size_t i = 1; i < n; ++i) v[0] = v[0] + a[i] * b[i]; (void)t; }"),
    # smoother variants in the V-cycle (readings A19, A20)
    "gsrb_black_before_red": ("oracle_gsrb_half(d[0], d[1], d[2], m->h[l], c,", "oracle_gsrb_half(d[0], d[1], d[2], m->h[l], 1 - c,"),
    "chebyshev_pre_uses_post_count": ("    level_smooth(m, l, n, it, 1);", "    level_smooth(m, l, m->post, it, 1);"),
    "chebyshev_step_order_reversed": ("oracle_chebyshev_gamma(m->h[l], n, it, m->rho)", "oracle_chebyshev_gamma(m->h[l], n, n - 1 - it, m->rho)"),
    # boundary conditions (reading A22) and variable coefficients (reading A23)
    "dirichlet_image_sign": ("return bc == 1 ? -xp : xp;", "return bc == 1 ? xp : -xp;"),
    "boundary_wraps": ("  if (bc == 0) return (j + n) % n;", "  return (j + n) % n;"),
    "vc_face_one_sided": ("t[q] = ((cp + cn) * 0.5) * (xn - xp);", "t[q] = cp * (xn - xp);"),
    "vc_boundary_face_coef": ("? cp : c[IDX(a, b, cc, nx, ny)];\n          t[q]", "? 0.5 * cp : c[IDX(a, b, cc, nx, ny)];\n          t[q]"),
    "vc_gamma_weight": ("const double g = 0.5 * (h * h);", "const double g = 0.25 * (h * h);"),
    "vc_coarse_coef_not_restricted": ("      oracle_restriction(m->n[l - 1][0], m->n[l - 1][1], m->n[l - 1][2], m->c[l - 1], m->c[l]);",
                                      "      for (size_t q = 0; q < lvl_n(m, l); ++q) m->c[l][q] = 1.0;"),
    "norm_drops_nan": ("if (a > mt || a != a) mt = a;", "if (a > mt) mt = a;"),
}


def main():
    orig = open(SRC).read()
    ok = True
    try:
        for name, (a, b) in MUTATIONS.items():
            assert a in orig, name
            open(SRC, "w").write(orig.replace(a, b, 1))
            r = subprocess.run([sys.executable, "-m", "pytest", "tests/test_oracle_pins.py",
                                "tests/test_oracle_pins_bc_vc.py", "-q", "-x",
                                "-p", "no:cacheprovider"], capture_output=True, text=True, cwd=ROOT)
            caught = r.returncode != 0
            ok &= caught
            print(f"{name:32s} {'CAUGHT' if caught else 'MISSED'}")
    finally:
        open(SRC, "w").write(orig)
        sys.path.insert(0, ROOT)
        import oracle
        oracle.build(force=True)
    return 0 if ok else 1


if __name__ == "__main__":
    sys.exit(main())
