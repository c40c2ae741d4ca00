"""CPU oracle for the brick-GMG V-cycle -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this package.  The
product package ``paper_conf_sc_antepara0jh24_b200`` never imports it; the two
share no code.

The arithmetic lives in ``mg_oracle.c`` (plain C, fp64, ``-ffp-contract=off``,
OpenMP over k-planes).  Every function there cites the PAPER.md passage it
follows.  This module only compiles it (gcc) and marshals numpy arrays via
ctypes.  Grids are global, lexicographic, periodic, cell-centred, shaped
``(nz, ny, nx)`` in numpy (i fastest in memory).

Variants beyond the paper: Chebyshev / red-black Gauss-Seidel smoothers, a CG
bottom, homogeneous Dirichlet / Neumann boundaries (reading A22) and variable coefficients
(reading A23) -- see ``OracleMG``'s arguments.

Parity status: every function is pinned by a
``-m "not gpu"`` test in ``tests/test_oracle_pins.py`` against closed forms,
invariants or an independent SciPy sparse-matrix V-cycle; nothing is
"parity unpinned" except the paper's "12 V-cycles" claim (reading A13), which
no function here depends on.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "mg_oracle.c")
_LIB = os.path.join(_HERE, "_mg_oracle.so")
_lock = threading.Lock()
_lib = None

CFLAGS = ["-O2", "-fopenmp", "-ffp-contract=off", "-fno-fast-math", "-fPIC", "-shared", "-std=c11"]


def build(force: bool = False) -> str:
    """Compile mg_oracle.c -> _mg_oracle.so (gcc).  Returns the .so path."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", *CFLAGS, _SRC, "-o", tmp, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    with _lock:
        if _lib is not None:
            return _lib
        lib = ctypes.CDLL(build())
        D, I, P, S = ctypes.c_double, ctypes.c_int, ctypes.c_void_p, ctypes.c_size_t
        sig = {
            "oracle_set_threads": (None, [I]),
            "oracle_get_threads": (I, []),
            "oracle_apply_op": (None, [I, I, I, D, P, P]),
            "oracle_apply_op_bc": (None, [I, I, I, D, I, P, P]),
            "oracle_apply_op_vc": (None, [I, I, I, D, I, P, P, P]),
            "oracle_vc_gamma": (None, [I, I, I, D, I, P, P]),
            "oracle_smooth_residual_field": (None, [S, P, P, P, P, P]),
            "oracle_max_norm_residual_ex": (D, [I, I, I, D, I, P, P, P]),
            "oracle_mg_set_bc": (I, [P, I]),
            "oracle_mg_set_coef": (I, [P, P]),
            "oracle_smooth": (None, [S, D, P, P, P]),
            "oracle_smooth_gamma": (None, [S, D, P, P, P]),
            "oracle_smooth_residual_gamma": (None, [S, D, P, P, P, P]),
            "oracle_chebyshev_gamma": (D, [D, I, I, I]),
            "oracle_gsrb_half": (None, [I, I, I, D, I, P, P, P, P]),
            "oracle_mg_set_smoother": (None, [P, I, I]),
            "oracle_mg_set_bottom_solver": (I, [P, I]),
            "oracle_dot_tree": (D, [S, P, P]),
            "oracle_cg": (None, [I, I, I, D, I, P, P]),
            "oracle_smooth_residual": (None, [S, D, P, P, P, P]),
            "oracle_restriction": (None, [I, I, I, P, P]),
            "oracle_init_zero": (None, [S, P]),
            "oracle_interpolation_increment": (None, [I, I, I, P, P]),
            "oracle_max_norm_residual": (D, [I, I, I, D, P, P]),
            "oracle_mg_create": (P, [I, I, I, I, D, I, I, I]),
            "oracle_mg_destroy": (None, [P]),
            "oracle_mg_set_b": (None, [P, P]),
            "oracle_mg_set_x": (None, [P, P]),
            "oracle_mg_get_x": (None, [P, P]),
            "oracle_mg_get_level": (I, [P, I, I, P]),
            "oracle_mg_vcycle": (None, [P]),
            "oracle_mg_norm": (D, [P]),
            "oracle_mg_solve": (I, [P, D, I, P]),
            "oracle_sweep_points": (None, [I, I, I, D, P, P, P, ctypes.c_int64, P, P]),
        }
        for name, (res, args) in sig.items():
            f = getattr(lib, name)
            f.restype = res
            f.argtypes = args
        _lib = lib
        return lib


def _ptr(a: np.ndarray):
    assert a.flags["C_CONTIGUOUS"], "oracle arrays must be C-contiguous"
    return a.ctypes.data_as(ctypes.c_void_p)


def _f64(a) -> np.ndarray:
    return np.ascontiguousarray(a, dtype=np.float64)


def set_threads(n: int) -> None:
    _load().oracle_set_threads(int(n))


def get_threads() -> int:
    return int(_load().oracle_get_threads())


def default_h0(shape) -> float:
    """Reading A7: h0 = 1 / max_d N_d (unit cube for cubic grids)."""
    return 1.0 / float(max(shape))


# ---------------------------------------------------------------- single ops
def apply_op(x: np.ndarray, h: float, bc: int = 0) -> np.ndarray:
    """The paper's 7-point operator; bc 1 / 2 = homogeneous Dirichlet / Neumann (reading A22)."""
    x = _f64(x)
    nz, ny, nx = x.shape
    out = np.empty_like(x)
    if bc:
        _load().oracle_apply_op_bc(nx, ny, nz, float(h), int(bc), _ptr(x), _ptr(out))
    else:
        _load().oracle_apply_op(nx, ny, nz, float(h), _ptr(x), _ptr(out))
    return out


def apply_op_vc(x: np.ndarray, c: np.ndarray, h: float, bc: int = 0) -> np.ndarray:
    """Variable-coefficient operator div(c grad x) with face values (c_p + c_n)/2 (reading A23)."""
    x, c = _f64(x), _f64(c)
    assert c.shape == x.shape
    nz, ny, nx = x.shape
    out = np.empty_like(x)
    _load().oracle_apply_op_vc(nx, ny, nz, float(h), int(bc), _ptr(c), _ptr(x), _ptr(out))
    return out


def vc_gamma(c: np.ndarray, h: float, bc: int = 0) -> np.ndarray:
    """Per-cell damped-Jacobi step (0.5 h^2) / (sum of the six face coefficients) (reading A23)."""
    c = _f64(c)
    nz, ny, nx = c.shape
    out = np.empty_like(c)
    _load().oracle_vc_gamma(nx, ny, nz, float(h), int(bc), _ptr(c), _ptr(out))
    return out


def smooth_residual_field(x: np.ndarray, Ax: np.ndarray, b: np.ndarray, gam: np.ndarray):
    """x + gamma_p (Ax - b) and r = b - Ax with a step per cell (reading A23)."""
    x = _f64(x).copy()
    Ax, b, gam = _f64(Ax), _f64(b), _f64(gam)
    r = np.empty_like(x)
    _load().oracle_smooth_residual_field(x.size, _ptr(gam), _ptr(x), _ptr(Ax), _ptr(b), _ptr(r))
    return x, r


def smooth(x: np.ndarray, Ax: np.ndarray, b: np.ndarray, h: float) -> np.ndarray:
    x = _f64(x).copy()
    Ax, b = _f64(Ax), _f64(b)
    _load().oracle_smooth(x.size, float(h), _ptr(x), _ptr(Ax), _ptr(b))
    return x


def smooth_residual(x: np.ndarray, Ax: np.ndarray, b: np.ndarray, h: float):
    x = _f64(x).copy()
    Ax, b = _f64(Ax), _f64(b)
    r = np.empty_like(x)
    _load().oracle_smooth_residual(x.size, float(h), _ptr(x), _ptr(Ax), _ptr(b), _ptr(r))
    return x, r


def smooth_gamma(x: np.ndarray, Ax: np.ndarray, b: np.ndarray, gamma: float) -> np.ndarray:
    """x + gamma*(Ax - b) with an explicit step (the Chebyshev smoother's sweeps)."""
    x = _f64(x).copy()
    Ax, b = _f64(Ax), _f64(b)
    _load().oracle_smooth_gamma(x.size, float(gamma), _ptr(x), _ptr(Ax), _ptr(b))
    return x


def gsrb_half(x: np.ndarray, Ax: np.ndarray, b: np.ndarray, h: float, colour: int):
    """One red (colour 0) or black (1) Gauss-Seidel half-sweep (reading A20); returns (x', r)."""
    x = _f64(x).copy()
    Ax, b = _f64(Ax), _f64(b)
    r = np.empty_like(x)
    nz, ny, nx = x.shape
    _load().oracle_gsrb_half(nx, ny, nz, float(h), int(colour), _ptr(x), _ptr(Ax), _ptr(b), _ptr(r))
    return x, r


def chebyshev_gamma(h: float, s: int, k: int, rho: int) -> float:
    """Step of sweep k of an s-sweep Chebyshev smoother over mu in [mu_max/rho, mu_max] (reading A19)."""
    return float(_load().oracle_chebyshev_gamma(float(h), int(s), int(k), int(rho)))


def dot_tree(a: np.ndarray, b: np.ndarray) -> float:
    """Fixed-order dot product of reading A21 (stride-doubling pairwise tree, lexicographic)."""
    a, b = _f64(a), _f64(b)
    assert a.size == b.size
    return float(_load().oracle_dot_tree(a.size, _ptr(a), _ptr(b)))


def cg(b: np.ndarray, h: float, iters: int) -> np.ndarray:
    """`iters` CG iterations on A x = b from x = 0 (reading A21, the CG bottom variant)."""
    b = _f64(b)
    x = np.zeros_like(b)
    nz, ny, nx = b.shape
    _load().oracle_cg(nx, ny, nz, h, int(iters), _ptr(x), _ptr(b))
    return x


def restriction(r: np.ndarray) -> np.ndarray:
    r = _f64(r)
    nz, ny, nx = r.shape
    out = np.empty((nz // 2, ny // 2, nx // 2), dtype=np.float64)
    _load().oracle_restriction(nx, ny, nz, _ptr(r), _ptr(out))
    return out


def interpolation_increment(xc: np.ndarray, x: np.ndarray) -> np.ndarray:
    xc = _f64(xc)
    x = _f64(x).copy()
    nz, ny, nx = x.shape
    assert xc.shape == (nz // 2, ny // 2, nx // 2)
    _load().oracle_interpolation_increment(nx, ny, nz, _ptr(xc), _ptr(x))
    return x


def max_norm_residual(x: np.ndarray, b: np.ndarray, h: float, bc: int = 0, c: np.ndarray | None = None) -> float:
    x, b = _f64(x), _f64(b)
    nz, ny, nx = x.shape
    if bc or c is not None:
        cp = None if c is None else _ptr(_f64(c))
        return float(_load().oracle_max_norm_residual_ex(nx, ny, nz, float(h), int(bc), cp, _ptr(x), _ptr(b)))
    return float(_load().oracle_max_norm_residual(nx, ny, nz, float(h), _ptr(x), _ptr(b)))


def sweep_points(x: np.ndarray, b: np.ndarray, h: float, pts: np.ndarray):
    """smooth+residual evaluated only at lexicographic indices ``pts``."""
    x, b = _f64(x), _f64(b)
    nz, ny, nx = x.shape
    pts = np.ascontiguousarray(pts, dtype=np.int64)
    xn = np.empty(pts.size, dtype=np.float64)
    r = np.empty(pts.size, dtype=np.float64)
    _load().oracle_sweep_points(nx, ny, nz, float(h), _ptr(x), _ptr(b), _ptr(pts), pts.size, _ptr(xn), _ptr(r))
    return xn, r


# ----------------------------------------------------------------- hierarchy
class OracleMG:
    """Alg 1 / Alg 2 on a global periodic grid of shape (nz, ny, nx)."""

    def __init__(self, shape, levels: int, pre: int = 12, post: int = 12, bottom: int = 100, h0: float | None = None,
                 smoother: int = 0, cheby_ratio: int = 6, bottom_solver: int = 0, bc: int = 0,
                 coef: np.ndarray | None = None):
        """bc: 0 periodic (the paper), 1 Dirichlet, 2 Neumann (reading A22); coef: level-0 cell
        coefficients c > 0 of the variable-coefficient operator (reading A23), None = the paper's."""
        nz, ny, nx = (int(s) for s in shape)
        self.shape = (nz, ny, nx)
        self.levels = int(levels)
        self.h0 = default_h0(shape) if h0 is None else float(h0)
        self._lib = _load()
        self._h = self._lib.oracle_mg_create(nx, ny, nz, self.levels, self.h0, int(pre), int(post), int(bottom))
        if not self._h:
            raise ValueError(f"oracle_mg_create failed for shape={shape} levels={levels}")
        self._lib.oracle_mg_set_smoother(self._h, int(smoother), int(cheby_ratio))
        if self._lib.oracle_mg_set_bc(self._h, int(bc)) != 0:
            raise ValueError(f"oracle: bc={bc} not supported")
        if coef is not None:
            coef = _f64(coef)
            assert coef.shape == self.shape
            if self._lib.oracle_mg_set_coef(self._h, _ptr(coef)) != 0:
                raise ValueError("oracle: variable coefficients not supported with this configuration")
        if self._lib.oracle_mg_set_bottom_solver(self._h, int(bottom_solver)) != 0:
            raise ValueError("oracle: the CG bottom needs the periodic constant-coefficient operator")

    def close(self):
        if getattr(self, "_h", None):
            self._lib.oracle_mg_destroy(self._h)
            self._h = None

    __del__ = close

    def set_b(self, b: np.ndarray):
        b = _f64(b)
        assert b.shape == self.shape
        self._lib.oracle_mg_set_b(self._h, _ptr(b))

    def set_x(self, x: np.ndarray | None):
        if x is None:
            self._lib.oracle_mg_set_x(self._h, None)
        else:
            x = _f64(x)
            assert x.shape == self.shape
            self._lib.oracle_mg_set_x(self._h, _ptr(x))

    def get_x(self) -> np.ndarray:
        out = np.empty(self.shape, dtype=np.float64)
        self._lib.oracle_mg_get_x(self._h, _ptr(out))
        return out

    def level_shape(self, l: int):
        return tuple(s >> l for s in self.shape)

    def get_level(self, l: int, which: str) -> np.ndarray:
        code = {"x": 0, "b": 1, "r": 2, "Ax": 3}[which]
        out = np.empty(self.level_shape(l), dtype=np.float64)
        rc = self._lib.oracle_mg_get_level(self._h, l, code, _ptr(out))
        assert rc == 0
        return out

    def vcycle(self):
        self._lib.oracle_mg_vcycle(self._h)

    def norm(self) -> float:
        return float(self._lib.oracle_mg_norm(self._h))

    def solve(self, tol: float = 1e-10, max_cycles: int = 20):
        norms = np.zeros(max_cycles + 1, dtype=np.float64)
        c = int(self._lib.oracle_mg_solve(self._h, float(tol), int(max_cycles), _ptr(norms)))
        return c, norms[: c + 1].copy()
