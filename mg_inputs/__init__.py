"""Seeded synthetic input generators shared by the oracle tests and the CUDA path.

This module holds NO arithmetic of the method (no stencil, smoother, transfer
operator or norm) -- only the inputs both sides consume, so that the oracle
(``oracle/``) and the product (``paper_conf_sc_antepara0jh24_b200``) can be fed
bit-identical arrays without importing each other.

Array convention: numpy shape ``(nz, ny, nx)``, C order, i.e. lexicographic
index ``i + nx*(j + ny*k)`` with i fastest (the order ``mg_set_rhs`` takes).

Recipes:

* ``sin_rhs``      -- the paper's model problem b = sin(2 pi x) sin(2 pi y)
  sin(2 pi z) at cell centres x_d = (i_d + 1/2) h0 of a periodic box
  of side L_d = N_d h0, h0 = 1/max_d N_d (reading A7), written as
  prod_d sin(2 pi x_d / L_d).  Zero mean by symmetry.
* ``random_rhs``   -- uniform(-1, 1) from ``numpy.random.default_rng(seed)``,
  minus its mean (periodic Poisson is singular; reading A12).
* ``random_field`` -- uniform(-1, 1), no mean removal (per-operator tests).

Rank slabs: ``local_block`` cuts the (k, j, i) block a rank owns under a
``proc_grid = (px, py, pz)`` decomposition with rank = cx + px*(cy + py*cz);
the same values as the global array, so decomposed runs see bit-identical
inputs.
"""
from __future__ import annotations

import numpy as np


def default_h0(shape) -> float:
    return 1.0 / float(max(shape))


def _axis_sin(n_global: int, h0: float, lo: int, n: int) -> np.ndarray:
    i = np.arange(lo, lo + n, dtype=np.float64)
    Ld = n_global * h0
    return np.sin(2.0 * np.pi * ((i + 0.5) * h0) / Ld)


def sin_rhs(global_shape, h0: float | None = None, offset=(0, 0, 0), local_shape=None) -> np.ndarray:
    """b = prod_d sin(2 pi x_d / L_d) on the block [offset, offset+local_shape) (k, j, i order)."""
    gz, gy, gx = (int(s) for s in global_shape)
    h0 = default_h0(global_shape) if h0 is None else float(h0)
    local_shape = global_shape if local_shape is None else local_shape
    nz, ny, nx = (int(s) for s in local_shape)
    oz, oy, ox = (int(s) for s in offset)
    sz = _axis_sin(gz, h0, oz, nz)
    sy = _axis_sin(gy, h0, oy, ny)
    sx = _axis_sin(gx, h0, ox, nx)
    return np.ascontiguousarray((sz[:, None, None] * sy[None, :, None]) * sx[None, None, :])


def random_field(shape, seed: int) -> np.ndarray:
    rng = np.random.default_rng(seed)
    return rng.uniform(-1.0, 1.0, size=tuple(int(s) for s in shape))


def random_rhs(shape, seed: int) -> np.ndarray:
    b = random_field(shape, seed)
    return np.ascontiguousarray(b - b.mean())


def rank_coords(rank: int, proc_grid):
    px, py, pz = proc_grid
    return rank % px, (rank // px) % py, rank // (px * py)


def local_block(global_array: np.ndarray, rank: int, proc_grid) -> np.ndarray:
    """The (nz/pz, ny/py, nx/px) block rank owns (rank = cx + px*(cy + py*cz))."""
    gz, gy, gx = global_array.shape
    px, py, pz = proc_grid
    cx, cy, cz = rank_coords(rank, proc_grid)
    lz, ly, lx = gz // pz, gy // py, gx // px
    return np.ascontiguousarray(global_array[cz * lz:(cz + 1) * lz, cy * ly:(cy + 1) * ly, cx * lx:(cx + 1) * lx])


def local_sin_rhs(global_shape, rank: int, proc_grid, h0: float | None = None) -> np.ndarray:
    gz, gy, gx = global_shape
    px, py, pz = proc_grid
    cx, cy, cz = rank_coords(rank, proc_grid)
    lz, ly, lx = gz // pz, gy // py, gx // px
    return sin_rhs(global_shape, h0, offset=(cz * lz, cy * ly, cx * lx), local_shape=(lz, ly, lx))


def random_coef(shape, seed: int, lo: float = 0.5, hi: float = 2.0) -> np.ndarray:
    """Cell coefficients c = U(lo, hi) > 0 of the variable-coefficient variant (reading A23): a rough
    field (a factor 4 between neighbours at most), the hard case for the face averages."""
    rng = np.random.default_rng(10_000 + seed)
    return np.ascontiguousarray(rng.uniform(lo, hi, size=tuple(int(s) for s in shape)))


def smooth_coef(global_shape, h0: float | None = None) -> np.ndarray:
    """c = 1 + 0.5 prod_d sin(2 pi x_d / L_d) at the cell centres (in [0.5, 1.5]): the smooth
    coefficient of the timing recipe for the variable-coefficient variant."""
    return np.ascontiguousarray(1.0 + 0.5 * sin_rhs(global_shape, h0))


def dirichlet_sin_rhs(global_shape, h0: float | None = None) -> np.ndarray:
    """b = prod_d sin(pi x_d / L_d): the lowest Dirichlet mode (vanishes on the domain faces), the
    timing right-hand side of the non-periodic variant (reading A22)."""
    gz, gy, gx = (int(s) for s in global_shape)
    h0 = default_h0(global_shape) if h0 is None else float(h0)

    def ax(n):
        return np.sin(np.pi * ((np.arange(n, dtype=np.float64) + 0.5) * h0) / (n * h0))

    return np.ascontiguousarray((ax(gz)[:, None, None] * ax(gy)[None, :, None]) * ax(gx)[None, None, :])
