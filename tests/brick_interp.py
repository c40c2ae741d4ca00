"""Host brick interpreter (TEST INFRASTRUCTURE; neither the oracle nor the product).

Runs the V-cycle in numpy directly on the library's brick layout tables
(adjacency, coords, parent map, exchange plans obtained through the C ABI's
host-only ``mg_layout_*`` queries), so the layout and the packing-free
exchange plans can be checked against the lexicographic oracle on a machine
without a GPU.  numpy float64 ufuncs are separately rounded IEEE ops, written
in the canonical order of DESIGN.md reading A8, so the comparison is bitwise.

Schedule: exchange x before EVERY sweep (no communication avoiding), b after
every restriction -- the simplest legal schedule; the CA schedules are
exercised on the GPU.
"""
from __future__ import annotations

import numpy as np


class RankLevel:
    def __init__(self, lay, level):
        self.info = lay.info(level)
        self.adj = lay.adjacency(level)
        self.coords = lay.coords(level)
        self.parent = lay.parent(level)
        self.sends = lay.plan(level, 0)
        self.recvs = lay.plan(level, 1)
        self.n_owned = self.info["owned"]
        self.n_alloc = self.info["alloc"]
        self.n = self.info["n"]  # x, y, z
        self.E = self.n[0] // self.info["nb"][0]  # brick edge (8, or 4)
        self.mirror = lay.mirror(level)  # non-periodic bc (reading A22): (ghost, source, reflected axes)
        self.mirror_sign = -1.0 if lay.p.bc == 1 else 1.0

    def zeros(self):
        E = self.E
        return np.zeros((self.n_alloc, E, E, E))  # [brick][k][j][i]

    def to_bricks(self, lex):  # lex (nz, ny, nx)
        out = self.zeros()
        c = self.coords[: self.n_owned]
        for q in range(self.n_owned):
            cx, cy, cz = c[q]
            E = self.E
            out[q] = lex[E * cz:E * cz + E, E * cy:E * cy + E, E * cx:E * cx + E]
        return out

    def from_bricks(self, br):
        nx, ny, nz = self.n
        lex = np.empty((nz, ny, nx))
        c = self.coords[: self.n_owned]
        for q in range(self.n_owned):
            cx, cy, cz = c[q]
            E = self.E
            lex[E * cz:E * cz + E, E * cy:E * cy + E, E * cx:E * cx + E] = br[q]
        return lex


def padded(x, adj, nb):
    """(nb, E+2, E+2, E+2) = each brick plus its 6 face halos via the adjacency table."""
    E = x.shape[-1]
    X = np.zeros((nb, E + 2, E + 2, E + 2))
    m = slice(1, E + 1)
    X[:, m, m, m] = x[:nb]
    X[:, m, m, 0] = x[adj[:nb, 0]][:, :, :, E - 1]  # W: neighbour's i = E - 1
    X[:, m, m, E + 1] = x[adj[:nb, 1]][:, :, :, 0]  # E
    X[:, m, 0, m] = x[adj[:nb, 2]][:, :, E - 1, :]  # S
    X[:, m, E + 1, m] = x[adj[:nb, 3]][:, :, 0, :]  # N
    X[:, 0, m, m] = x[adj[:nb, 4]][:, E - 1, :, :]  # B
    X[:, E + 1, m, m] = x[adj[:nb, 5]][:, 0, :, :]  # T
    return X


def coeffs(h):
    inv = 1.0 / (h * h)
    return -6.0 * inv, inv, (h * h) / 12.0


def sweep(x, b, adj, nb, h):
    """Returns (x', r) on bricks [0, nb): a = alpha x + beta sum6; r = b - a; x' = x + gamma (a - b)."""
    al, be, ga = coeffs(h)
    E = x.shape[-1]
    X = padded(x, adj, nb)
    m, lo, hi = slice(1, E + 1), slice(0, E), slice(2, E + 2)
    c = X[:, m, m, m]
    s = ((X[:, m, m, lo] + X[:, m, m, hi]) + (X[:, m, lo, m] + X[:, m, hi, m])) + (X[:, lo, m, m] + X[:, hi, m, m])
    a = al * c + be * s
    xn = x.copy()
    r = np.zeros_like(x)
    r[:nb] = b[:nb] - a
    xn[:nb] = c + ga * (a - b[:nb])
    return xn, r


def restrict(rf, fine: RankLevel, bc):
    H = fine.E // 2
    for q in range(fine.n_owned):
        pr = int(fine.parent[q])
        cb, o = pr >> 3, pr & 7
        ox, oy, oz = o & 1, (o >> 1) & 1, o >> 2
        f = rf[q]
        v = 0.125 * (((f[0::2, 0::2, 0::2] + f[0::2, 0::2, 1::2]) + (f[0::2, 1::2, 0::2] + f[0::2, 1::2, 1::2]))
                     + ((f[1::2, 0::2, 0::2] + f[1::2, 0::2, 1::2]) + (f[1::2, 1::2, 0::2] + f[1::2, 1::2, 1::2])))
        bc[cb, H * oz:H * oz + H, H * oy:H * oy + H, H * ox:H * ox + H] = v


def interp(xf, fine: RankLevel, xc):
    H = fine.E // 2
    for q in range(fine.n_owned):
        pr = int(fine.parent[q])
        cb, o = pr >> 3, pr & 7
        ox, oy, oz = o & 1, (o >> 1) & 1, o >> 2
        blk = xc[cb, H * oz:H * oz + H, H * oy:H * oy + H, H * ox:H * ox + H]
        xf[q] = xf[q] + np.repeat(np.repeat(np.repeat(blk, 2, 0), 2, 1), 2, 2)


def apply_mirror(f, L: RankLevel):
    """Domain-face ghost bricks from their reflected sources (after the receives)."""
    for dst, src, mask in L.mirror:
        blk = f[src]
        for a, ax in ((0, 2), (1, 1), (2, 0)):  # brick array axes [k][j][i]
            if mask >> a & 1:
                blk = np.flip(blk, axis=ax)
        f[dst] = blk * (L.mirror_sign ** bin(int(mask)).count("1"))


def exchange_local(fields, levels):
    """In-process exchange of ghost bricks for all ranks (fields[r] is that rank's array)."""
    out = [f.copy() for f in fields]
    for r, L in enumerate(levels):
        for peer, d, run, local, remote, count in L.recvs:
            out[r][local:local + count] = fields[peer][remote:remote + count]
    for r, L in enumerate(levels):
        apply_mirror(out[r], L)
    return out


def replicated_bottom(b_own, gathered_fn, src, mine, gadj, h, bottom):
    """The library's replicated bottom (Layout::repl): all-gather the owned coarsest b bricks
    (rank-major), permute them into the global coarsest level by `src`, `bottom` sweeps from x = 0 on
    that periodic grid, this rank's owned x by `mine`.  gathered_fn(b_own) -> [world * n_own] bricks."""
    gb = gathered_fn(b_own)[src]
    ng = len(src)
    x = np.zeros((ng,) + b_own.shape[1:])
    for _ in range(bottom):
        x, _ = sweep(x, gb, gadj, ng, h)
    return x[mine]


def vcycle_ranks(xs, bs, ranks, L, h0, pre, post, bottom, exchange=exchange_local, bottom_fn=None):
    """One V-cycle (Alg 2) over every rank's brick fields.  ranks[r][l] = RankLevel.
    xs, bs: per-rank lists of per-level arrays (level-0 b must already hold valid ghosts).
    `exchange(fields, levels)` fills ghost bricks (in-process or over torch.distributed).
    bottom_fn(xs, bs, h) (optional) replaces the exchanged bottom sweeps."""
    R = len(ranks)
    own = lambda r, l: ranks[r][l].n_owned  # noqa: E731
    rs = [[None] * L for _ in range(R)]
    for l in range(L - 1):
        h = h0 * 2**l
        for s in range(pre):
            xs_l = exchange([xs[r][l] for r in range(R)], [ranks[r][l] for r in range(R)])
            for r in range(R):
                xs[r][l], rs[r][l] = sweep(xs_l[r], bs[r][l], ranks[r][l].adj, own(r, l), h)
        for r in range(R):
            bs[r][l + 1] = ranks[r][l + 1].zeros()
            restrict(rs[r][l], ranks[r][l], bs[r][l + 1])
            xs[r][l + 1] = ranks[r][l + 1].zeros()
        bl = exchange([bs[r][l + 1] for r in range(R)], [ranks[r][l + 1] for r in range(R)])
        for r in range(R):
            bs[r][l + 1] = bl[r]
    h = h0 * 2 ** (L - 1)
    if bottom_fn is not None:
        bottom_fn(xs, bs, h)
        bottom = 0
    for s in range(bottom):
        xl = exchange([xs[r][L - 1] for r in range(R)], [ranks[r][L - 1] for r in range(R)])
        for r in range(R):
            xs[r][L - 1], _ = sweep(xl[r], bs[r][L - 1], ranks[r][L - 1].adj, own(r, L - 1), h)
    for l in range(L - 2, -1, -1):
        h = h0 * 2**l
        for r in range(R):
            interp(xs[r][l], ranks[r][l], xs[r][l + 1])
        for s in range(post):
            xl = exchange([xs[r][l] for r in range(R)], [ranks[r][l] for r in range(R)])
            for r in range(R):
                xs[r][l], _ = sweep(xl[r], bs[r][l], ranks[r][l].adj, own(r, l), h)
    return xs
