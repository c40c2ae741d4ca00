"""CPU tests of the brick layout, adjacency, region ordering and exchange plans
(host-only C-ABI queries; no GPU), plus a bitwise V-cycle of the host brick
interpreter on those tables against the lexicographic oracle."""
import os
import itertools

import numpy as np
import pytest

import mg_inputs
from paper_conf_sc_antepara0jh24_b200 import mg
from tests import brick_interp as bi

FACE = [(-1, 0, 0), (1, 0, 0), (0, -1, 0), (0, 1, 0), (0, 0, -1), (0, 0, 1)]


def layouts(n_local, proc_grid, L, ghost_mode=0, **kw):
    p = mg.params(n_local, proc_grid, num_levels=L, ghost_mode=ghost_mode, **kw)
    world = proc_grid[0] * proc_grid[1] * proc_grid[2]
    return p, [mg.Layout(p, r, world) for r in range(world)]


CASES = [((32, 32, 32), (1, 1, 1), 3, 0), ((32, 32, 32), (1, 1, 1), 3, 1), ((32, 16, 16), (2, 1, 1), 2, 0),
         ((16, 16, 16), (2, 2, 2), 2, 0), ((16, 16, 32), (1, 2, 3), 2, 0), ((48, 32, 16), (3, 1, 2), 2, 0)]


@pytest.mark.parametrize("n_local,pg,L,gm", CASES)
def test_adjacency_consistent_with_coords(n_local, pg, L, gm):
    """adj[b][face] is the brick at coords(b) + face (periodic wrap on non-ghost axes;
    the zero brick past the ghost shell), and adjacency is symmetric."""
    _, lays = layouts(n_local, pg, L, gm)
    for lay in lays:
        for l in range(L):
            inf = lay.info(l)
            adj, co = lay.adjacency(l), lay.coords(l)
            stored = inf["owned"] + inf["nghost"]
            index = {tuple(c): q for q, c in enumerate(co)}
            assert len(index) == stored  # no duplicates
            assert np.all(adj[:, 6] == np.arange(stored))
            for q in range(stored):
                for f, d in enumerate(FACE):
                    e = [int(co[q][a]) + d[a] for a in range(3)]
                    for a in range(3):
                        if not inf["ghost"][a]:
                            e[a] %= inf["nb"][a]
                    want = index.get(tuple(e), inf["zero_brick"])
                    assert adj[q, f] == want
                    if q < inf["owned"]:  # owned bricks: every neighbour exists, symmetric
                        assert want != inf["zero_brick"]
                        back = adj[want, f ^ 1]
                        assert back == q


@pytest.mark.parametrize("n_local,pg,L,gm", CASES)
def test_region_order_interior_first_and_ghost_coverage(n_local, pg, L, gm):
    """Owned bricks: interior region first; ghosts: every ghost brick received
    exactly once from one contiguous run (packing-free)."""
    _, lays = layouts(n_local, pg, L, gm)
    for lay in lays:
        for l in range(L):
            inf = lay.info(l)
            co = lay.coords(l)
            nb, g = inf["nb"], inf["ghost"]
            own = co[: inf["owned"]]
            on_surface = np.zeros(inf["owned"], dtype=bool)
            for a in range(3):
                if g[a]:
                    on_surface |= (own[:, a] == 0) | (own[:, a] == nb[a] - 1)
            assert inf["interior"] == int((~on_surface).sum())
            assert not on_surface[: inf["interior"]].any() and on_surface[inf["interior"]:].all()
            recv = lay.plan(l, 1)
            hit = np.zeros(inf["nghost"], dtype=int)
            for peer, d, run, local, remote, count in recv:
                hit[local - inf["owned"]: local - inf["owned"] + count] += 1
                assert 0 <= remote and remote + count <= inf["owned"]
            assert np.all(hit == 1)


def test_42_messages_for_26_neighbours():
    """With the searched region order, a 3D decomposition needs 42 contiguous
    runs for the 26 neighbours (BrickLib-style message consolidation)."""
    _, lays = layouts((64, 64, 64), (2, 2, 2), 1)
    inf = lays[0].info(0)
    assert inf["send_runs"] == 42 and inf["recv_runs"] == 42
    assert inf["nghost"] == 10**3 - 8**3


def test_ghost_counts_match_survey():
    """512^3 per GPU ghost-shell bricks 8192 / 16640 / 25352 at 2 / 4 / 8 GPUs."""
    for pg, want in (((2, 1, 1), 8192), ((2, 2, 1), 16640), ((2, 2, 2), 25352)):
        p = mg.params((512, 512, 512), pg, num_levels=1)
        assert mg.Layout(p, 0, pg[0] * pg[1] * pg[2]).info(0)["nghost"] == want


@pytest.mark.parametrize("n_local,pg,L,gm", CASES)
def test_plans_match_pairwise_in_order(n_local, pg, L, gm):
    """NCCL matches sends and recvs of a rank pair in posting order: rank S's
    sends to R must equal R's recvs from S, run for run, in the same order."""
    _, lays = layouts(n_local, pg, L, gm)
    world = len(lays)
    for l in range(L):
        sends = [lay.plan(l, 0) for lay in lays]
        recvs = [lay.plan(l, 1) for lay in lays]
        for S in range(world):
            for R in range(world):
                s = sends[S][sends[S][:, 0] == R] if len(sends[S]) else np.zeros((0, 6))
                r = recvs[R][recvs[R][:, 0] == S] if len(recvs[R]) else np.zeros((0, 6))
                assert len(s) == len(r)
                for a, b in zip(s, r):
                    assert a[1] == b[1] and a[2] == b[2] and a[5] == b[5]  # dir, run, count
                    assert a[3] == b[4] and a[4] == b[3]  # sender local == receiver remote, and back


@pytest.mark.parametrize("n_local,pg,L,gm", CASES)
def test_parent_map(n_local, pg, L, gm):
    """Fine brick e -> coarse brick floor(e/2), octant e mod 2 (brick-by-brick
    inter-level operators)."""
    _, lays = layouts(n_local, pg, L, gm)
    lay = lays[-1]
    for l in range(L - 1):
        co, cco = lay.coords(l), lay.coords(l + 1)
        par = lay.parent(l)
        inf = lay.info(l)
        for q in range(inf["owned"]):
            pr = int(par[q])
            assert pr >= 0
            cb, o = pr >> 3, pr & 7
            e = co[q]
            assert tuple(cco[cb]) == tuple(int(v) // 2 for v in e)
            assert o == (e[0] % 2) + 2 * (e[1] % 2) + 4 * (e[2] % 2)


def global_to_ranks(glob, pg, L, lays):
    R = len(lays)
    ranks = [[bi.RankLevel(lays[r], l) for l in range(L)] for r in range(R)]
    return ranks


@pytest.mark.parametrize("n_local,pg,L,gm", CASES)
def test_brick_interpreter_vcycle_bitwise_vs_oracle(oracle_mod, n_local, pg, L, gm):
    """The layout tables + exchange plans reproduce the oracle's V-cycle bit for
    bit (12/12/100 scaled down to 3/3/20 for CPU time)."""
    p, lays = layouts(n_local, pg, L, gm)
    gshape = (n_local[2] * pg[2], n_local[1] * pg[1], n_local[0] * pg[0])
    b = mg_inputs.random_rhs(gshape, 7)
    pre, post, bottom = 3, 3, 20
    h0 = mg_inputs.default_h0(gshape)
    orc = oracle_mod.OracleMG(gshape, L, pre, post, bottom, h0)
    orc.set_b(b)
    orc.set_x(None)
    orc.vcycle()
    want = orc.get_x()
    R = len(lays)
    ranks = [[bi.RankLevel(lays[r], l) for l in range(L)] for r in range(R)]
    xs = [[ranks[r][l].zeros() for l in range(L)] for r in range(R)]
    bs = [[None] * L for _ in range(R)]
    for r in range(R):
        bs[r][0] = ranks[r][0].to_bricks(mg_inputs.local_block(b, r, pg))
    b0 = bi.exchange_local([bs[r][0] for r in range(R)], [ranks[r][0] for r in range(R)])
    for r in range(R):
        bs[r][0] = b0[r]
    xs = bi.vcycle_ranks(xs, bs, ranks, L, h0, pre, post, bottom)
    got = np.zeros(gshape)
    px, py, pz = pg
    for r in range(R):
        cx, cy, cz = mg_inputs.rank_coords(r, pg)
        nx, ny, nz = n_local
        got[cz * nz:(cz + 1) * nz, cy * ny:(cy + 1) * ny, cx * nx:(cx + 1) * nx] = ranks[r][0].from_bricks(xs[r][0])
    assert np.array_equal(got, want)


BC_CASES = [((32, 32, 32), (1, 1, 1), 3, 1), ((16, 32, 16), (2, 1, 1), 2, 1), ((16, 16, 16), (2, 2, 2), 2, 2),
            ((16, 16, 32), (1, 2, 3), 2, 1), ((32, 32, 32), (2, 1, 1), 3, 2)]


@pytest.mark.parametrize("n_local,pg,L,bc", BC_CASES)
def test_mirror_tables_and_dropped_runs(n_local, pg, L, bc):
    """Non-periodic bc (reading A22): every axis has a ghost shell; no run crosses a domain face;
    every ghost brick is filled exactly once, by a receive or by a mirror entry whose source is the
    brick reflected across exactly the domain faces it lies beyond (owned or received)."""
    _, lays = layouts(n_local, pg, L, bc=bc)
    for r, lay in enumerate(lays):
        cx, cy, cz = mg_inputs.rank_coords(r, pg)
        rc = (cx, cy, cz)
        for l in range(L):
            inf = lay.info(l)
            assert all(inf["ghost"])
            co = lay.coords(l)
            index = {tuple(c): q for q, c in enumerate(co)}
            got = np.zeros(inf["owned"] + inf["nghost"], dtype=int)
            for peer, d, run, local, remote, count in lay.plan(l, 1):
                got[local:local + count] += 1
                dd = (d % 3 - 1, (d // 3) % 3 - 1, d // 9 - 1)
                assert all(0 <= rc[a] + dd[a] < pg[a] for a in range(3))  # never across a domain face
            for peer, d, run, local, remote, count in lay.plan(l, 0):
                dd = (d % 3 - 1, (d // 3) % 3 - 1, d // 9 - 1)
                assert all(0 <= rc[a] - dd[a] < pg[a] for a in range(3))
            for dst, src, mask in lay.mirror(l):
                got[dst] += 1
                e, q = list(co[dst]), list(co[src])
                for a in range(3):
                    beyond = (e[a] < 0 and rc[a] == 0) or (e[a] >= inf["nb"][a] and rc[a] == pg[a] - 1)
                    assert bool(mask >> a & 1) == beyond
                    assert q[a] == (min(max(e[a], 0), inf["nb"][a] - 1) if beyond else e[a])
            assert np.all(got[inf["owned"]:] == 1) and np.all(got[:inf["owned"]] == 0)


@pytest.mark.parametrize("n_local,pg,L,bc", BC_CASES)
def test_brick_interpreter_bc_vcycle_bitwise_vs_oracle(oracle_mod, n_local, pg, L, bc):
    """Dirichlet / Neumann (reading A22) on the library's layout tables: exchanges plus mirror
    fills reproduce the oracle's V-cycle (3/3/20 sweeps) bit for bit, decomposed or not."""
    p, lays = layouts(n_local, pg, L, bc=bc)
    gshape = (n_local[2] * pg[2], n_local[1] * pg[1], n_local[0] * pg[0])
    b = mg_inputs.random_field(gshape, 17)
    pre, post, bottom = 3, 3, 20
    h0 = mg_inputs.default_h0(gshape)
    orc = oracle_mod.OracleMG(gshape, L, pre, post, bottom, h0, bc=bc)
    orc.set_b(b)
    orc.set_x(None)
    orc.vcycle()
    want = orc.get_x()
    R = len(lays)
    ranks = [[bi.RankLevel(lays[r], l) for l in range(L)] for r in range(R)]
    xs = [[ranks[r][l].zeros() for l in range(L)] for r in range(R)]
    bs = [[None] * L for _ in range(R)]
    for r in range(R):
        bs[r][0] = ranks[r][0].to_bricks(mg_inputs.local_block(b, r, pg))
    b0 = bi.exchange_local([bs[r][0] for r in range(R)], [ranks[r][0] for r in range(R)])
    for r in range(R):
        bs[r][0] = b0[r]
    xs = bi.vcycle_ranks(xs, bs, ranks, L, h0, pre, post, bottom)
    got = np.zeros(gshape)
    for r in range(R):
        cx, cy, cz = mg_inputs.rank_coords(r, pg)
        nx, ny, nz = n_local
        got[cz * nz:(cz + 1) * nz, cy * ny:(cy + 1) * ny, cx * nx:(cx + 1) * nx] = ranks[r][0].from_bricks(xs[r][0])
    assert np.array_equal(got, want)


def test_invalid_params_rejected():
    bad = [mg.params((30, 32, 32), num_levels=1),  # not a multiple of 8
           mg.params((32, 32, 32), num_levels=4),  # 32 not a multiple of 8*2^3
           mg.params((32, 32, 32), (2, 1, 1), num_levels=1)]  # proc grid != world 1
    for p in bad:
        with pytest.raises(mg.MGError):
            mg.Layout(p, 0, 1)
    p = mg.params((32, 32, 32), num_levels=2, ca_period=9)
    with pytest.raises(mg.MGError):
        mg.Layout(p, 0, 1)
    # CG bottom (reading A21) needs a coarsest grid of <= 8 bricks (here 64, and 64 globally)
    for pg in ((1, 1, 1), (2, 2, 2)):
        p = mg.params((64, 64, 64), pg, num_levels=2, bottom_solver=1)
        with pytest.raises(mg.MGError):
            mg.Layout(p, 0, pg[0] * pg[1] * pg[2])
    mg.Layout(mg.params((64, 64, 64), num_levels=4, bottom_solver=1), 0, 1)  # 8^3 coarsest: accepted


# ------------------------------------------------- two-sweep pencil plans (sweep2p.cu, kind 3)
W_, E_, S_, N_, B_, T_ = range(6)


@pytest.mark.parametrize("n_local,pg,L,gm", [((128, 128, 128), (1, 1, 1), 3, 0), ((256, 128, 64), (1, 1, 1), 2, 0),
                                            ((128, 128, 128), (1, 1, 1), 2, 1), ((128, 128, 128), (2, 1, 1), 2, 0),
                                            ((512, 512, 512), (1, 1, 1), 2, 0)])
@pytest.mark.parametrize("tb", [3])
def test_pencil_plan_covers_owned_bricks(n_local, pg, L, gm, tb):
    """Every owned brick is swept exactly once per half by the pencil chunk streams; each record's
    16 ids are the tile layer's bricks and neighbours by the adjacency table; tiles sit on even
    brick coordinates (one coarse brick's x-y octants 0-3); runs are [warm-up, layers linked by T,
    cool-down] with the B / T neighbour layers; every CTA gets the same work to within a run."""
    p, lays = layouts(n_local, pg, L, gm, temporal_blocking=tb)
    lay = lays[0]
    inf = lay.info(0)
    adj, crd = lay.adjacency(0), lay.coords(0)
    par = lay.parent(0) if L > 1 else None
    allp = [pl for pl in lay.pass_plans(0) if pl[0] == tb]
    plans = [pl for pl in allp if pl[5] == 0]
    # the owned range (tiles on even owned coordinates: restriction), and with a ghost shell the
    # whole stored range (tiles on the extended box, ghost-sweeping passes)
    want = [(0, inf["owned"])] + ([(0, inf["owned"] + inf["nghost"])] if inf["nghost"] else [])
    assert [(pl[1], pl[2]) for pl in plans] == want
    for _, b0, b1, meta, ctas, _ in plans:
        owned = b1 == inf["owned"]
        g = np.array(inf["ghost"][:2]) * (0 if owned else 1)
        assert (_check_pencil_plan(meta, ctas, b1, adj, crd, par if owned else None, g) == 1).all()
        # with a ghost shell: the same units split into those that read no ghost brick (swept while
        # the exchange fills the ghosts) and the rest; together they cover every brick once per half
        parts = {pl[5]: pl for pl in allp if pl[5] and (pl[1], pl[2]) == (b0, b1)}
        assert sorted(parts) == ([1, 2] if inf["nghost"] else [])
        if parts:
            seen = sum(_check_pencil_plan(parts[k][3], parts[k][4], b1, adj, crd, par if owned else None, g)
                       for k in (1, 2))
            assert (seen == 1).all()
            ids = parts[1][3].reshape(-1, 20)[:, 1:17]
            assert not ((ids >= inf["owned"]) & (ids < inf["owned"] + inf["nghost"])).any()
            ids2 = parts[2][3].reshape(-1, 20)[:, 1:17]
            assert ((ids2 >= inf["owned"]) & (ids2 < inf["owned"] + inf["nghost"])).any()


def _check_pencil_plan(meta, ctas, nrange, adj, crd, par, g):
    # neighbours past the outermost ghosts are the zero brick (index = stored count), whose own
    # neighbours are the zero brick again
    adj = np.vstack([adj, np.full((1, 8), adj.shape[0], dtype=adj.dtype)])
    rec = meta.reshape(-1, 20)
    seen = np.zeros((nrange, 2), dtype=np.int64)
    work = []
    for first, count in ctas:
        chunks = rec[first:first + count]
        types = (chunks[:, 0] >> 1) & 3
        halves = chunks[:, 0] & 1
        w, m = 0, 0
        while m < count:
            assert types[m] == 1 and halves[m] == 1  # warm-up half 1
            e = m + 1
            while types[e] == 0:
                e += 1
            assert types[e] == 2 and halves[e] == 0  # cool-down half 0
            rng = chunks[m + 1:e]
            assert len(rng) % 2 == 0 and (halves[m + 1:e] == np.tile([0, 1], len(rng) // 2)).all()
            layers = rng[::2, 1]
            assert chunks[m, 1] == adj[layers[0], B_] and chunks[e, 1] == adj[layers[-1], T_]
            assert all(adj[a, T_] == b for a, b in zip(layers[:-1], layers[1:]))
            w += 4 * len(layers) + 1
            m = e + 1
        work.append(w)
        for r in chunks:
            b00, b10, b01, b11, W0, W1, E0, E1, S0, S1, N0, N1, SW, NW, SE, NE, pa = r[1:18]
            assert (b10, b01, b11) == (adj[b00, E_], adj[b00, N_], adj[b10, N_]) and adj[b01, E_] == b11
            assert (W0, W1, E0, E1) == (adj[b00, W_], adj[b01, W_], adj[b10, E_], adj[b11, E_])
            assert (S0, S1, N0, N1) == (adj[b00, S_], adj[b10, S_], adj[b01, N_], adj[b11, N_])
            assert (SW, NW, SE, NE) == (adj[W0, S_], adj[W1, N_], adj[E0, S_], adj[E1, N_])
            if (r[0] >> 1) & 3 == 0:
                assert (crd[b00, 0] + g[0]) % 2 == 0 and (crd[b00, 1] + g[1]) % 2 == 0
                for k, b in enumerate((b00, b10, b01, b11)):
                    seen[b, r[0] & 1] += 1
                    if par is not None:
                        assert pa % 4 == 0 and par[b] == pa + k
    ideal = sum(work) / len(work)
    assert max(work) <= ideal * 1.15 + 8
    return seen


def test_variant_combinations_rejected():
    """bc != periodic with GSRB / the CG bottom, var_coef with a smoother variant, the CG bottom or the
    paper's kernel set, and out-of-range codes are refused at parameter validation (no GPU needed)."""
    bad = [dict(bc=1, smoother=2), dict(bc=2, bottom_solver=1), dict(bc=3), dict(var_coef=1, smoother=1),
           dict(var_coef=1, bottom_solver=1), dict(var_coef=1, fusion=1), dict(var_coef=2)]
    for kw in bad:
        p = mg.params((32, 32, 32), num_levels=2, **kw)
        with pytest.raises(mg.MGError):
            mg.mg_workspace_bytes(p, 0, 1)
    for kw in (dict(bc=1), dict(bc=2, smoother=1), dict(var_coef=1, bc=1)):
        assert mg.mg_workspace_bytes(mg.params((32, 32, 32), num_levels=2, **kw), 0, 1) > 0


def test_var_coef_workspace_holds_a_coefficient_field():
    """var_coef adds one field (n_alloc bricks) per level; bc adds the ghost shell on every axis."""
    base = mg.mg_workspace_bytes(mg.params((32, 32, 32), num_levels=2, sweep_kernel=1, temporal_blocking=0,
                                           bottom_mode=1), 0, 1)
    vc = mg.mg_workspace_bytes(mg.params((32, 32, 32), num_levels=2, var_coef=1), 0, 1)
    lay = mg.Layout(mg.params((32, 32, 32), num_levels=2), 0, 1)
    field_bytes = sum(lay.info(l)["alloc"] * 512 * 8 for l in range(2))
    assert field_bytes <= vc - base <= field_bytes + 4096 * 2


@pytest.mark.parametrize("n_local,pg,L,bc", BC_CASES)
def test_workspace_is_rank_independent(n_local, pg, L, bc):
    """Every rank carves the same workspace layout (the loopback group and the peer transport address
    other ranks' objects at their own offsets), also when a non-periodic bc drops the runs across
    domain faces, which differ from rank to rank."""
    world = pg[0] * pg[1] * pg[2]
    for vc in (0, 1):
        p = mg.params(n_local, pg, num_levels=L, bc=bc, var_coef=vc)
        sizes = {mg.mg_workspace_bytes(p, r, world) for r in range(world)}
        assert len(sizes) == 1, sizes


B4_CASES = [((16, 16, 16), (1, 1, 1), 3, 0, 0), ((16, 16, 16), (1, 1, 1), 2, 1, 0), ((8, 16, 8), (2, 1, 1), 2, 0, 0),
            ((8, 8, 8), (2, 2, 2), 2, 0, 1), ((8, 8, 16), (1, 2, 3), 2, 0, 2), ((16, 8, 8), (2, 1, 1), 2, 0, 1)]


@pytest.mark.parametrize("n_local,pg,L,gm,bc", B4_CASES)
def test_brick4_layout_and_interpreter_bitwise_vs_oracle(oracle_mod, n_local, pg, L, gm, bc):
    """4^3 bricks (brick_edge = 4, P:L154 Sunspot): the same layout machinery with a
    4-cell brick -- adjacency consistent with the coords, every ghost brick filled exactly once --
    and the host brick interpreter on those tables reproduces the oracle's V-cycle bit for bit
    (periodic, self-exchanged ghost shells, decompositions, Dirichlet / Neumann)."""
    p, lays = layouts(n_local, pg, L, gm, brick_edge=4, bc=bc)
    for lay in lays:
        for l in range(L):
            inf = lay.info(l)
            assert inf["nb"] == [n >> l >> 2 for n in n_local]
            adj, co = lay.adjacency(l), lay.coords(l)
            index = {tuple(c): q for q, c in enumerate(co)}
            for q in range(inf["owned"]):
                for f, d in enumerate(FACE):
                    e = [int(co[q][a]) + d[a] for a in range(3)]
                    for a in range(3):
                        if not inf["ghost"][a]:
                            e[a] %= inf["nb"][a]
                    assert adj[q, f] == index[tuple(e)]
            got = np.zeros(inf["owned"] + inf["nghost"], dtype=int)
            for peer, d, run, local, remote, count in lay.plan(l, 1):
                got[local:local + count] += 1
            for dst, src, mask in lay.mirror(l):
                got[dst] += 1
            assert np.all(got[inf["owned"]:] == 1)
    gshape = (n_local[2] * pg[2], n_local[1] * pg[1], n_local[0] * pg[0])
    b = mg_inputs.random_field(gshape, 19) if bc == 1 else mg_inputs.random_rhs(gshape, 19)
    pre, post, bottom = 3, 2, 15
    h0 = mg_inputs.default_h0(gshape)
    orc = oracle_mod.OracleMG(gshape, L, pre, post, bottom, h0, bc=bc)
    orc.set_b(b)
    orc.set_x(None)
    orc.vcycle()
    R = len(lays)
    ranks = [[bi.RankLevel(lays[r], l) for l in range(L)] for r in range(R)]
    assert ranks[0][0].E == 4
    xs = [[ranks[r][l].zeros() for l in range(L)] for r in range(R)]
    bs = [[None] * L for _ in range(R)]
    for r in range(R):
        bs[r][0] = ranks[r][0].to_bricks(mg_inputs.local_block(b, r, pg))
    b0 = bi.exchange_local([bs[r][0] for r in range(R)], [ranks[r][0] for r in range(R)])
    for r in range(R):
        bs[r][0] = b0[r]
    xs = bi.vcycle_ranks(xs, bs, ranks, L, h0, pre, post, bottom)
    got = np.zeros(gshape)
    for r in range(R):
        cx, cy, cz = mg_inputs.rank_coords(r, pg)
        nx, ny, nz = n_local
        got[cz * nz:(cz + 1) * nz, cy * ny:(cy + 1) * ny, cx * nx:(cx + 1) * nx] = ranks[r][0].from_bricks(xs[r][0])
    assert np.array_equal(got, orc.get_x())


def test_brick4_params():
    """brick_edge 4: n_local a multiple of 4*2^(L-1), ca_period <= 4, no CG bottom; 5 is refused."""
    ok = mg.params((12, 8, 4), num_levels=1, brick_edge=4)
    assert mg.mg_workspace_bytes(ok, 0, 1) > 0
    for p in (mg.params((12, 8, 4), num_levels=2, brick_edge=4), mg.params((16, 16, 16), num_levels=2, brick_edge=5),
              mg.params((16, 16, 16), num_levels=2, brick_edge=4, ca_period=5),
              mg.params((16, 16, 16), num_levels=2, brick_edge=4, bottom_solver=1)):
        with pytest.raises(mg.MGError):
            mg.mg_workspace_bytes(p, 0, 1)


@pytest.mark.parametrize("n,L", [(64, 3), (128, 4)])
@pytest.mark.parametrize("transport", [mg.MG_TRANSPORT_LOCAL, mg.MG_TRANSPORT_PEER, mg.MG_TRANSPORT_NCCL])
@pytest.mark.parametrize("period", [0, 1, 3, 8])
def test_depth_limited_exchange_bytes(n, L, transport, period):
    """Bytes one x-exchange sends (the schedule's own plan, host-only): with a ghost shell on every axis a
    copy transport (local, peer) moves exactly the ghost cells within the CA period d of the owned box,
    ((n + 2 d)^3 - n^3) * 8 B (faces d planes, edges d x d columns, corners d^3), NCCL the whole one-brick
    shell ((n + 16)^3 - n^3) * 8 B; the auto period is 2 at level 0 and 8 below."""
    p = mg.params((n, n, n), num_levels=L, ghost_mode=1, transport=transport,
                  ca_period=period if period else None)
    lay = mg.Layout(p, 0, 1)
    exchanges, nbytes = lay.exchange_plan()
    for l in range(L):
        nl = n >> l
        if l == L - 1:  # the replicated bottom gathers the coarsest level: no ghost exchange of x
            assert exchanges[l] == 0
            continue
        d = period if period else (2 if l == 0 else 8)
        if transport == mg.MG_TRANSPORT_NCCL:
            d = 8
        assert nbytes[l] == ((nl + 2 * d) ** 3 - nl ** 3) * 8, (l, d)
        assert exchanges[l] > 0
    # two-sweep pencil passes at level 0 (128^3): one exchange of two cell layers before each of the 12
    # passes at the auto period 2
    if n == 128 and transport != mg.MG_TRANSPORT_NCCL and period == 0:
        assert exchanges[0] == 12


@pytest.mark.parametrize("pg", [(2, 1, 1), (2, 2, 1), (2, 2, 2), (1, 2, 3)])
def test_depth_limited_exchange_bytes_decomposed(pg):
    """Every rank of a decomposition sends, per x-exchange, exactly the cells the peers' ghost regions
    within the CA period d need: the ghost shell of the decomposed axes only, ((n + 2 d_a) product) - n^3
    with d_a = d on decomposed axes and 0 on the wrapped ones (level 0 at the auto period 2 on the
    peer transport; level 1 whole bricks, d = 8)."""
    n = 64
    p = mg.params((n, n, n), pg, num_levels=3, transport=mg.MG_TRANSPORT_PEER)
    world = pg[0] * pg[1] * pg[2]
    for r in range(world):
        lay = mg.Layout(p, r, world)
        _, nbytes = lay.exchange_plan()
        for l, d in ((0, 2), (1, 8)):
            nl = n >> l
            ext = np.prod([nl + (2 * d if g > 1 else 0) for g in pg])
            assert nbytes[l] == (ext - nl ** 3) * 8, (r, l)


@pytest.mark.parametrize("transport", [mg.MG_TRANSPORT_PEER, mg.MG_TRANSPORT_LOCAL, mg.MG_TRANSPORT_NCCL])
def test_fused_levels_take_period_two(transport):
    """Levels whose x exchanges fuse into their pencil passes (a pencil plan over the
    owned range -- >= 4096 bricks --, a periodic box, constant coefficients, a copy transport) take the CA
    period 2 like level 0: at 256^3 with a ghost shell on every axis level 1 (128^3, 4096 bricks) exchanges
    two cell layers before each of its 11 x-passes (+ b's after the restriction), level 2 (64^3, 512
    bricks, one-brick kernels) keeps whole bricks at period 8; NCCL keeps whole bricks everywhere."""
    n, L = 256, 4
    p = mg.params((n, n, n), num_levels=L, ghost_mode=1, transport=transport)
    exchanges, nbytes = mg.Layout(p, 0, 1).exchange_plan()
    fused = os.environ.get("MG_NO_FUSED_EXCH") is None and transport != mg.MG_TRANSPORT_NCCL
    for l, d in ((0, 2), (1, 2 if fused else 8), (2, 8)):
        if transport == mg.MG_TRANSPORT_NCCL:
            d = 8
        nl = n >> l
        assert nbytes[l] == ((nl + 2 * d) ** 3 - nl ** 3) * 8, (l, d, nbytes)
    if fused:
        assert exchanges[1] == 12, exchanges


@pytest.mark.parametrize("pg", [(2, 1, 1), (2, 2, 1), (2, 2, 2)])
def test_fused_exchange_source_table(pg):
    """The fused exchange's source table (mg_layout_fused_pid: what a level-0 pencil pass stages its ghost
    bricks' x from) checked against the geometry alone: every record entry naming an owned brick stays
    local (-1); every ghost brick at extended coords X is read from the rank that owns the periodic image
    of X in the process grid, at the brick of that rank's own layout with coords X mod nb -- never from the
    receive runs the table was built from.  128^3 per rank (level 0: 4096 bricks, pencil plan)."""
    n = 128
    world = pg[0] * pg[1] * pg[2]
    p = mg.params((n, n, n), pg, num_levels=3, transport=mg.MG_TRANSPORT_PEER)
    lays = [mg.Layout(p, r, world) for r in range(world)]
    owned_ids = []
    for lay in lays:
        inf = lay.info(0)
        c = lay.coords(0)[: inf["owned"]]
        owned_ids.append({tuple(v): i for i, v in enumerate(c.tolist())})
    nb = np.array(lays[0].info(0)["nb"])
    for r, lay in enumerate(lays):
        inf = lay.info(0)
        pid = lay.fused_pid(0)
        assert pid is not None
        plan = [t for t in lay.pass_plans(0) if t[0] == 3 and t[1] == 0 and t[2] == inf["owned"] and t[5] == 0]
        assert len(plan) == 1
        meta = plan[0][3].reshape(-1, 20)
        assert meta.shape[0] == pid.shape[0]
        coords = lay.coords(0)
        rc = np.array([r % pg[0], (r // pg[0]) % pg[1], r // (pg[0] * pg[1])])
        remote = 0
        for ch in range(meta.shape[0]):
            for e in range(16):
                bid = meta[ch, 1 + e]
                if bid < inf["owned"]:
                    assert pid[ch, e] == -1, (r, ch, e)
                    continue
                X = coords[bid]
                off = np.floor_divide(X, nb)
                oc = (rc + off) % np.array(pg)
                owner = int(oc[0] + pg[0] * (oc[1] + pg[1] * oc[2]))
                rid = owned_ids[owner][tuple(int(v) for v in np.mod(X, nb))]
                assert pid[ch, e] == (owner << 24) | rid, (r, ch, e, X.tolist(), owner, rid, pid[ch, e])
                remote += 1
        assert remote > 0
