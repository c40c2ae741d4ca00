// layout.cpp -- brick grids, adjacency, region ordering and exchange plans.
//
// Implements the data layout the paper's method rests on:
//  * bricks: 8^3 blocks stored contiguously; an adjacency table replaces ijk
//    indexing ("the brick data layout provides indirection from ijk stencil
//    grids"; bricks P:L17, L59, L154);
//  * communication avoiding: the ghost zone is one brick deep (8 cells), so
//    several smooths run per exchange, with 26 neighbours;
//  * packing/unpacking-free exchange: owned bricks are physically ordered by
//    surface region, so each neighbour's data is a few contiguous brick runs
//    sent straight from the field, and ghost bricks are stored in arrival
//    order ("optimal brick layout", "packing- and unpacking-free
//    communication buffers").  The order of the 26 surface regions below was
//    found by tools/region_order_search.py: 42 runs for 26 neighbours.
#include <cstdlib>
#include <algorithm>
#include <array>
#include <cstdio>
#include <tuple>

#include "mg_internal.h"

namespace mgb {

// Surface regions s in {-1,0,1}^3 \ 0 in physical storage order (after the
// interior region).  Found offline (tools/region_order_search.py).
static const int kRegionOrder[26][3] = {
    {0, 1, 0},   {0, 1, -1},  {1, 1, -1},  {1, 1, 0},   {1, 1, 1},   {0, 1, 1},  {-1, 1, 1},
    {-1, 1, 0},  {-1, 1, -1}, {-1, 0, -1}, {-1, -1, -1}, {0, -1, -1}, {0, 0, -1}, {1, 0, -1},
    {1, -1, -1}, {1, -1, 0},  {1, 0, 0},   {-1, 0, 0},  {-1, 0, 1},  {0, 0, 1},  {1, 0, 1},
    {1, -1, 1},  {0, -1, 1},  {-1, -1, 1}, {-1, -1, 0}, {0, -1, 0}};

int neighbour_rank(const Layout& lay, int dx, int dy, int dz) {
  const int* P = lay.p.proc_grid;
  const int cx = (lay.coords[0] + dx + P[0]) % P[0];
  const int cy = (lay.coords[1] + dy + P[1]) % P[1];
  const int cz = (lay.coords[2] + dz + P[2]) % P[2];
  return cx + P[0] * (cy + P[1] * cz);
}

// true if rank coords + (dx,dy,dz) leaves the global domain on an axis (non-periodic bc only)
bool crosses_boundary(const Layout& lay, int dx, int dy, int dz) {
  if (lay.p.bc == MG_BC_PERIODIC) return false;
  const int d[3] = {dx, dy, dz};
  for (int a = 0; a < 3; ++a) {
    const int c = lay.coords[a] + d[a];
    if (c < 0 || c >= lay.p.proc_grid[a]) return true;
  }
  return false;
}

int64_t LevelLayout::ext_index(int x, int y, int z) const {
  const int ex = nb[0] + 2 * g[0], ey = nb[1] + 2 * g[1];
  const int ez = nb[2] + 2 * g[2];
  const int X = x + g[0], Y = y + g[1], Z = z + g[2];
  if (X < 0 || Y < 0 || Z < 0 || X >= ex || Y >= ey || Z >= ez) return -1;
  return ext2idx[(size_t)X + (size_t)ex * ((size_t)Y + (size_t)ey * Z)];
}

// Region code per axis: 0 mid, 1 low, 2 high, 3 both (one brick on that axis).
static int axis_code(int c, int nb, int g) {
  if (!g) return 0;
  const bool lo = c == 0, hi = c == nb - 1;
  return (lo && hi) ? 3 : lo ? 1 : hi ? 2 : 0;
}

static int region_rank(int cx, int cy, int cz) {
  if (cx == 0 && cy == 0 && cz == 0) return 0;
  if (cx == 3 || cy == 3 || cz == 3) return 100 + cx + 4 * cy + 16 * cz;
  auto s = [](int c) { return c == 0 ? 0 : (c == 1 ? -1 : 1); };
  const int sx = s(cx), sy = s(cy), sz = s(cz);
  for (int r = 0; r < 26; ++r)
    if (kRegionOrder[r][0] == sx && kRegionOrder[r][1] == sy && kRegionOrder[r][2] == sz) return 1 + r;
  return 99;  // unreachable
}

static void build_level(const Layout& lay, int l, LevelLayout& L) {
  const mg_params& p = lay.p;
  for (int a = 0; a < 3; ++a) {
    L.n[a] = p.n_local[a] >> l;
    L.nb[a] = L.n[a] / lay.E;
    // a one-brick ghost shell on decomposed axes, on every axis in MG_GHOST_ALL, and on every axis
    // with a non-periodic boundary (its domain-face ghosts hold the reflected values, reading A22)
    L.g[a] = (p.ghost_mode == MG_GHOST_ALL || p.proc_grid[a] > 1 || p.bc != MG_BC_PERIODIC) ? 1 : 0;
  }
  const int nbx = L.nb[0], nby = L.nb[1], nbz = L.nb[2];
  const int ex = nbx + 2 * L.g[0], ey = nby + 2 * L.g[1], ez = nbz + 2 * L.g[2];
  L.ext2idx.assign((size_t)ex * ey * ez, -1);

  // ---- owned bricks, region-ordered ----
  struct Key {
    int rr, z, y, x;
  };
  std::vector<Key> owned;
  owned.reserve((size_t)nbx * nby * nbz);
  for (int z = 0; z < nbz; ++z)
    for (int y = 0; y < nby; ++y)
      for (int x = 0; x < nbx; ++x) {
        const int rr = region_rank(axis_code(x, nbx, L.g[0]), axis_code(y, nby, L.g[1]), axis_code(z, nbz, L.g[2]));
        owned.push_back({rr, z, y, x});
      }
  std::stable_sort(owned.begin(), owned.end(), [](const Key& a, const Key& b) {
    return std::tie(a.rr, a.z, a.y, a.x) < std::tie(b.rr, b.z, b.y, b.x);
  });
  L.n_owned = (int64_t)owned.size();
  L.n_interior = 0;
  L.coord.clear();
  for (size_t i = 0; i < owned.size(); ++i) {
    const Key& k = owned[i];
    if (k.rr == 0) ++L.n_interior;
    L.coord.push_back(k.x);
    L.coord.push_back(k.y);
    L.coord.push_back(k.z);
    L.ext2idx[(size_t)(k.x + L.g[0]) + (size_t)ex * ((size_t)(k.y + L.g[1]) + (size_t)ey * (k.z + L.g[2]))] =
        (int32_t)i;
  }
  auto own_idx = [&](int x, int y, int z) -> int64_t { return L.ext_index(x, y, z); };

  // ---- ghost bricks, by receiver direction, in the sender's storage order ----
  L.sends.clear();
  L.recvs.clear();
  L.n_recv_slots = 0;
  int64_t next = L.n_owned;
  for (int d = 0; d < 27; ++d) {
    int dx, dy, dz;
    dir_from_index(d, dx, dy, dz);
    if (dx == 0 && dy == 0 && dz == 0) continue;
    const int dd[3] = {dx, dy, dz};
    bool ok = true;
    for (int a = 0; a < 3; ++a)
      if (dd[a] != 0 && !L.g[a]) ok = false;
    if (!ok) continue;
    // sender-side brick set: c_a = nb-1 if d_a=-1, 0 if d_a=+1, all if 0
    int lo[3], hi[3];
    for (int a = 0; a < 3; ++a) {
      if (dd[a] == -1) {
        lo[a] = L.nb[a] - 1;
        hi[a] = L.nb[a];
      } else if (dd[a] == 1) {
        lo[a] = 0;
        hi[a] = 1;
      } else {
        lo[a] = 0;
        hi[a] = L.nb[a];
      }
    }
    std::vector<std::pair<int64_t, std::array<int, 3>>> set;  // (sender own idx, sender coords)
    for (int z = lo[2]; z < hi[2]; ++z)
      for (int y = lo[1]; y < hi[1]; ++y)
        for (int x = lo[0]; x < hi[0]; ++x) set.push_back({own_idx(x, y, z), {x, y, z}});
    std::sort(set.begin(), set.end());
    const int recv_peer = neighbour_rank(lay, dx, dy, dz);     // my ghost d comes from me+d
    const int send_peer = neighbour_rank(lay, -dx, -dy, -dz);  // my bricks go to me-d (its ghost d)
    // non-periodic boundary (reading A22): nothing crosses a domain face -- ghosts beyond it are
    // filled by the mirror table below, and a rank on the face sends nothing across it
    const bool recv_cross = crosses_boundary(lay, dx, dy, dz), send_cross = crosses_boundary(lay, -dx, -dy, -dz);
    const int64_t gstart = next;
    int run = 0;
    for (size_t m = 0; m < set.size();) {
      size_t e = m + 1;
      while (e < set.size() && set[e].first == set[e - 1].first + 1) ++e;
      const int64_t cnt = (int64_t)(e - m);
      const int64_t goff = gstart + (int64_t)m;
      ++L.n_recv_slots;  // (counted with the dropped ones: the workspace carve must not depend on the rank)
      if (!recv_cross) L.recvs.push_back({recv_peer, d, run, goff, set[m].first, cnt});
      if (!send_cross) L.sends.push_back({send_peer, d, run, set[m].first, goff, cnt});
      ++run;
      m = e;
    }
    // ghost bricks: extended coords of receiver ghost region d
    for (size_t m = 0; m < set.size(); ++m) {
      const auto& c = set[m].second;
      int e3[3];
      for (int a = 0; a < 3; ++a) e3[a] = dd[a] == -1 ? -1 : dd[a] == 1 ? L.nb[a] : c[a];
      L.coord.push_back(e3[0]);
      L.coord.push_back(e3[1]);
      L.coord.push_back(e3[2]);
      L.ext2idx[(size_t)(e3[0] + L.g[0]) + (size_t)ex * ((size_t)(e3[1] + L.g[1]) + (size_t)ey * (e3[2] + L.g[2]))] =
          (int32_t)(gstart + (int64_t)m);
    }
    next += (int64_t)set.size();
  }
  L.n_stored = next;
  L.n_ghost = next - L.n_owned;
  // mirror table (reading A22, method of images): a ghost brick beyond a domain face is the owned (or
  // received) brick reflected across every domain face it lies beyond, cells reversed on those axes,
  // times -1 per reflection (Dirichlet) or +1 (Neumann); filled after the receives of an exchange
  L.mirror.clear();
  if (p.bc != MG_BC_PERIODIC) {
    for (int64_t b = L.n_owned; b < L.n_stored; ++b) {
      const int* e = &L.coord[(size_t)b * 3];
      int q[3], mask = 0;
      for (int a = 0; a < 3; ++a) {
        q[a] = e[a];
        if (e[a] < 0 && lay.coords[a] == 0) q[a] = 0, mask |= 1 << a;
        if (e[a] >= L.nb[a] && lay.coords[a] == p.proc_grid[a] - 1) q[a] = L.nb[a] - 1, mask |= 1 << a;
      }
      if (!mask) continue;
      const int64_t src = L.ext_index(q[0], q[1], q[2]);
      L.mirror.push_back((int32_t)b);
      L.mirror.push_back((int32_t)src);
      L.mirror.push_back(mask);
    }
  }
  L.zero_brick = next;
  L.n_alloc = next + 1;
  // NCCL matches sends/recvs between a pair in posting order: sort both by (peer, dir, run)
  auto cmp = [](const Run& a, const Run& b) { return std::tie(a.peer, a.dir, a.run) < std::tie(b.peer, b.dir, b.run); };
  std::sort(L.sends.begin(), L.sends.end(), cmp);
  std::sort(L.recvs.begin(), L.recvs.end(), cmp);

  // ---- adjacency: W,E,S,N,B,T,self,0 ----
  L.adj.assign((size_t)L.n_stored * 8, 0);
  static const int F[6][3] = {{-1, 0, 0}, {1, 0, 0}, {0, -1, 0}, {0, 1, 0}, {0, 0, -1}, {0, 0, 1}};
  for (int64_t b = 0; b < L.n_stored; ++b) {
    const int* e = &L.coord[(size_t)b * 3];
    for (int f = 0; f < 6; ++f) {
      int q[3];
      bool zero = false;
      for (int a = 0; a < 3; ++a) {
        q[a] = e[a] + F[f][a];
        if (!L.g[a]) {
          q[a] = (q[a] % L.nb[a] + L.nb[a]) % L.nb[a];
        } else if (q[a] < -1 || q[a] > L.nb[a]) {
          zero = true;
        }
      }
      int64_t idx = zero ? -1 : L.ext_index(q[0], q[1], q[2]);
      L.adj[(size_t)b * 8 + f] = (int32_t)(idx < 0 ? L.zero_brick : idx);
    }
    L.adj[(size_t)b * 8 + 6] = (int32_t)b;
    L.adj[(size_t)b * 8 + 7] = 0;
  }
  // one-CTA resident bottom under a non-periodic bc: when every ghost of the level is a reflection
  // (one rank), the owned bricks' adjacency with each domain face marked -1 (the face cell's image
  // is the cell itself, resident.cuh); empty when a ghost comes from another rank
  L.radj.clear();
  if (p.bc != MG_BC_PERIODIC && lay.world == 1 && L.recvs.empty()) {
    std::vector<int32_t> src((size_t)L.n_ghost, -1), msk((size_t)L.n_ghost, 0);
    for (size_t e = 0; e + 2 < L.mirror.size(); e += 3) {
      src[(size_t)(L.mirror[e] - L.n_owned)] = L.mirror[e + 1];
      msk[(size_t)(L.mirror[e] - L.n_owned)] = L.mirror[e + 2];
    }
    L.radj.assign((size_t)L.n_owned * 8, 0);
    bool ok = true;
    for (int64_t b = 0; b < L.n_owned && ok; ++b) {
      for (int f = 0; f < 6; ++f) {
        const int32_t nb = L.adj[(size_t)b * 8 + f];
        if (nb < L.n_owned) {
          L.radj[(size_t)b * 8 + f] = nb;
        } else {
          const int64_t g = nb - L.n_owned;
          ok = g < L.n_ghost && src[(size_t)g] == b && msk[(size_t)g] == (1 << (f >> 1));
          L.radj[(size_t)b * 8 + f] = -1;
        }
      }
      L.radj[(size_t)b * 8 + 6] = (int32_t)b;
    }
    if (!ok) L.radj.clear();
  }
}

static void build_parents(LevelLayout& F, const LevelLayout& C) {
  F.parent.assign((size_t)F.n_alloc, -1);  // zero brick has no parent
  for (int64_t b = 0; b < F.n_stored; ++b) {
    const int* e = &F.coord[(size_t)b * 3];
    int E[3], o[3];
    for (int a = 0; a < 3; ++a) {
      E[a] = (e[a] >= 0) ? e[a] / 2 : -1;  // floor(e/2) for e >= -1
      o[a] = e[a] - 2 * E[a];
    }
    const int64_t ci = C.ext_index(E[0], E[1], E[2]);
    if (ci >= 0) F.parent[(size_t)b] = (int32_t)(ci * 8 + o[0] + 2 * o[1] + 4 * o[2]);
  }
}

// smallest level with two-sweep passes under the auto kernel choice (MG_PAIR_MIN_BRICKS: A/B runs only)
static int64_t pair_min_bricks() {
  static const int64_t v = getenv("MG_PAIR_MIN_BRICKS") ? atoll(getenv("MG_PAIR_MIN_BRICKS")) : kPairMinBricks;
  return v;
}

mg_status build_layout(const mg_params& p, int rank, int world, Layout& out, std::string& msg) {
  char buf[256];
  if (world < 1 || rank < 0 || rank >= world) {
    msg = "rank/world_size out of range";
    return MG_ERR_INVALID_ARG;
  }
  if (p.proc_grid[0] < 1 || p.proc_grid[1] < 1 || p.proc_grid[2] < 1 ||
      (int64_t)p.proc_grid[0] * p.proc_grid[1] * p.proc_grid[2] != world) {
    snprintf(buf, sizeof buf, "proc_grid %dx%dx%d does not match world_size %d", p.proc_grid[0], p.proc_grid[1],
             p.proc_grid[2], world);
    msg = buf;
    return MG_ERR_INVALID_ARG;
  }
  if (p.num_levels < 1 || p.num_levels > MG_MAX_LEVELS) {
    msg = "num_levels must be in [1, 16]";
    return MG_ERR_INVALID_ARG;
  }
  if (p.brick_edge != 0 && p.brick_edge != 4 && p.brick_edge != 8) {
    msg = "brick_edge must be 0 / 8 (8^3 bricks) or 4 (4^3 bricks)";
    return MG_ERR_INVALID_ARG;
  }
  const int E = p.brick_edge == 4 ? 4 : kB;
  out.E = E;
  out.BV = (int64_t)E * E * E;
  const int64_t unit = (int64_t)E << (p.num_levels - 1);
  for (int a = 0; a < 3; ++a) {
    if (p.n_local[a] <= 0 || p.n_local[a] % unit != 0) {
      snprintf(buf, sizeof buf, "n_local[%d]=%d must be a positive multiple of %d*2^(num_levels-1)=%lld", a,
               p.n_local[a], E, (long long)unit);
      msg = buf;
      return MG_ERR_INVALID_ARG;
    }
  }
  if (p.pre_smooths < 0 || p.post_smooths < 0 || p.bottom_smooths < 0) {
    msg = "sweep counts must be >= 0";
    return MG_ERR_INVALID_ARG;
  }
  for (int l = 0; l < MG_MAX_LEVELS; ++l) {
    if (p.ca_period[l] < 0 || p.ca_period[l] > E) {
      msg = "ca_period must be in [0, brick edge] (ghost depth = brick edge, P:L156)";
      return MG_ERR_INVALID_ARG;
    }
    if (p.fusion[l] < 0 || p.fusion[l] > MG_FUSION_FULL) {
      msg = "fusion must be in [0, 3]";
      return MG_ERR_INVALID_ARG;
    }
  }
  if (p.bc < MG_BC_PERIODIC || p.bc > MG_BC_NEUMANN) {
    msg = "bc must be 0 (periodic), 1 (Dirichlet) or 2 (Neumann)";
    return MG_ERR_INVALID_ARG;
  }
  if (p.bc != MG_BC_PERIODIC && (p.smoother == 2 || p.bottom_solver == 1)) {
    msg = "a non-periodic bc needs smoother 0/1 and bottom_solver 0 (reading A22)";
    return MG_ERR_INVALID_ARG;
  }
  if (p.temporal_blocking != 0 && p.temporal_blocking != 1 && p.temporal_blocking != 3) {
    msg = "temporal_blocking must be 0 (one sweep per pass), 1 (one-brick two-sweep streams) or 3 (2x2-brick "
          "pencils, the default)";
    return MG_ERR_INVALID_ARG;
  }
  if (p.ghost_mode != MG_GHOST_AUTO && p.ghost_mode != MG_GHOST_ALL) {
    msg = "ghost_mode must be 0 or 1";
    return MG_ERR_INVALID_ARG;
  }
  out.p = p;
  out.rank = rank;
  out.world = world;
  out.coords[0] = rank % p.proc_grid[0];
  out.coords[1] = (rank / p.proc_grid[0]) % p.proc_grid[1];
  out.coords[2] = rank / (p.proc_grid[0] * p.proc_grid[1]);
  out.L = p.num_levels;
  out.lv.assign(out.L, LevelLayout());
  for (int l = 0; l < out.L; ++l) build_level(out, l, out.lv[l]);
  const int64_t min_b = p.sweep_kernel == 1 ? INT64_MAX : p.sweep_kernel == 2 ? 0 : kColMinBricks;
  for (int l = 0; l < out.L; ++l) build_col_tables(out.lv[l], min_b);
  for (int l = 0; l + 1 < out.L; ++l) build_parents(out.lv[l], out.lv[l + 1]);
  if (p.temporal_blocking != 0)
    for (int l = 0; l < out.L; ++l)
      build_pair_tables(out.lv[l], p.sweep_kernel == 0 ? pair_min_bricks() : min_b,
                        p.temporal_blocking == 3 ? 3 : 1);
  // replicated bottom: the global coarsest level as one rank would store it
  const LevelLayout& B = out.lv[(size_t)out.L - 1];
  out.repl = false;
  if (out.L >= 2 && B.n_ghost > 0 && p.bottom_smooths > 0 && p.bottom_mode != MG_BOTTOM_SWEEPS &&
      p.bc == MG_BC_PERIODIC) {
    Layout g;
    g.p = p;
    g.E = out.E;
    g.BV = out.BV;
    for (int a = 0; a < 3; ++a) {
      g.p.n_local[a] = p.n_local[a] * p.proc_grid[a];
      g.p.proc_grid[a] = 1;
    }
    g.p.ghost_mode = MG_GHOST_AUTO;
    g.L = out.L;
    LevelLayout G;
    build_level(g, out.L - 1, G);
    if (G.n_owned <= kReplMaxBricks) {
      out.gb = std::move(G);
      const int nbx = B.nb[0], nby = B.nb[1], nbz = B.nb[2];
      out.gb_src.assign((size_t)out.gb.n_owned, -1);
      for (int64_t q = 0; q < out.gb.n_owned; ++q) {
        const int X = out.gb.coord[(size_t)q * 3], Y = out.gb.coord[(size_t)q * 3 + 1], Z = out.gb.coord[(size_t)q * 3 + 2];
        const int r = X / nbx + p.proc_grid[0] * (Y / nby + p.proc_grid[1] * (Z / nbz));
        out.gb_src[(size_t)q] = (int32_t)(r * B.n_owned + B.ext_index(X % nbx, Y % nby, Z % nbz));
      }
      out.gb_mine.assign((size_t)B.n_owned, -1);
      for (int64_t i = 0; i < B.n_owned; ++i)
        out.gb_mine[(size_t)i] = (int32_t)out.gb.ext_index(B.coord[(size_t)i * 3] + out.coords[0] * nbx,
                                                           B.coord[(size_t)i * 3 + 1] + out.coords[1] * nby,
                                                           B.coord[(size_t)i * 3 + 2] + out.coords[2] * nbz);
      out.repl = true;
    }
  }
  if (p.bottom_solver == 1) {  // CG bottom (reading A21): one CTA holds the whole coarsest grid
    const int64_t nb = out.repl ? out.gb.n_owned : (B.n_ghost > 0 ? -1 : B.n_owned);
    if (nb < 0 || nb > 8) {
      msg = "bottom_solver = 1 (CG) needs a coarsest grid of <= 8 bricks (globally when decomposed), "
            "without bottom_mode = sweeps on a ghost-shell level";
      return MG_ERR_INVALID_ARG;
    }
  }
  return MG_OK;
}

}  // namespace mgb

namespace mgb {

// Column plans for the streaming sweep (kernels.cu sweep_col_kernel): every
// brick of [b0,b1) exactly once, as z-chains following the adjacency T link
// (periodic columns are cycles; ghost-shell columns end at the zero brick),
// each chain cut into near-equal segments of <= kColSeg bricks.
// The bricks of [b0,b1) as z-chains along the T link, each brick exactly once,
// chains in order of their first brick's storage index.
static std::vector<std::vector<int32_t>> z_chains(const LevelLayout& L, int64_t b0, int64_t b1) {
  std::vector<std::vector<int32_t>> out;
  std::vector<char> vis((size_t)(b1 - b0), 0);
  auto in = [&](int64_t q) { return q >= b0 && q < b1; };
  for (int64_t q = b0; q < b1; ++q) {
    if (vis[(size_t)(q - b0)]) continue;
    int64_t s = q;
    for (;;) {
      const int64_t pb = L.adj[(size_t)s * 8 + 4];
      if (!in(pb) || vis[(size_t)(pb - b0)] || pb == q) break;
      s = pb;
    }
    std::vector<int32_t> chain;
    for (int64_t c = s; in(c) && !vis[(size_t)(c - b0)]; c = L.adj[(size_t)c * 8 + 5]) {
      vis[(size_t)(c - b0)] = 1;
      chain.push_back((int32_t)c);
    }
    out.push_back(std::move(chain));
  }
  return out;
}

static LevelLayout::ColTable col_table(const LevelLayout& L, int64_t b0, int64_t b1) {
  LevelLayout::ColTable t;
  t.b0 = b0;
  t.b1 = b1;
  for (const auto& chain : z_chains(L, b0, b1)) {
    const int64_t len = (int64_t)chain.size();
    const int64_t nseg = (len + kColSeg - 1) / kColSeg;
    int64_t off = 0;
    for (int64_t g = 0; g < nseg; ++g) {
      const int64_t cnt = len / nseg + (g < len % nseg ? 1 : 0);
      t.segs.push_back((int32_t)t.bricks.size());
      t.segs.push_back((int32_t)cnt);
      for (int64_t m = 0; m < cnt; ++m) {
        const int32_t id = chain[(size_t)(off + m)];
        t.bricks.push_back(id);
        for (int f = 0; f < 4; ++f) t.side.push_back(L.adj[(size_t)id * 8 + f]);
      }
      off += cnt;
    }
  }
  return t;
}

void build_col_tables(LevelLayout& L, int64_t min_bricks) {
  L.cols.clear();
  if (L.n_stored < min_bricks) return;
  const int64_t ranges[5][2] = {{0, L.n_owned},
                                {0, L.n_stored},
                                {0, L.n_interior},
                                {L.n_interior, L.n_owned},
                                {L.n_interior, L.n_stored}};
  for (auto& r : ranges) {
    if (r[1] <= r[0]) continue;
    bool dup = false;
    for (auto& c : L.cols) dup |= (c.b0 == r[0] && c.b1 == r[1]);
    if (!dup) L.cols.push_back(col_table(L, r[0], r[1]));
  }
}

// Item streams for the two-sweep kernel (sweep2.cu), one per resident CTA
// (G = kPairCtas).  Whole z-chains are dealt round-robin -- CTA g takes chains
// g, g+G, g+2G, ... -- so the CTAs running at any moment work on neighbouring
// columns at about the same height and their side-face reads hit L2.  The
// chains of the last, incomplete round are concatenated and cut into G equal
// pieces, so every CTA gets the same number of bricks.  Each run of bricks of
// one chain becomes [warm-up, run..., cool-down], warm-up / cool-down being the
// B / T neighbours of the run's ends: the kernel computes the first sweep on
// them too (their x1 planes 7 / 0 are k-halos of the run's second sweep).
static LevelLayout::PairTable pair_table(const LevelLayout& L, int64_t b0, int64_t b1) {
  LevelLayout::PairTable t;
  t.b0 = b0;
  t.b1 = b1;
  const auto chains = z_chains(L, b0, b1);
  const int64_t nch = (int64_t)chains.size();
  int64_t nb = 0;
  for (const auto& c : chains) nb += (int64_t)c.size();
  const int64_t G = std::max<int64_t>(1, std::min<int64_t>(kPairCtas, nb / 8));
  auto adj = [&](int64_t id, int f) -> int32_t {
    return id >= L.n_stored ? (int32_t)L.zero_brick : L.adj[(size_t)id * 8 + f];
  };
  std::vector<std::vector<int32_t>> stream((size_t)G);  // per CTA: its item metadata
  auto push_item = [&](std::vector<int32_t>& v, int32_t id, int32_t flags) {
    const int32_t W = adj(id, 0), E = adj(id, 1), S = adj(id, 2), N = adj(id, 3);
    const int32_t par = (id < L.n_stored && !L.parent.empty()) ? L.parent[(size_t)id] : -1;
    const int32_t m[kPairMeta] = {id, flags, W, E, S, N, adj(W, 2), adj(W, 3), adj(E, 2), adj(E, 3), par};
    v.insert(v.end(), m, m + kPairMeta);
  };
  auto push_run = [&](std::vector<int32_t>& v, const int32_t* run, int64_t len) {
    push_item(v, adj(run[0], 4), 2);  // warm-up (only its plane 7 of x1 is needed)
    for (int64_t q = 0; q < len; ++q) push_item(v, run[q], q > 0 ? 1 : 0);
    push_item(v, adj(run[len - 1], 5), 1 | 4);  // cool-down (only its plane 0 of x1 is needed)
  };
  const int64_t full = (nch / G) * G;  // chains dealt round-robin
  for (int64_t c = 0; c < full; ++c) push_run(stream[(size_t)(c % G)], chains[(size_t)c].data(), chains[(size_t)c].size());
  std::vector<int32_t> rest, rest_chain;
  for (int64_t c = full; c < nch; ++c)
    for (int32_t id : chains[(size_t)c]) {
      rest.push_back(id);
      rest_chain.push_back((int32_t)c);
    }
  const int64_t nr = (int64_t)rest.size();
  int64_t off = 0;
  for (int64_t g = 0; g < G && nr > 0; ++g) {
    const int64_t cnt = nr / G + (g < nr % G ? 1 : 0);
    for (int64_t m = off; m < off + cnt;) {
      int64_t e = m + 1;
      while (e < off + cnt && rest_chain[(size_t)e] == rest_chain[(size_t)m]) ++e;
      push_run(stream[(size_t)g], &rest[(size_t)m], e - m);
      m = e;
    }
    off += cnt;
  }
  for (int64_t g = 0; g < G; ++g) {
    const auto& v = stream[(size_t)g];
    if (v.empty()) continue;
    t.ctas.push_back((int32_t)((int64_t)t.meta.size() / kPairMeta));
    t.ctas.push_back((int32_t)((int64_t)v.size() / kPairMeta));
    t.meta.insert(t.meta.end(), v.begin(), v.end());
  }
  return t;
}

// Chunk streams for the pencil two-sweep kernel (sweep2p.cu), one per resident CTA
// (G = kPenCtas).  Only for the owned range of a level whose x / y brick counts are even: the
// owned bricks are cut into 2x2-brick tiles aligned to even owned coordinates (so a tile layer
// is one coarse brick's x-y extent and the kernel's restriction writes whole coarse columns);
// a tile column (its z-chain of layers along T) plays the role of a brick chain in pair_table:
// runs of its layers are dealt round-robin (below).  A run of layers
// becomes chunks [warm-up layer half 1, (layer half 0, half 1)..., cool-down layer half 0], each
// a record of kPenRec ints (code, the tile layer's 16 brick ids, parent);
// warm-up / cool-down are the B / T neighbour layers (their x1 planes 7 / 0 are the k-halos of
// the run's second sweep).  Also for the whole stored range of a level with a ghost shell
// (two-sweep passes that sweep the ghosts redundantly, so one exchange serves several passes):
// there the tiles cover the extended box (owned + ghost layer), aligned to its origin, and no
// restriction runs.  Returns kind 0 if the range does not tile.
// part 1 / 2 (levels with a ghost shell): only the units whose records name no ghost brick /
// the others, so the first can run while an exchange fills the ghost bricks (part 1 on one CTA
// slot per SM fewer, which the exchange's kernels then find free).
// kind 3: G = kPenCtas (sweep2p.cu, two-warp CTAs).
static LevelLayout::PairTable pencil_table(const LevelLayout& L, int64_t b0, int64_t b1, int part = 0,
                                           int kind = 3) {
  LevelLayout::PairTable t;
  t.kind = 0;
  const bool owned = b0 == 0 && b1 == L.n_owned;
  const bool stored = b0 == 0 && b1 == L.n_stored && L.n_ghost > 0;
  if ((!owned && !stored) || L.n_owned <= 0) return t;
  const int gx = stored ? L.g[0] : 0, gy = stored ? L.g[1] : 0, gz = stored ? L.g[2] : 0;
  const int ex = L.nb[0] + 2 * gx, ey = L.nb[1] + 2 * gy;
  if ((ex & 1) || (ey & 1)) return t;
  auto adj = [&](int64_t id, int f) -> int32_t {
    return id >= L.n_stored ? (int32_t)L.zero_brick : L.adj[(size_t)id * 8 + f];
  };
  auto par = [&](int64_t id) -> int32_t {
    return (id < L.n_stored && !L.parent.empty()) ? L.parent[(size_t)id] : -1;
  };
  const int tx = ex / 2, ty = ey / 2, nz = L.nb[2] + 2 * gz;
  // items of every tile layer: [tile][z]
  std::vector<std::array<int32_t, kPenMeta>> layers((size_t)tx * ty * nz);
  auto make_item = [&](int32_t b00) -> std::array<int32_t, kPenMeta> {
    std::array<int32_t, kPenMeta> m{};
    const int32_t b10 = adj(b00, 1), b01 = adj(b00, 3), b11 = adj(b10, 3);
    const int32_t W0 = adj(b00, 0), W1 = adj(b01, 0), E0 = adj(b10, 1), E1 = adj(b11, 1);
    const int32_t S0 = adj(b00, 2), S1 = adj(b10, 2), N0 = adj(b01, 3), N1 = adj(b11, 3);
    const int32_t v[17] = {b00, b10, b01, b11, W0, W1, E0, E1, S0, S1, N0, N1,
                           adj(W0, 2), adj(W1, 3), adj(E0, 2), adj(E1, 3), par(b00)};
    for (int f = 0; f < 17; ++f) m[(size_t)f] = v[f];
    return m;
  };
  for (int py = 0; py < ty; ++py)
    for (int px = 0; px < tx; ++px)
      for (int z = 0; z < nz; ++z) {
        const int X = 2 * px - gx, Y = 2 * py - gy, Z = z - gz;
        const int64_t b00 = L.ext_index(X, Y, Z);
        if (b00 < 0 || b00 >= b1) return t;
        auto m = make_item((int32_t)b00);
        // the tile must be the 2x2 block of bricks at (X.., Y..) and (owned range, for the fused
        // restriction) one coarse brick's octants 0..3 (+4 for odd z)
        if (m[1] != L.ext_index(X + 1, Y, Z) || m[2] != L.ext_index(X, Y + 1, Z) ||
            m[3] != L.ext_index(X + 1, Y + 1, Z) || adj(m[2], 1) != m[3])
          return t;
        if (owned && m[16] >= 0)
          for (int k = 1; k < 4; ++k)
            if (par(m[(size_t)k]) != m[16] + k || (m[16] & 3) != 0) return t;
        layers[((size_t)py * tx + px) * nz + z] = m;
      }
  t.kind = kind;
  t.b0 = b0;
  t.b1 = b1;
  t.part = part;
  const int64_t ncol = (int64_t)tx * ty;
  static const int64_t gpen = getenv("MG_PEN_CTAS") ? atoll(getenv("MG_PEN_CTAS")) : kPenCtas;  // (experiments)
  const int64_t gmax = gpen;
  const int64_t per_sm = kPenCtasPerSm;
  const int64_t G = std::max<int64_t>(1, std::min<int64_t>(gmax, ncol * nz));
  std::vector<std::vector<int32_t>> stream((size_t)G);  // per CTA: its chunk records
  // one 20-int record per chunk: code (type << 1 | half), the 16 brick ids, parent of b00
  auto push_chunk = [&](std::vector<int32_t>& v, const std::array<int32_t, kPenMeta>& m, int type, int half) {
    v.push_back((type << 1) | half);
    v.insert(v.end(), m.begin(), m.begin() + 17);
    v.push_back(0);
    v.push_back(0);
  };
  // the B / T neighbour layer of a tile layer (warm-up / cool-down): every brick's B / T link
  auto shifted = [&](const std::array<int32_t, kPenMeta>& m, int f) {
    return make_item(adj(m[0], f));
  };
  auto push_run = [&](std::vector<int32_t>& v, int64_t col, int z0, int len) {
    const auto& first = layers[(size_t)col * nz + z0];
    const auto& last = layers[(size_t)col * nz + ((z0 + len - 1) % nz)];
    push_chunk(v, shifted(first, 4), 1, 1);  // warm-up: half 1
    for (int q = 0; q < len; ++q) {
      push_chunk(v, layers[(size_t)col * nz + ((z0 + q) % nz)], 0, 0);
      push_chunk(v, layers[(size_t)col * nz + ((z0 + q) % nz)], 0, 1);
    }
    push_chunk(v, shifted(last, 5), 2, 0);  // cool-down: half 0
  };
  // Units = (z-run, tile column): the column's layers cut into nzr near-equal runs.  Units are
  // ordered z-run-major, column-minor (x fastest) and dealt round-robin, so the CTAs working at
  // the same moment hold a compact band of columns at the same height: the side slabs they read
  // are their neighbours' own bricks, fetched from HBM by the neighbour at about the same time
  // (L2 hits).  nzr minimises the busiest CTA's work (the kernel is latency-bound, so a CTA's
  // speed does not depend on how many CTAs share its SM: every CTA must get the same work), in
  // quarter layers: a run of n layers costs 4n + 1 (its warm-up / cool-down steps).
  auto zr0 = [&](int nzr, int r) { return (int)((int64_t)r * nz / nzr); };
  int best = 1;
  int64_t best_cost = INT64_MAX;
  for (int nzr = 1; nzr <= nz; ++nzr) {
    std::vector<int64_t> cta((size_t)G, 0);
    for (int64_t u = 0; u < ncol * nzr; ++u) {
      const int r = (int)(u / ncol);
      cta[(size_t)(u % G)] += 4 * (zr0(nzr, r + 1) - zr0(nzr, r)) + 1;
    }
    const int64_t cost = *std::max_element(cta.begin(), cta.end());
    if (cost < best_cost) best_cost = cost, best = nzr;
  }
  // Second candidate (whole range only): runs of Lmax layers plus each column's remainder run, dealt
  // band by band (z-run-major, column-minor, as above) to the least-loaded CTA (ties: the lowest
  // index, so a band's long runs still land on consecutive CTAs).  When the columns' layers do not
  // split evenly over the CTAs (level 1 at 512^3: 256 columns of 32 layers on 888 CTAs), one long
  // run per CTA and the short remainders on the CTAs left over beat equal runs dealt round-robin
  // (busiest CTA 41 instead of 43 quarter layers).
  struct HRun {
    int64_t col;
    int z0, len;
  };
  std::vector<std::vector<HRun>> hybrid;
  // (only when it trims the busiest CTA by >= 2%: level 0's equal runs keep their exact banding)
  const int64_t equal_cost = best_cost;
  if (part == 0) {
    for (int lmax = 1; lmax < nz; ++lmax) {
      std::vector<HRun> runs;
      for (int z0 = 0; z0 < nz; z0 += lmax)
        for (int64_t col = 0; col < ncol; ++col) runs.push_back({col, z0, std::min(lmax, nz - z0)});
      std::vector<int64_t> load((size_t)G, 0);
      std::vector<std::vector<HRun>> deal((size_t)G);
      // least-loaded CTA, lowest index first (loads only grow: a simple scan stays O(runs x G) on
      // the host at setup; G <= 888)
      int64_t worst = 0;
      for (const HRun& r : runs) {
        size_t g = 0;
        for (size_t q = 1; q < (size_t)G; ++q)
          if (load[q] < load[g]) g = q;
        load[g] += 4 * r.len + 1;
        worst = std::max(worst, load[g]);
        deal[g].push_back(r);
        if (worst >= best_cost) break;
      }
      if (worst < best_cost && 50 * worst <= 49 * equal_cost) {
        best_cost = worst;
        hybrid = std::move(deal);
      }
    }
  }
  if (part == 0 && !hybrid.empty()) {
    for (int64_t g = 0; g < G; ++g)
      for (const HRun& r : hybrid[(size_t)g]) push_run(stream[(size_t)g], r.col, r.z0, r.len);
  } else if (part == 0) {
    for (int64_t u = 0; u < ncol * best; ++u) {
      const int r = (int)(u / ncol);
      const int64_t col = u % ncol;
      push_run(stream[(size_t)(u % G)], col, zr0(best, r), zr0(best, r + 1) - zr0(best, r));
    }
  } else {  // the units of one part, in the same order, dealt round-robin over Gp CTAs
    const int64_t Gp = std::max<int64_t>(1, part == 1 ? G - G / per_sm : G);
    int64_t k = 0;
    std::vector<int32_t> run;
    for (int64_t u = 0; u < ncol * best; ++u) {
      const int r = (int)(u / ncol);
      const int64_t col = u % ncol;
      run.clear();
      push_run(run, col, zr0(best, r), zr0(best, r + 1) - zr0(best, r));
      bool ghost = false;
      for (size_t e = 0; e < run.size(); e += kPenRec)
        for (int f = 1; f <= 16; ++f) {
          const int32_t id = run[e + (size_t)f];
          ghost |= id >= L.n_owned && id < L.n_stored;
        }
      if (ghost != (part == 2)) continue;
      auto& v = stream[(size_t)(k++ % Gp)];
      v.insert(v.end(), run.begin(), run.end());
    }
    if (k == 0) t.kind = 0;
  }
  for (int64_t g = 0; g < G; ++g) {
    const auto& v = stream[(size_t)g];
    if (v.empty()) continue;
    t.ctas.push_back((int32_t)(t.meta.size() / kPenRec));
    t.ctas.push_back((int32_t)(v.size() / kPenRec));
    t.meta.insert(t.meta.end(), v.begin(), v.end());
  }
  return t;
}

void build_pair_tables(LevelLayout& L, int64_t min_bricks, int kind) {
  L.pairs.clear();
  if (L.n_stored < min_bricks) return;
  // owned, interior / surface (overlap), and the same with the ghost shell (two-sweep passes
  // that also sweep the ghosts redundantly, so an exchange serves several passes)
  const int64_t ranges[5][2] = {{0, L.n_owned},
                                {0, L.n_interior},
                                {L.n_interior, L.n_owned},
                                {0, L.n_stored},
                                {L.n_interior, L.n_stored}};
  for (auto& r : ranges) {
    if (r[1] <= r[0]) continue;
    bool dup = false;
    for (auto& c : L.pairs) dup |= (c.b0 == r[0] && c.b1 == r[1]);
    if (dup) continue;
    LevelLayout::PairTable t;
    t.kind = 0;
    if (kind == 3) t = pencil_table(L, r[0], r[1], 0, kind);
    if (t.kind == 0) t = pair_table(L, r[0], r[1]);
    if (t.kind != 0) L.pairs.push_back(std::move(t));
  }
  // pencil passes over a level with a ghost shell: the units split by whether they read a ghost
  // brick, for the overlap of the exchange with the interior units (both parts or neither)
  if (kind == 3 && L.n_ghost > 0)
    for (const int64_t b1 : {L.n_owned, L.n_stored}) {
      bool have = false;
      for (const auto& c : L.pairs) have |= c.kind == kind && c.part == 0 && c.b0 == 0 && c.b1 == b1;
      if (!have) continue;
      LevelLayout::PairTable p1 = pencil_table(L, 0, b1, 1, kind), p2 = pencil_table(L, 0, b1, 2, kind);
      if (p1.kind != kind || p2.kind != kind) continue;
      L.pairs.push_back(std::move(p1));
      L.pairs.push_back(std::move(p2));
    }
}

}  // namespace mgb
