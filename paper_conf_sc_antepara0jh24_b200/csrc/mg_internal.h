// mg_internal.h -- host-side structures of the B200 brick-GMG library.
//
// Brick layout: every level's local subdomain is cut
// into 8^3 bricks, each stored contiguously (512 doubles, cell (i,j,k) of the
// brick at i + 8j + 64k, reading A16).  A brick table gives, per stored brick,
// its 6 face neighbours (adjacency), so kernels never compute ijk -> address.
//
// Storage order per level:  [interior owned | surface owned (26 regions in
// kRegionOrder) | ghost bricks (by direction, in the sender's order) | zero brick]
// Periodic axes that are not decomposed are closed by wrapping the adjacency;
// decomposed axes (or all axes in MG_GHOST_ALL) get a one-brick ghost shell
// (P:L156).
#pragma once

#include <cmath>

#include <cstdint>
#include <string>
#include <vector>

#include "../../include/mg.h"

namespace mgb {

constexpr int kB = MG_BRICK;          // brick edge
constexpr int kBV = kB * kB * kB;     // values per brick (512)

// One message of an exchange: contiguous bricks [local, local+count) on this
// rank are sent to / received from `peer`.  `remote` is the brick offset of
// the same run on the peer (known because every rank has the same layout).
struct Run {
  int32_t peer;
  int32_t dir;      // direction index 0..26 of the RECEIVER's ghost region (d+1 base 3)
  int32_t run;      // index of the run within (peer, dir)
  int64_t local;    // brick offset on this rank
  int64_t remote;   // brick offset on the peer
  int64_t count;    // bricks
};

struct LevelLayout {
  int n[3] = {0, 0, 0};    // cells per axis
  int nb[3] = {0, 0, 0};   // owned bricks per axis
  int g[3] = {0, 0, 0};    // ghost layer on axis (0 = periodic wrap inside the rank)
  int64_t n_owned = 0, n_interior = 0, n_ghost = 0, n_stored = 0, n_alloc = 0;
  int64_t zero_brick = 0;  // index of the all-zero brick (neighbour of the outermost ghosts)
  std::vector<int32_t> adj;     // [n_stored][8]
  std::vector<int32_t> coord;   // [n_stored][3] extended brick coords
  std::vector<int32_t> parent;  // [n_stored] coarse brick * 8 + octant, -1 if none
  std::vector<Run> sends, recvs;
  int64_t n_recv_slots = 0;     // receive runs before a non-periodic bc drops those across domain faces
  std::vector<int32_t> mirror;  // [n][3] ghost brick, source brick, reflected-axes mask (bc != periodic)
  std::vector<int32_t> radj;    // [n_owned][8] owned adjacency with domain faces = -1 (one-rank bc != periodic)
  int64_t ext_index(int x, int y, int z) const;  // -1 if not stored
  std::vector<int32_t> ext2idx;  // dense map over the extended box
  // Column plans for the streaming sweep kernel: the bricks of a range [b0,b1)
  // arranged as z-columns (chains along the adjacency T link) cut into
  // segments of <= kColSeg bricks; one CTA streams one segment.
  struct ColTable {
    int64_t b0 = 0, b1 = 0;
    std::vector<int32_t> bricks;  // brick ids, segment after segment
    std::vector<int32_t> side;    // [bricks][4] W,E,S,N neighbour ids
    std::vector<int32_t> segs;    // [nseg][2] offset into bricks, count
  };
  std::vector<ColTable> cols;     // one per distinct range the schedule sweeps
  // Item streams for the two-sweep (temporally blocked) kernel: the bricks of a
  // range as z-chains, cut into near-equal CTA pieces; each piece is preceded by
  // its warm-up brick (the B neighbour of its first brick) and followed by its
  // cool-down brick (T neighbour of its last): item = (id, flags, W,E,S,N,
  // SW,NW,SE,NE, parent), flags bit0 = "previous item is a range brick", bit1 = warm-up,
  // bit2 = cool-down (the kernel computes only the x1 planes the run needs from those).
  struct PairTable {
    int kind = 1;
    int64_t b0 = 0, b1 = 0;
    // kind 3 on a level with a ghost shell: 0 = every unit of the range; 1 = the units that read
    // no ghost brick (swept while the exchange fills the ghosts), 2 = the others (after it)
    int part = 0;
    std::vector<int32_t> meta;   // [items][kPairMeta] (kind 1) / [chunks][kPenRec] (kind 3)
    std::vector<int32_t> ctas;   // [nctas][2] offset (items / chunks), count
  };
  std::vector<PairTable> pairs;
};

// Step of sweep k of an s-sweep pre / post phase at spacing h (reading A19): damped
// Jacobi h^2/12, or the Chebyshev variant h^2/(12 nu_k) with nu_k the Chebyshev nodes of
// [1/rho, 1], small and large steps interleaved.  Written out from the reading alone; the
// same IEEE operations on the same host libm give the same bits.
inline double cheb_nu(int s, int k, int rho) {
  const int j = (k % 2 == 0) ? k / 2 : s - 1 - (k - 1) / 2;
  const double th = 0.5 * (1.0 + 1.0 / (double)rho), de = 0.5 * (1.0 - 1.0 / (double)rho);
  return th + de * std::cos(3.14159265358979323846 * (double)(2 * j + 1) / (double)(2 * s));
}
inline double sweep_gamma(const mg_params& p, double h, int s, int k) {
  return p.smoother == 1 ? (h * h) / (12.0 * cheb_nu(s, k, p.cheby_ratio)) : (h * h) / 12.0;
}

constexpr int kPairMeta = 11;
constexpr int kPairCtasPerSm = 4;                   // resident two-sweep CTAs per SM (shared-memory bound)
constexpr int64_t kPairCtas = 148 * kPairCtasPerSm;  // one item stream per resident two-sweep CTA
// kind 3 (sweep2p.cu): 2x2-brick pencils.  meta = one record per half-layer chunk: code (type << 1 |
// half; type 0 range, 1 warm-up, 2 cool-down), the tile layer's bricks b00, b10, b01, b11 (own, x then
// y), W0, W1 (W of b00, b01), E0, E1 (E of b10, b11), S0, S1 (S of b00, b10), N0, N1 (N of b01, b11),
// SW, NW, SE, NE (diagonal corners), parent of b00, 0, 0; ctas = (first record, record count).
constexpr int kPenMeta = 20;  // host-side tile-layer item: the 16 ids, parent, 0, 0, 0
constexpr int kPenRec = 20;   // chunk record (80 bytes: one 1D bulk copy)
constexpr int kPenCtasPerSm = 6;                    // resident pencil CTAs per SM (shared-memory bound)
constexpr int64_t kPenCtas = 148 * kPenCtasPerSm;
// kind 1: CTA item streams (sweep2.cu), kind 3: 2x2-brick
// pencil chunk streams (sweep2p.cu) for the owned range where the level tiles into aligned 2x2 pencils
// (other ranges, and levels that do not tile, get kind 1)
void build_pair_tables(LevelLayout& L, int64_t min_bricks, int kind);

constexpr int kColSeg = 16;             // bricks per streamed segment
constexpr int64_t kColMinBricks = 16384;  // levels smaller than this use the one-brick-per-CTA kernel
// two-sweep passes (auto kernel choice) from this level size on: at 512^3 levels 0-2 (level 2 =
// 128^3, 4096 bricks: pencil passes 0.29 vs 0.43 ms of single sweeps per cycle; pencil passes on
// levels 3-4 too (512 / 64 bricks) measured 0.16 vs 0.19 ms instrumented at level 3 but within the
// box noise in graph replay: 10.17-10.19 vs 10.12-10.22 ms)
constexpr int64_t kPairMinBricks = 4096;
void build_col_tables(LevelLayout& L, int64_t min_bricks);

// Replicated bottom: when the coarsest level has a ghost shell (decomposed, or self-exchange) and
// the global coarsest grid is small, every rank gathers the owned b bricks of all ranks and runs the
// bottom sweeps on the whole periodic coarsest grid itself -- the same per-cell expressions on the
// same values as the decomposed sweeps, without the ghost exchange every 8 sweeps (the
// bottom's communication dominates).
constexpr int64_t kReplMaxBricks = 64;  // global coarsest bricks (the cluster solve's capacity)

struct Layout {
  mg_params p{};
  int E = kB;     // brick edge (params brick_edge: 8, or 4 for the generic kernels)
  int64_t BV = kBV;  // doubles per brick
  int rank = 0, world = 1;
  int coords[3] = {0, 0, 0};
  int L = 0;
  std::vector<LevelLayout> lv;
  bool repl = false;             // replicated bottom in use
  LevelLayout gb;                // the global coarsest level (one rank: periodic wrap, no ghosts)
  std::vector<int32_t> gb_src;   // [gb.n_owned] source of each global brick: rank * n_owned + owned index
  std::vector<int32_t> gb_mine;  // [n_owned of the coarsest level] global index of each owned brick
};

// Validates params and builds every level.  Returns MG_OK or an error with msg.
mg_status build_layout(const mg_params& p, int rank, int world, Layout& out, std::string& msg);

// ---- neighbour helpers ----
inline int dir_index(int dx, int dy, int dz) { return (dx + 1) + 3 * (dy + 1) + 9 * (dz + 1); }
inline void dir_from_index(int d, int& dx, int& dy, int& dz) {
  dx = d % 3 - 1;
  dy = (d / 3) % 3 - 1;
  dz = d / 9 - 1;
}
int neighbour_rank(const Layout& lay, int dx, int dy, int dz);
bool crosses_boundary(const Layout& lay, int dx, int dy, int dz);

}  // namespace mgb
