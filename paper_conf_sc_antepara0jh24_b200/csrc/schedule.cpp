// schedule.cpp -- compiles Alg 2 into device ops; see schedule.h.
#include "schedule.h"

#include <cstdlib>

#include <algorithm>

#include "kernels.h"

namespace mgb {

Builder::Builder(const Layout& l) : lay(l) {
  for (int i = 0; i < MG_MAX_LEVELS; ++i) fusion_override[i] = 0;
}

int Builder::fusion(int l) const {
  if (fusion_override[l]) return fusion_override[l];
  const int f = lay.p.fusion[l];
  return f ? f : MG_FUSION_FULL;
}

int Builder::period(int l) const {
  const int k = lay.p.ca_period[l];
  if (k) return k;
  // auto (measured, one B200, self-exchanged ghost shell on every axis, profiles/r02_exchange.md):
  // where an exchange is a device copy kernel (local copies on one GPU, peer memory between
  // processes) it copies only the ghost cells within the period of the owned region, so at level 0
  // a period of 2 -- an exchange of the two nearest cell layers before every two-sweep pass over the
  // owned bricks -- costs less than the redundant ghost-shell sweeping a longer period needs; the
  // coarser levels are better at 8 (fewer launches).  NCCL moves whole bricks: period 8.
  const bool box = lay.p.transport != MG_TRANSPORT_NCCL;
  if (box)
    if (const char* e = getenv("MG_CA_AUTO")) {  // (experiments) per-level auto periods "k0,k1,..."
      int k = 0, i = 0;
      for (const char* q = e; *q; ++q) {
        if (*q == ',') {
          if (i++ == l) break;
          k = 0;
        } else {
          k = 10 * k + (*q - '0');
        }
      }
      if (i == l && k > 0) return std::min(k, lay.E);
    }
  // a level whose exchanges fuse into its pencil passes (api.cu fill_fused_tables: no exchange kernel,
  // no redundant ghost sweeping) takes period 2 like level 0 (MG_FUSED_P8=1: period 8, A/B runs)
  static const bool p8 = getenv("MG_FUSED_P8") != nullptr;
  if (box && l > 0 && !p8 && fused_level(l)) return std::min(2, lay.E);
  return (l == 0 && box) ? std::min(2, lay.E) : lay.E;
}

bool fused_exchange_enabled() {
  static const bool off = getenv("MG_NO_FUSED_EXCH") != nullptr;
  return !off;
}

// the conditions under which the executor fuses this level's x exchanges into its pencil passes
// (api.cu make_plan / fill_fused_tables): copy transport, periodic box, constant coefficients, a
// pencil plan over the owned range, <= 8 ranks, no pencil overlap (any smoother: Jacobi, Chebyshev,
// red-black Gauss-Seidel half-sweep pairs)
bool Builder::fused_level(int l) const {
  const LevelLayout& L = lay.lv[l];
  static const bool pen_ov = getenv("MG_PENCIL_OVERLAP") && atoi(getenv("MG_PENCIL_OVERLAP")) != 0;
  return fused_exchange_enabled() && lay.p.transport != MG_TRANSPORT_NCCL && lay.p.bc == 0 && !lay.p.var_coef &&
         L.n_ghost > 0 && lay.world <= 8 && !(pen_ov && lay.p.overlap) &&
         fusion(l) != MG_FUSION_PAPER && lay.p.temporal_blocking && pencil_table(l);
}

int Builder::xdepth(int l) const {
  static const bool whole = getenv("MG_EXCH_WHOLE") && atoi(getenv("MG_EXCH_WHOLE"));  // (A/B runs)
  if (whole || lay.p.transport == MG_TRANSPORT_NCCL) return lay.E;
  return std::max(1, std::min(period(l), lay.E));
}

bool Builder::has_pair_table(int l, int64_t b0, int64_t b1) const {
  for (const auto& pt : lay.lv[l].pairs)
    if (pt.b0 == b0 && pt.b1 == b1 && pt.part == 0) return true;
  return false;
}

bool Builder::pencil_table(int l) const {
  for (const auto& pt : lay.lv[l].pairs)
    if (pt.b0 == 0 && pt.b1 == lay.lv[l].n_owned && pt.part == 0) return pt.kind == 3;
  return false;
}

bool Builder::pair_zero_ok(int l) const {
  for (const auto& pt : lay.lv[l].pairs)
    if (pt.b0 == 0 && pt.b1 == lay.lv[l].n_owned && pt.part == 0) return pt.kind == 3;
  return false;
}

bool Builder::pencil_ghosts(int l) const {
  const LevelLayout& L = lay.lv[l];
  if (L.n_ghost == 0) return false;
  for (const auto& pt : L.pairs)
    if (pt.b0 == 0 && pt.b1 == L.n_stored && pt.part == 0) return pt.kind == 3;
  return false;
}

bool Builder::pair_ok(int l) const {
  if (!lay.p.temporal_blocking || fusion(l) == MG_FUSION_PAPER) return false;
  const LevelLayout& L = lay.lv[l];
  if (!has_pair_table(l, 0, L.n_owned)) return false;
  if (ghosts(l)) {
    if (period(l) < 2) return false;  // a pair is two sweeps per exchange
    if (lay.p.overlap && L.n_interior > 0 &&
        !(has_pair_table(l, 0, L.n_interior) && has_pair_table(l, L.n_interior, L.n_owned)))
      return false;
  }
  return true;
}

bool Builder::pair_ghosts_ok(int l) const {
  const LevelLayout& L = lay.lv[l];
  if (!has_pair_table(l, 0, L.n_stored)) return false;
  if (pencil_table(l) && pencil_ghosts(l)) return true;  // pencil passes run unsplit
  return !(lay.p.overlap && L.n_interior > 0) || has_pair_table(l, L.n_interior, L.n_stored);
}

void Builder::phase(int l, int n, bool zero_first, int last, bool interp_first, int timer) {
  const double h = lay.p.h0 * (double)(1 << l);
  // pre / post sweeps take the smoother's steps; the bottom stays damped Jacobi.  The red-black
  // Gauss-Seidel variant (reading A20) turns each of the n sweeps into a red and a black
  // half-sweep with the Gauss-Seidel step h^2/6; every half-sweep counts as a sweep below.
  const bool gs = timer == MG_OP_SWEEP && lay.p.smoother == 2;
  const int nh = gs ? 2 * n : n;
  auto step = [&](int s) {
    if (gs) return (h * h) / 6.0;
    return timer == MG_OP_SWEEP ? sweep_gamma(lay.p, h, n, s) : (h * h) / 12.0;
  };
  auto colour = [&](int s) { return gs ? (s & 1) : -1; };
  const bool g = ghosts(l);
  const int k = period(l);
  const bool paper = fusion(l) == MG_FUSION_PAPER;
  const bool pairs = pair_ok(l);
  LevelState& S = st[l];
  // the one-warp pencil kernel folds initZero into its first sweep (x0 == 0): the first pair of a
  // coarse level's pre-smoothing needs no single sweep
  const bool zero_pair = pairs && pair_zero_ok(l);
  for (int s = 0; s < nh; ++s) {
    const bool single_only = (zero_first && s == 0 && !zero_pair) || (interp_first && s == 0);
    if (pairs && !single_only && s + 1 < nh) {
      // sweeps s and s+1 in one pass (temporal blocking); x1 never leaves the chip
      Op o;
      o.kind = OP_SWEEP2;
      o.level = l;
      o.timer = timer;
      o.g1 = step(s);
      o.g2 = step(s + 1);
      o.c1 = colour(s);
      o.c2 = colour(s + 1);
      o.zero = zero_first && s == 0;  // the first sweep reads x0 == 0 (SW_ZERO_X)
      const bool ex = g && !o.zero && (S.dx < 2 || S.since + 2 > k);
      if (ex) {
        S.dx = xdepth(l);
        S.since = 0;
      }
      o.exch_before = ex;
      // pencil passes exchange first and then sweep the whole range (they do not tile the surface
      // shell, so there is no interior / surface overlap split)
      o.nosplit = pencil_table(l);
      // ghost validity after two sweeps over the ghost shell too (x1 needs x0 one cell further
      // out and b at its own depth; x2 likewise from x1): min(d_x - 2, d_b - 1)
      const int d_inc = std::min(S.dx - 2, S.db - 1);
      const bool last_p = s + 1 == nh - 1;
      o.ghosts = g && !last_p && d_inc >= 1 && (S.since + 2) < k && pair_ghosts_ok(l);
      if (last_p && last == 1) o.flags |= SW_WRITE_R;
      if (last_p && last == 2) o.flags |= SW_RESTRICT;
      o.src = S.cur;
      o.dst = 1 - S.cur;
      S.cur = o.dst;
      S.dx = o.ghosts ? d_inc : 0;
      S.since += 2;
      ops.push_back(o);
      ++s;
      continue;
    }
    Op o;
    o.kind = OP_SWEEP;
    o.level = l;
    o.paper = paper;
    o.timer = timer;
    o.g1 = step(s);
    o.c1 = colour(s);
    const bool zero = zero_first && s == 0;
    const bool ex = g && !zero && (S.dx < 1 || S.since >= k);
    if (ex) {
      S.dx = xdepth(l);
      S.since = 0;
    }
    o.exch_before = ex;
    const int d_inc = zero ? S.db : std::min(S.dx - 1, S.db);
    const bool last_s = s == nh - 1;
    o.ghosts = g && !last_s && d_inc >= 1 && (S.since + 1) < k;
    if (zero) o.flags |= SW_ZERO_X;
    if (interp_first && s == 0) {
      o.flags |= SW_INTERP;
      o.cbuf = st[l + 1].cur;
    }
    if (last_s && last == 1) o.flags |= SW_WRITE_R;
    if (last_s && last == 2) o.flags |= SW_RESTRICT;
    o.src = S.cur;
    o.dst = paper ? S.cur : 1 - S.cur;
    S.cur = o.dst;
    S.dx = o.ghosts ? d_inc : 0;
    S.since += 1;
    ops.push_back(o);
  }
}

void Builder::exchange_b(int l) {
  if (!ghosts(l)) return;
  if (lay.repl && l == lay.L - 1) return;  // the replicated bottom gathers owned b only
  Op o;
  o.kind = OP_EXCH;
  o.level = l;
  o.field = 1;
  o.timer = MG_OP_EXCHANGE;
  ops.push_back(o);
  st[l].db = xdepth(l);
}

void Builder::restrict_op(int l) {
  Op o;
  o.kind = OP_RESTRICT;
  o.level = l;
  o.timer = MG_OP_RESTRICT;
  ops.push_back(o);
  exchange_b(l + 1);
}

void Builder::zero_op(int l) {
  Op o;
  o.kind = OP_ZERO;
  o.level = l;
  o.src = o.dst = st[l].cur;
  o.timer = MG_OP_ZERO;
  ops.push_back(o);
  st[l].dx = lay.E;  // zero is the true value of every ghost too
  st[l].since = 0;
}

void Builder::interp_op(int l) {
  Op o;
  o.kind = OP_INTERP;
  o.level = l;
  o.src = o.dst = st[l].cur;
  o.cbuf = st[l + 1].cur;
  o.timer = MG_OP_INTERP;
  ops.push_back(o);
  st[l].dx = 0;  // owned bricks only: ghosts stale until the next exchange
}

void Builder::bottom(int l, int n, bool zero) {
  if (n <= 0) return;
  if (lay.p.bottom_solver == 1 && !(lay.repl && l == lay.L - 1)) {  // CG bottom (reading A21), from x = 0
    Op o;
    o.kind = OP_BOTTOM_CG;
    o.level = l;
    o.src = st[l].cur;
    o.dst = 1 - st[l].cur;
    o.n = n;
    o.timer = MG_OP_BOTTOM;
    ops.push_back(o);
    st[l].cur = o.dst;
    st[l].dx = 0;
    return;
  }
  if (lay.repl && l == lay.L - 1 && (zero || lay.p.bottom_solver == 1) && fusion(l) != MG_FUSION_PAPER) {
    // replicated bottom
    Op o;
    o.kind = OP_BOTTOM_REPL;
    o.level = l;
    o.src = st[l].cur;
    o.dst = 1 - st[l].cur;
    o.n = n;
    o.timer = MG_OP_BOTTOM;
    ops.push_back(o);
    st[l].cur = o.dst;
    st[l].dx = 0;  // ghosts not filled: the interpolation reads owned coarse bricks only
    return;
  }
  const LevelLayout& L = lay.lv[l];
  const int bm = lay.p.bottom_mode;
  // (a one-rank non-periodic level: the owned bricks with the domain faces as images, L.radj)
  // (<= 8 bricks: one CTA, resident.cuh; <= 64: one cluster, bottom_cluster.cu)
  const int64_t max_res = cluster_bottom_enabled() ? kClusterBottomMaxBricks : kResidentMaxBricks;
  const bool can_res = (!ghosts(l) && L.n_stored <= max_res) || (!L.radj.empty() && L.n_owned <= max_res);
  const bool res = can_res && (bm == MG_BOTTOM_RESIDENT ||
                                ((bm == MG_BOTTOM_AUTO || bm == MG_BOTTOM_CLUSTER || bm == MG_BOTTOM_GRID) && fusion(l) != MG_FUSION_PAPER));
  const bool fold_zero = zero && fusion(l) == MG_FUSION_FULL;
  if (res) {
    Op o;
    o.kind = OP_BOTTOM_RES;
    o.level = l;
    o.src = st[l].cur;
    o.dst = 1 - st[l].cur;
    o.n = n;
    o.zero = fold_zero;
    o.timer = MG_OP_BOTTOM;
    st[l].cur = o.dst;
    st[l].dx = 0;
    ops.push_back(o);
    return;
  }
  phase(l, n, fold_zero, 0, false, MG_OP_BOTTOM);
}

int Builder::coarse_start() const {
  const int L = lay.L;
  const int bm = lay.p.bottom_mode;
  // opt-in: measured slower than graph-replayed per-level launches below 512^3
  if (L < 2 || (bm != MG_BOTTOM_CLUSTER && bm != MG_BOTTOM_GRID)) return -1;
  if (lay.p.bottom_solver != 0) return -1;  // their bottoms are Jacobi smooths
  if (lay.p.pre_smooths < 1) return -1;
  if (lay.p.smoother == 1 && (lay.p.pre_smooths > kCoarseMaxCheb || lay.p.post_smooths > kCoarseMaxCheb)) return -1;
  if (lay.p.smoother == 2) return -1;  // red-black half-sweeps: per-level kernels only
  if (bm == MG_BOTTOM_GRID) {  // grid-resident solve: the deepest ghost-free run of levels >= 1
    int l0 = L;                // with <= kGridCoarseMaxBricks bricks (fields stay in HBM / L2)
    static const int64_t maxb = getenv("MG_GRID_MAX_BRICKS") ? atoll(getenv("MG_GRID_MAX_BRICKS"))
                                                              : kGridCoarseMaxBricks;  // (experiments)
    while (l0 - 1 >= 1 && !ghosts(l0 - 1) && fusion(l0 - 1) != MG_FUSION_PAPER &&
           lay.lv[l0 - 1].n_owned <= maxb && L - (l0 - 1) <= kCoarseMaxLevels)
      --l0;
    if (l0 >= L || ghosts(L - 1) || fusion(L - 1) == MG_FUSION_PAPER) return -1;
    return l0;
  }
  // the deepest run of levels >= 1 without ghosts, paper kernel set excluded, whose first level
  // fits the cluster (<= 8 bricks per CTA) and whose fields fit its shared memory
  int l0 = L;
  while (l0 - 1 >= 1 && !ghosts(l0 - 1) && fusion(l0 - 1) != MG_FUSION_PAPER &&
         lay.lv[l0 - 1].n_owned <= 8 * kCoarseCtas && L - (l0 - 1) <= kCoarseMaxLevels)
    --l0;
  if (l0 >= L || ghosts(L - 1) || fusion(L - 1) == MG_FUSION_PAPER) return -1;
  CoarseArgs a{};
  a.nlev = L - l0;
  for (int l = l0; l < L; ++l) a.lv[l - l0].nb = (int)lay.lv[l].n_owned;
  while (a.nlev > 1 && coarse_smem_bytes(a) > kCoarseMaxSmem) {  // drop the largest level
    for (int i = 0; i + 1 < a.nlev; ++i) a.lv[i] = a.lv[i + 1];
    --a.nlev;
    ++l0;
  }
  if (coarse_smem_bytes(a) > kCoarseMaxSmem) return -1;
  return l0;
}

void Builder::vcycle() {
  const int L = lay.L;
  const mg_params& p = lay.p;
  const int lc = coarse_start();  // levels lc .. L-1 run in one cluster launch (-1: none)
  // Coarse x is dead at the start of a cycle (zeroed below): normalise its buffer.
  for (int l = 1; l < L; ++l) {
    st[l].cur = 0;
    st[l].dx = 0;
    st[l].db = 0;
    st[l].since = 1 << 20;
  }
  // level-0 ghosts of x are conservatively stale at the start of a cycle
  st[0].dx = 0;
  st[0].since = 1 << 20;
  if (L == 1) {
    bottom(0, p.bottom_smooths, false);
    return;
  }
  const int top = lc > 0 ? lc : L;  // levels handled one op at a time: 0 .. top-1
  for (int l = 0; l + 1 < top || (lc > 0 && l + 1 == top); ++l) {  // Alg 2 steps 1-8
    const bool full = fusion(l) == MG_FUSION_FULL;
    const bool zero_first = l > 0 && full;
    phase(l, p.pre_smooths, zero_first, full ? 2 : 1, false, MG_OP_SWEEP);
    if (full)
      exchange_b(l + 1);  // restriction fused into the last pre-sweep
    else
      restrict_op(l);
    if (l + 1 == lc) break;  // the cluster solve zeroes its own levels
    // the fold needs a first coarse sweep to absorb it (pre_smooths >= 1 is validated)
    const bool fold = fusion(l + 1) == MG_FUSION_FULL && (l + 2 < L || p.bottom_smooths > 0);
    if (!fold)  // initZero as its own kernel (Alg 2 step 8)
      zero_op(l + 1);
    else {
      st[l + 1].dx = lay.E;  // folded into the first coarse sweep
      st[l + 1].since = 0;
    }
  }
  if (lc > 0) {  // steps 1-23 of levels lc .. L-1 in one launch
    Op o;
    o.kind = OP_COARSE;
    o.level = lc;
    o.src = o.dst = 0;
    o.timer = MG_OP_BOTTOM;
    ops.push_back(o);
    st[lc].cur = 0;
    st[lc].dx = 0;
  } else {
    bottom(L - 1, p.bottom_smooths, true);  // steps 10-15
  }
  for (int l = top - (lc > 0 ? 1 : 2); l >= 0; --l) {  // steps 16-23
    // interpolation fused into the first post-sweep -- except where pencil passes run (their
    // kernel has no interpolation input): a separate interpolation then lets all post-sweeps pair
    // up (measured faster: one-brick interp-fused sweeps are the slowest single sweeps)
    const int nh = lay.p.smoother == 2 ? 2 * p.post_smooths : p.post_smooths;  // (half-)sweeps
    const bool pencil_pairs = pair_ok(l) && pencil_table(l) && nh % 2 == 0;
    const bool fuse_i = fusion(l) == MG_FUSION_FULL && !ghosts(l) && p.post_smooths > 0 && !pencil_pairs;
    if (!fuse_i) interp_op(l);
    phase(l, p.post_smooths, false, 0, fuse_i, MG_OP_SWEEP);
  }
}

int64_t op_launches(const Op& o, const Layout& lay, bool overlap, bool pencil_overlap, bool local_exchange) {
  // kernels of this library one op launches (NCCL's own kernels not counted); an exchange over the
  // local (or peer) transport is one copy kernel (copy_runs_kernel) when the level has receives, over
  // NCCL none of ours, plus the mirror kernel of a non-periodic bc
  const LevelLayout& L = lay.lv[o.level];
  const int64_t ex = (local_exchange && !L.recvs.empty() ? 1 : 0) + (L.mirror.empty() ? 0 : 1);
  switch (o.kind) {
    case OP_SWEEP:
    case OP_SWEEP2: {
      const int per = o.paper ? 2 : 1;  // applyOp + smooth(+residual)
      const int64_t end = o.ghosts ? L.n_stored : L.n_owned;
      const int64_t x = o.fused ? o.fused - 1 : o.exch_before ? ex : 0;
      bool pen_split = false;
      if (o.kind == OP_SWEEP2 && o.exch_before && overlap && pencil_overlap)
        for (const auto& pt : L.pairs) pen_split |= pt.b0 == 0 && pt.b1 == end && pt.part == 1;
      if (pen_split) return 2 + x;
      const bool split = o.exch_before && overlap && lay.lv[o.level].n_interior > 0 && !o.nosplit;
      return (split ? (o.paper ? 3 : 2) : per) + x;  // a split paper sweep: 2 applyOps, one smooth
    }
    case OP_RESTRICT:  // restrict_kernel
    case OP_INTERP:    // interp4_kernel / interp_kernel
    case OP_ZERO:      // zero_kernel
    case OP_BOTTOM_CG:  // bottom_cg_kernel
    case OP_BOTTOM_RES:  // bottom_resident_kernel
    case OP_COARSE:      // one cluster / grid launch
      return 1;
    case OP_BOTTOM_REPL:  // gather copies, the solve, the scatter copies (+ NCCL's all-gather)
      return 3;
    case OP_EXCH:
      return ex;
    default:
      return 0;
  }
}

}  // namespace mgb
