// schedule.h -- the V-cycle as a host-compiled list of device operations.
//
// Alg 2 is compiled once per starting state into a flat list of ops
// (sweeps, transfers, exchanges).  The builder applies the per-level fusion
// policy and the communication-avoiding ghost rule (DESIGN.md
// "Ghost-validity rule"): it tracks, per level, how many cells deep the ghost
// bricks of x and b are valid, inserts an x-exchange only when a sweep would
// read a stale ghost (or the CA period is reached), and sweeps ghost bricks
// redundantly only when the next sweep will read them without an exchange.
// Every schedule computes bit-identical values; only traffic changes.
#pragma once

#include <vector>

#include "mg_internal.h"

namespace mgb {

enum OpKind { OP_SWEEP = 0, OP_RESTRICT, OP_INTERP, OP_ZERO, OP_EXCH, OP_BOTTOM_RES, OP_SWEEP2, OP_COARSE,
              OP_BOTTOM_REPL, OP_BOTTOM_CG };
// OP_BOTTOM_CG: `n` CG iterations from x = 0 on the (ghost-free) coarsest level into buffer `dst`.
// OP_BOTTOM_REPL: the replicated bottom (Layout::repl): all-gather the owned b bricks of the
// coarsest level, `n` sweeps from x = 0 on the global coarsest grid, owned x into buffer `dst`.
// OP_COARSE: levels `level` .. L-1 of the cycle in one cluster launch (coarse.cu); x of `level`
// ends in buffer `dst`.
// OP_SWEEP2: two consecutive plain sweeps in one pass (sweep2.cu); `flags` are the
// second sweep's (r / restriction); owned bricks only; needs ghost depth >= 2.

struct Op {
  int kind = OP_SWEEP;
  int level = 0;
  int src = 0, dst = 0;     // x buffers (ping-pong) at `level`
  int cbuf = 0;             // coarse x buffer (interp)
  unsigned flags = 0;       // SW_* (kernels.h)
  bool paper = false;       // applyOp + smooth(+residual) kernels instead of the fused sweep
  bool ghosts = false;      // also sweep the ghost bricks (redundant CA computation)
  bool exch_before = false; // exchange x[src] ghosts before the sweep
  int field = 0;            // OP_EXCH: 0 = x[src], 1 = b
  int n = 0;                // OP_BOTTOM_RES: sweeps
  bool zero = false;        // OP_BOTTOM_RES: x == 0 on entry; OP_SWEEP2: the first sweep reads x0 == 0
  int timer = 0;            // MG_OP_*
  double g1 = 0, g2 = 0;    // smoothing steps of the (first, second) sweep; 0 = the level's Jacobi h^2/12
  int c1 = -1, c2 = -1;     // red-black colour of the (first, second) half-sweep (GSRB); -1 = every cell
  bool nosplit = false;     // exchange before the whole sweep (pencil passes: no interior / surface split)
  int fused = 0;            // OP_SWEEP2 with exch_before over the owned range: the exchange fused into the
                            // pencil pass (SW_PEER; set by the executor's plan): 1 no sync needed (one
                            // rank / a lockstep group), 2 after a peer handshake kernel (processes)
};

struct LevelState {
  int cur = 0;       // which x buffer holds x
  int dx = 0;        // valid ghost depth of x (cells)
  int db = 0;        // valid ghost depth of b (cells)
  int since = 1 << 20;  // sweeps since the last x exchange
};

struct Builder {
  const Layout& lay;
  std::vector<Op> ops;
  LevelState st[MG_MAX_LEVELS];
  int fusion_override[MG_MAX_LEVELS];

  explicit Builder(const Layout& l);
  bool ghosts(int l) const { return lay.lv[l].n_ghost > 0; }
  int fusion(int l) const;
  int period(int l) const;
  // cells of a ghost brick an exchange of level l refreshes, counted from the owned region: the
  // period (depth-limited copies, local and peer transports) or the whole brick (NCCL)
  int xdepth(int l) const;
  bool pair_ok(int l) const;  // two-sweep passes possible at level l
  bool pencil_table(int l) const;
  bool fused_level(int l) const;    // level l's x exchanges fuse into its pencil passes (period 2)  // the owned range of level l has a 2x2-brick pencil plan (kind 3)
  bool pencil_ghosts(int l) const;  // ... and so has its whole stored range (owned + ghost shell)
  bool pair_zero_ok(int l) const;   // the owned range's pencil kernel folds x0 == 0 into a pair (SW_ZERO_X)
  bool pair_ghosts_ok(int l) const;  // two-sweep passes may include the ghost shell at level l
  bool has_pair_table(int l, int64_t b0, int64_t b1) const;
  // `n` smooth(+residual) sweeps at level l.  last: 0 none, 1 write r, 2 fused restriction.
  void phase(int l, int n, bool zero_first, int last, bool interp_first, int timer);
  void restrict_op(int l);  // b_{l+1} = R r_l (+ b ghost exchange)
  void zero_op(int l);
  void interp_op(int l);
  void bottom(int l, int n, bool zero);
  void exchange_b(int l);
  int coarse_start() const;  // first level of the cluster-resident coarse solve, or -1
  void vcycle();
};

// own kernel launches of one op (local_exchange: exchanges run as one copy kernel, else NCCL)
bool fused_exchange_enabled();  // MG_NO_FUSED_EXCH=1: the separate exchange kernel everywhere (A/B)
int64_t op_launches(const Op& o, const Layout& lay, bool overlap, bool pencil_overlap, bool local_exchange);

}  // namespace mgb
