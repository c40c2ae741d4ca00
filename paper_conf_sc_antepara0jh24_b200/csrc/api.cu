// api.cu -- C ABI (include/mg.h), device workspace, executor, exchange transport.
//
// Runtime structure:
//   mg_setup     validate -> host layout (layout.cpp) -> carve the caller's
//                workspace into per-level brick fields + tables -> upload tables
//                -> NCCL communicator (ncclCommInitRank from a torch-broadcast id)
//   mg_vcycle    Builder (schedule.cpp) compiles Alg 2 into ops once per starting
//                state; the op list is captured into ONE CUDA graph and replayed
//                (kernels + NCCL send/recv + event fork/join for overlap)
//   exchange     ghost bricks arrive as contiguous brick runs straight from the
//                peer's field (no packing): ncclSend/ncclRecv per run inside one
//                ncclGroup, or device copies for the in-process loopback group
//   norm         fused applyOp + |b - Ax| + block max + atomicMax on the uint64
//                bits (exact, order-free), ncclAllReduce(MAX) of 1 value
#include <cuda.h>
#include <cuda_runtime.h>
#include <cudaTypedefs.h>
#include <nccl.h>

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstring>
#include <string>
#include <vector>

#include "kernels.h"
#include "copyrun.cuh"
#include "mg_internal.h"
#include "schedule.h"

using namespace mgb;

namespace {
thread_local std::string g_err = "no error";

mg_status set_err(mg_status s, const std::string& m) {
  g_err = m;
  return s;
}

struct DevLevel {
  double* x[2] = {nullptr, nullptr};
  double* b = nullptr;
  double* r = nullptr;
  double* Ax = nullptr;
  double* cf = nullptr;  // variable coefficients (reading A23): cell coefficients c, ghosts exchanged once
  int32_t* adj = nullptr;
  int32_t* parent = nullptr;
  int32_t* coord = nullptr;
  int32_t* radj = nullptr;  // resident-bottom adjacency of a one-rank non-periodic level (LevelLayout::radj)
  Coeffs c{};
  double h = 0;
  struct Col {
    int64_t b0, b1;
    ColArgs args;
  };
  std::vector<Col> cols;  // streaming-sweep plans (column segments) per brick range
  FaceMaps fmaps[2];      // TMA face-halo tensor maps over x[0], x[1] (levels with column plans)
  FaceMaps cfmaps{};      // ... and over the coefficients (variable-coefficient variant)
  struct Pair {
    int64_t b0, b1;
    int part;  // LevelLayout::PairTable::part
    PairArgs args;
  };
  std::vector<Pair> pairs;  // two-sweep item streams per brick range
  PairMaps pmaps[2];        // tensor maps for the two-sweep kernel reading x[0] / x[1]
  PairMaps nmaps[2];        // the same with 4-plane boxes for the pencil kernel (sweep2p.cu)
  // local-transport exchange: [x[0] | x[1] | b][recv run] copy descriptors (device), one launch
  CopyRun* cruns = nullptr;
  int ncruns = 0;
  int64_t cmax = 0;
  // non-periodic bc (reading A22): domain-face ghost bricks <- reflected source bricks (int3 each)
  int32_t* mirror = nullptr;
  int nmirror = 0;
  double mirror_sign = 1.0;
  // the exchange fused into the level's pencil passes (SW_PEER): ghost brick -> (owner
  // rank, its brick id), [2 buffers][world] x base pointers and x tensor maps (xwe, xsn, xcor) of the owners
  bool fused = false;
  int32_t* pid = nullptr;  // [chunks of the owned pencil plan][16] (PairArgs::pid)
  CUtensorMap* rmaps = nullptr;
  std::vector<const double*> rbase;  // [2][rworld] (PairMaps::rbase)
  int rworld = 0;
};

struct Plan {
  std::vector<Op> ops;
  LevelState final_st[MG_MAX_LEVELS];
  int64_t launches = 0;
};

struct TimerRec {
  int slot;
  cudaEvent_t a, b;
};

size_t align256(size_t v) { return (v + 255) & ~(size_t)255; }
}  // namespace

struct mg_group;

struct mg_ctx {
  Layout lay;
  int device = 0;
  cudaStream_t stream = nullptr;
  cudaStream_t comm = nullptr;
  cudaStream_t cap = nullptr;  // private stream the V-cycle graph is captured on (the caller's may be legacy)
  cudaEvent_t ev_fork = nullptr, ev_join = nullptr;
  std::vector<DevLevel> dl;
  double* stage[2] = {nullptr, nullptr};  // host-upload staging fields
  int stage_k = 0;
  cudaStream_t h2d = nullptr;              // copy stream of host uploads
  cudaEvent_t ev_h2d[2] = {nullptr, nullptr}, ev_free[2] = {nullptr, nullptr};
  cudaEvent_t ev_norm = nullptr;           // completion of the last enqueued residual norm
  bool norm_pending = false;
  bool coef_ready = false;  // var_coef: mg_set_coefficients (+ the group commit) has run
  unsigned long long* acc = nullptr;
  double* h_pinned = nullptr;
  ncclComm_t nccl = nullptr;
  bool use_nccl = false;
  // peer-memory transport (MG_TRANSPORT_PEER, peer.cu): the other ranks' workspaces mapped by CUDA
  // IPC; exchanges, the norm's global max and the replicated bottom's gather are device-side
  bool use_peer = false, peer_ready = false;
  std::vector<char*> peer_ws;     // [world] every rank's workspace in this address space
  std::vector<void*> peer_open;   // IPC mappings to close
  PeerSync ps_nb{}, ps_all{};     // participants: the neighbour ranks / every other rank
  unsigned long long** d_remote_vals = nullptr;  // [world] the ranks' norm value slots (device array)
  struct PeerArea {
    unsigned long long* flags = nullptr;  // [world][2] slots of kPeerSlotU64
    unsigned long long* vals = nullptr;   // [world] norm values
    unsigned long long* epoch = nullptr;
    unsigned* done = nullptr;
    CopyRun* dummy = nullptr;
  } pa;
  mg_group* group = nullptr;
  int grank = 0;
  LevelState st[MG_MAX_LEVELS];
  bool poisoned = false;
  bool timing = false;
  bool use_col = true;  // streaming column kernel where a plan exists (sweep_kernel == 1 disables)
  // pencil passes on ghost-shell levels: the units that read no ghost brick overlap the exchange.
  // Default: only for exchanges with other processes (NCCL, world_size > 1); measured slower with a
  // local self-exchange (0.16 ms of copies per cycle do not pay for the split).
  // MG_PENCIL_OVERLAP=0/1 overrides (tests, measurements).
  bool pencil_overlap = false;
  // replicated bottom (Layout::repl): the global coarsest level's fields and the copy tables that
  // gather b into it and scatter this rank's owned x out of it
  struct Repl {
    double* x[2] = {nullptr, nullptr};
    double* b = nullptr;
    int32_t* adj = nullptr;
    int32_t* coord = nullptr;  // global brick coords (the CG bottom's lexicographic order)
    double* gbuf = nullptr;  // all-gather landing buffer [world][n_owned bricks] (NCCL)
    CopyRun* gather = nullptr;
    CopyRun* scatter = nullptr;  // [2][n_owned]: into x[0] / x[1] of the coarsest level
    bool allgather = false;
  } rp;
  std::vector<void*> allocs;  // library-owned device buffers allocated on first use (freed by mg_destroy)
  std::vector<double> tm;
  std::vector<TimerRec> trec;
  std::vector<std::pair<int, double>> recs;  // (level*MG_NUM_OPS + op, ms) per timed op, since mg_set_timing
  std::vector<cudaEvent_t> evpool;
  size_t evnext = 0;
  cudaGraphExec_t gexec[2] = {nullptr, nullptr};
  Plan gplan[2];
  bool gvalid[2] = {false, false};
  int64_t last_launches = 0;
};

struct mg_group {
  std::vector<mg_ctx*> r;
  cudaStream_t stream = nullptr;
  cudaStream_t cap = nullptr;
  cudaGraphExec_t gexec[2] = {nullptr, nullptr};
  Plan gplan[2];
  bool gvalid[2] = {false, false};
};

#define CKC(ctx, call)                                                                        \
  do {                                                                                        \
    cudaError_t e_ = (call);                                                                  \
    if (e_ != cudaSuccess) {                                                                  \
      if (ctx) (ctx)->poisoned = true;                                                        \
      return set_err(MG_ERR_CUDA, std::string(#call) + ": " + cudaGetErrorString(e_));        \
    }                                                                                         \
  } while (0)

#define CKN(ctx, call)                                                                        \
  do {                                                                                        \
    ncclResult_t e_ = (call);                                                                 \
    if (e_ != ncclSuccess) {                                                                  \
      if (ctx) (ctx)->poisoned = true;                                                        \
      return set_err(MG_ERR_NCCL, std::string(#call) + ": " + ncclGetErrorString(e_));        \
    }                                                                                         \
  } while (0)

#define CKS(expr)                  \
  do {                             \
    mg_status s_ = (expr);         \
    if (s_ != MG_OK) return s_;    \
  } while (0)

namespace {

// ------------------------------------------------------------- workspace
size_t carve(const Layout& lay, char* base, std::vector<DevLevel>* out, double** stage, unsigned long long** acc,
             mg_ctx::Repl* rp = nullptr, mg_ctx::PeerArea* pa = nullptr) {
  size_t off = 0;
  auto take = [&](size_t bytes) -> char* {
    const size_t o = align256(off);
    off = o + bytes;
    return base ? base + o : nullptr;
  };
  if (out) out->assign(lay.L, DevLevel());
  for (int l = 0; l < lay.L; ++l) {
    const LevelLayout& L = lay.lv[l];
    const size_t fb = (size_t)L.n_alloc * lay.BV * sizeof(double);
    DevLevel d;
    d.x[0] = (double*)take(fb);
    d.x[1] = (double*)take(fb);
    d.b = (double*)take(fb);
    d.r = (double*)take(fb);
    // Ax only for the paper's kernel set (MG_FUSION_PAPER: applyOp writes it, smooth+residual reads
    // it); a per-op call that asks for the paper set on another level allocates it lazily (ensure_ax)
    if (lay.p.fusion[l] == MG_FUSION_PAPER) d.Ax = (double*)take(fb);
    if (lay.p.var_coef) d.cf = (double*)take(fb);
    d.adj = (int32_t*)take((size_t)L.n_stored * 8 * sizeof(int32_t));
    d.parent = (int32_t*)take((size_t)L.n_alloc * sizeof(int32_t));
    d.coord = (int32_t*)take((size_t)L.n_stored * 3 * sizeof(int32_t));
    if (!L.radj.empty()) d.radj = (int32_t*)take(L.radj.size() * sizeof(int32_t));
    for (const auto& ct : L.cols) {
      DevLevel::Col col;
      col.b0 = ct.b0;
      col.b1 = ct.b1;
      col.args.bricks = (const int32_t*)take(ct.bricks.size() * sizeof(int32_t));
      col.args.side = (const int4*)take(ct.side.size() * sizeof(int32_t));
      col.args.segs = (const int2*)take(ct.segs.size() * sizeof(int32_t));
      col.args.nseg = (int64_t)ct.segs.size() / 2;
      d.cols.push_back(col);
    }
    for (const auto& pt : L.pairs) {
      DevLevel::Pair pr;
      pr.b0 = pt.b0;
      pr.b1 = pt.b1;
      pr.part = pt.part;
      pr.args.kind = pt.kind;
      pr.args.meta = (const int32_t*)take(pt.meta.size() * sizeof(int32_t));
      pr.args.ctas = (const int2*)take(pt.ctas.size() * sizeof(int32_t));
      pr.args.nctas = (int64_t)pt.ctas.size() / 2;
      d.pairs.push_back(pr);
    }
    // (sized rank-independently: every rank of a run carves the same layout -- the loopback group and the
    // peer transport address other ranks' objects at this rank's offsets)
    d.ncruns = (int)L.recvs.size();
    d.cruns = (CopyRun*)take((size_t)L.n_recv_slots * 4 * sizeof(CopyRun));
    d.nmirror = (int)(L.mirror.size() / 3);
    d.mirror = (int32_t*)take(lay.p.bc != MG_BC_PERIODIC ? (size_t)L.n_ghost * 3 * sizeof(int32_t) : 0);
    d.mirror_sign = lay.p.bc == MG_BC_DIRICHLET ? -1.0 : 1.0;
    d.h = lay.p.h0 * (double)(1 << l);
    d.c = level_coeffs(d.h);
    if (out) (*out)[l] = d;
  }
  // (the two host-upload staging fields are allocated on first use of the host-buffer calls,
  // ensure_stage: a device-only caller does not pay 2 level-0 fields for them)
  (void)stage;
  if (lay.repl) {  // replicated bottom
    const size_t gfb = (size_t)lay.gb.n_alloc * lay.BV * sizeof(double);
    const int64_t nown = lay.lv[(size_t)lay.L - 1].n_owned;
    mg_ctx::Repl r;
    r.x[0] = (double*)take(gfb);
    r.x[1] = (double*)take(gfb);
    r.b = (double*)take(gfb);
    r.adj = (int32_t*)take((size_t)lay.gb.n_stored * 8 * sizeof(int32_t));
    r.coord = (int32_t*)take((size_t)lay.gb.n_stored * 3 * sizeof(int32_t));
    r.gbuf = (double*)take((size_t)lay.world * nown * lay.BV * sizeof(double));
    r.gather = (CopyRun*)take((size_t)lay.gb.n_owned * sizeof(CopyRun));
    r.scatter = (CopyRun*)take((size_t)2 * nown * sizeof(CopyRun));
    if (rp) *rp = r;
  }
  {  // peer-transport sync area (every run carves it: a few KB; a one-rank peer self-exchange uses it too)
    unsigned long long* fl = (unsigned long long*)take((size_t)lay.world * 2 * kPeerSlotU64 * 8);
    unsigned long long* vals = (unsigned long long*)take((size_t)lay.world * 8);
    unsigned long long* ep = (unsigned long long*)take(64);
    unsigned* dn = (unsigned*)take(64);
    CopyRun* dm = (CopyRun*)take(sizeof(CopyRun));
    if (pa) pa->flags = fl, pa->vals = vals, pa->epoch = ep, pa->done = dn, pa->dummy = dm;
  }
  // norm accumulator (word 0) and the grid coarse solve's barrier words (from byte 64, kGridBarWords)
  unsigned long long* ac = (unsigned long long*)take(64 + kGridBarWords * sizeof(unsigned));
  if (acc) *acc = ac;
  return align256(off);
}

mg_params normalized(const mg_params* p) {
  mg_params q = *p;
  if (q.h0 <= 0) {
    int64_t m = 0;
    for (int a = 0; a < 3; ++a) {
      const int64_t n = (int64_t)q.n_local[a] * q.proc_grid[a];
      if (n > m) m = n;
    }
    q.h0 = m > 0 ? 1.0 / (double)m : 1.0;
  }
  if (q.cheby_ratio <= 0) q.cheby_ratio = 6;
  if (q.var_coef || q.brick_edge == 4) {  // A23 / 4^3 bricks: no pencil passes, per-sweep bottoms
    q.temporal_blocking = 0;
    q.bottom_mode = MG_BOTTOM_SWEEPS;
    // 4^3 bricks: the one-brick kernels of generic.cu only; variable coefficients: the TMA column
    // kernel's coefficient variant on the large levels, the one-brick kernel elsewhere
    if (q.brick_edge == 4) q.sweep_kernel = 1;
  }
  return q;
}

mg_status check_params(const mg_params& p) {
  if (p.num_levels > 1 && p.pre_smooths < 1)
    return set_err(MG_ERR_INVALID_ARG, "pre_smooths must be >= 1 when num_levels > 1 (restriction reads its r)");
  if (p.transport < 0 || p.transport > MG_TRANSPORT_PEER) return set_err(MG_ERR_INVALID_ARG, "bad transport");
  if (p.bottom_mode < 0 || p.bottom_mode > MG_BOTTOM_GRID) return set_err(MG_ERR_INVALID_ARG, "bad bottom_mode");
  if (p.launch_pdl < 0 || p.launch_pdl > 2) return set_err(MG_ERR_INVALID_ARG, "launch_pdl must be 0, 1 or 2");
  if (p.bottom_solver < 0 || p.bottom_solver > 1)
    return set_err(MG_ERR_INVALID_ARG, "bottom_solver must be 0 (Jacobi smooths) or 1 (CG)");
  if (p.smoother < 0 || p.smoother > 2)
    return set_err(MG_ERR_INVALID_ARG, "smoother must be 0 (Jacobi), 1 (Chebyshev) or 2 (red-black Gauss-Seidel)");
  if (p.var_coef < 0 || p.var_coef > 1) return set_err(MG_ERR_INVALID_ARG, "var_coef must be 0 or 1");
  if (p.brick_edge == 4 && p.bottom_solver != 0)
    return set_err(MG_ERR_INVALID_ARG, "4^3 bricks: the CG bottom kernel holds 8^3 bricks (bottom_solver must be 0)");
  if (p.var_coef) {
    if (p.smoother != 0 || p.bottom_solver != 0)
      return set_err(MG_ERR_INVALID_ARG, "var_coef needs smoother 0 and bottom_solver 0 (reading A23)");
    for (int l = 0; l < MG_MAX_LEVELS; ++l)
      if (p.fusion[l] == MG_FUSION_PAPER)
        return set_err(MG_ERR_INVALID_ARG, "var_coef: the paper's kernel set has no coefficient variant");
  }
  return MG_OK;
}

cudaEvent_t pool_event(mg_ctx* c) {
  if (c->evnext == c->evpool.size()) {
    cudaEvent_t e;
    cudaEventCreate(&e);
    c->evpool.push_back(e);
  }
  return c->evpool[c->evnext++];
}

// buffers allocated on first use (outside graph capture: callers run these before a plan executes)
mg_status ensure_ax(mg_ctx* c, int l) {
  DevLevel& d = c->dl[l];
  if (d.Ax) return MG_OK;
  void* p = nullptr;
  CKC(c, cudaMalloc(&p, (size_t)c->lay.lv[l].n_alloc * c->lay.BV * sizeof(double)));
  c->allocs.push_back(p);
  d.Ax = (double*)p;
  return MG_OK;
}

mg_status ensure_stage(mg_ctx* c) {
  if (c->stage[0]) return MG_OK;
  for (int k = 0; k < 2; ++k) {
    void* p = nullptr;
    CKC(c, cudaMalloc(&p, (size_t)c->lay.lv[0].n_owned * c->lay.BV * sizeof(double)));
    c->allocs.push_back(p);
    c->stage[k] = (double*)p;
  }
  return MG_OK;
}

// every buffer a plan's ops need exists (Ax of the levels that run the paper's kernel set)
mg_status prepare_plan(mg_ctx* c, mg_group* g, const std::vector<Op>& ops) {
  for (const Op& o : ops)
    if (o.paper) {
      if (g) {
        for (mg_ctx* r : g->r) CKS(ensure_ax(r, o.level));
      } else {
        CKS(ensure_ax(c, o.level));
      }
    }
  return MG_OK;
}

// ------------------------------------------------------------- exchange
// field 0: x[xbuf], 1: b, 2: the coefficients (variable-coefficient variant)
double* field_ptr(mg_ctx* c, int l, int field, int xbuf) {
  return field == 0 ? c->dl[l].x[xbuf] : field == 1 ? c->dl[l].b : c->dl[l].cf;
}

// ghost cells (from the owned region) an exchange of x or b at level l makes valid (schedule.cpp)
int exch_depth(const mg_ctx* c, int l) { return Builder(c->lay).xdepth(l); }

// the cells per brick an exchange of x or b copies for a run of ghost direction r.dir: a sub-box
// [lo, hi) per axis, the whole brick when the exchange depth is the brick edge; returns the count
int64_t exch_box(const Layout& lay, int l, const Run& r, int32_t* box) {
  const int E = lay.E, dep = Builder(lay).xdepth(l);
  *box = 0;
  if (dep >= E) return lay.BV;
  int dd[3], lo[3], hi[3];
  dir_from_index(r.dir, dd[0], dd[1], dd[2]);
  int64_t cells = 1;
  for (int a = 0; a < 3; ++a) {  // ghost below the owned box: its top cells; above: its bottom ones
    lo[a] = dd[a] < 0 ? E - dep : 0;
    hi[a] = dd[a] > 0 ? dep : E;
    cells *= hi[a] - lo[a];
  }
  *box = copy_box(lo[0], hi[0], lo[1], hi[1], lo[2], hi[2], E);
  return cells;
}

mg_status do_exchange(mg_ctx* c, int l, int field, int xbuf, cudaStream_t s) {
  const LevelLayout& L = c->lay.lv[l];
  double* f = field_ptr(c, l, field, xbuf);
  const size_t bb = (size_t)c->lay.BV;
  if (c->use_peer) {
    if (!c->peer_ready) return set_err(MG_ERR_STATE, "peer transport: call mg_peer_connect first");
    const DevLevel& d = c->dl[l];
    const int fv = field == 0 ? xbuf : field + 1;
    CKC(c, launch_peer_copy(d.cruns + (size_t)fv * d.ncruns, d.ncruns, d.cmax, c->ps_nb, s));
  } else if (c->use_nccl) {
    CKN(c, ncclGroupStart());
    for (const Run& r : L.recvs)
      CKN(c, ncclRecv(f + r.local * bb, (size_t)r.count * bb, ncclFloat64, r.peer, c->nccl, s));
    for (const Run& r : L.sends)
      CKN(c, ncclSend(f + r.local * bb, (size_t)r.count * bb, ncclFloat64, r.peer, c->nccl, s));
    CKN(c, ncclGroupEnd());
  } else {
    // every run of the exchange in one copy kernel (tables built by fill_copy_tables)
    const DevLevel& d = c->dl[l];
    const int fv = field == 0 ? xbuf : field + 1;
    CKC(c, launch_copy_runs(d.cruns + (size_t)fv * d.ncruns, d.ncruns, d.cmax, s));
  }
  // the domain-face ghosts (non-periodic bc, reading A22): reflections of owned / just received
  // bricks, so after the receives on the same stream
  const DevLevel& d = c->dl[l];
  // (the coefficients are reflected evenly whatever the bc: the face coefficient at a domain face is c_p)
  if (d.nmirror > 0) CKC(c, launch_mirror(f, d.mirror, d.nmirror, field == 2 ? 1.0 : d.mirror_sign, s, c->lay.E));
  return MG_OK;
}

// Replicated bottom tables: global brick q <- its owner's owned b brick (from the all-gather
// buffer on NCCL, straight from the owner's field in a loopback group or a one-rank run), and this
// rank's owned coarsest bricks <- their global bricks (the solve leaves x in rp.x[1]).
mg_status fill_repl_tables(mg_ctx* c) {
  const Layout& lay = c->lay;
  if (!lay.repl) return MG_OK;
  const int lb = lay.L - 1;
  const int64_t nown = lay.lv[(size_t)lb].n_owned;
  const size_t bb = (size_t)c->lay.BV;
  c->rp.allgather = c->use_nccl;  // (a one-rank NCCL run too: the self-exchange tests cover the path)
  std::vector<CopyRun> g((size_t)lay.gb.n_owned), sc((size_t)2 * nown);
  for (int64_t q = 0; q < lay.gb.n_owned; ++q) {
    const int32_t src = lay.gb_src[(size_t)q];
    const int r = (int)(src / nown);
    const int64_t i = src % nown;
    const double* from;
    if (c->rp.allgather)
      from = c->rp.gbuf + (size_t)src * bb;
    else if (c->use_peer)  // the owner's b field through its IPC mapping
      from = (const double*)(c->peer_ws[(size_t)r] + ((const char*)c->dl[(size_t)lb].b - (const char*)c->peer_ws[(size_t)c->lay.rank])) +
             (size_t)i * bb;
    else if (c->group)
      from = c->group->r[(size_t)r]->dl[(size_t)lb].b + (size_t)i * bb;
    else
      from = c->dl[(size_t)lb].b + (size_t)i * bb;
    g[(size_t)q] = {from, c->rp.b + (size_t)q * bb, (int64_t)bb};
  }
  for (int xb = 0; xb < 2; ++xb)
    for (int64_t i = 0; i < nown; ++i)
      sc[(size_t)xb * nown + i] = {c->rp.x[1] + (size_t)lay.gb_mine[(size_t)i] * bb,
                                   c->dl[(size_t)lb].x[xb] + (size_t)i * bb, (int64_t)bb};
  CKC(c, cudaMemcpy(c->rp.gather, g.data(), g.size() * sizeof(CopyRun), cudaMemcpyHostToDevice));
  CKC(c, cudaMemcpy(c->rp.scatter, sc.data(), sc.size() * sizeof(CopyRun), cudaMemcpyHostToDevice));
  return MG_OK;
}

// Copy descriptors of the local transport: receiver ghost run <- sender surface run, for the
// three exchanged fields (x[0], x[1], b).  Needs every rank's workspace carved (loopback groups).
// The exchange fused into the pencil passes (SW_PEER): on a level whose owned range has a pencil plan,
// a periodic box (no mirrored faces) and constant coefficients, a pass that would follow an x exchange
// instead stages the side slabs, corner columns and warm-up / cool-down bricks of its ghost bricks
// straight from the owners' fields (the receive runs say which brick of which rank a ghost mirrors).
// MG_NO_FUSED_EXCH=1 keeps the separate exchange (A/B).

// The fused exchange's per-chunk source table of level L (PairArgs::pid) from its owned pencil plan and
// receive runs: [chunks][16] -1 (a local brick) or (rank << 24) | the brick of that rank's layout the
// ghost mirrors.  False if the level has no owned pencil plan or a ghost brick without a source.
static bool fused_pid_table(const LevelLayout& L, int W, std::vector<int32_t>& pid) {
  pid.clear();
  if (L.n_ghost == 0) return false;
  const LevelLayout::PairTable* pt = nullptr;
  for (const auto& t : L.pairs)
    if (t.b0 == 0 && t.b1 == L.n_owned && t.part == 0 && t.kind == 3) pt = &t;
  if (!pt) return false;
  std::vector<int2> g((size_t)L.n_ghost, make_int2(-1, -1));  // ghost brick -> (owner rank, its brick)
  for (const Run& r : L.recvs)
    for (int64_t k = 0; k < r.count; ++k)
      if (r.local + k >= L.n_owned && r.local + k < L.n_stored)
        g[(size_t)(r.local + k - L.n_owned)] = make_int2(r.peer, (int)(r.remote + k));
  const size_t nch = pt->meta.size() / kPenRec;
  pid.assign(nch * 16, -1);
  for (size_t ch = 0; ch < nch; ++ch)
    for (int e = 0; e < 16; ++e) {
      const int32_t id = pt->meta[ch * kPenRec + 1 + (size_t)e];
      if (id < L.n_owned) continue;
      if (id >= L.n_stored) return false;
      const int2 src = g[(size_t)(id - L.n_owned)];
      if (src.x < 0 || src.x >= W || src.y >= (1 << 24)) return false;
      pid[ch * 16 + (size_t)e] = (src.x << 24) | src.y;
    }
  return true;
}

static mg_status fill_fused_tables(mg_ctx* c) {
  if (!fused_exchange_enabled() || c->use_nccl) return MG_OK;
  const int W = c->group ? (int)c->group->r.size() : c->lay.world;
  if (W > 8) return MG_OK;  // (PairMaps::rbase)
  for (int l = 0; l < c->lay.L; ++l) {
    const LevelLayout& L = c->lay.lv[l];
    DevLevel& d = c->dl[l];
    d.fused = false;
    if (d.ncruns == 0 || L.n_ghost == 0 || d.nmirror > 0 || d.cf) continue;
    std::vector<int32_t> pid;
    if (!fused_pid_table(L, W, pid)) continue;
    std::vector<CUtensorMap> maps((size_t)2 * W * 3);
    d.rbase.assign((size_t)2 * W, nullptr);
    for (int xb = 0; xb < 2; ++xb)
      for (int r = 0; r < W; ++r) {
        const double* f = d.x[xb];
        if (c->group) f = c->group->r[(size_t)r]->dl[l].x[xb];
        else if (c->use_peer)
          f = (const double*)(c->peer_ws[(size_t)r] + ((const char*)d.x[xb] - (const char*)c->peer_ws[(size_t)c->lay.rank]));
        else if (r != c->lay.rank) return set_err(MG_ERR_STATE, "fused exchange: no mapping of another rank");
        PairMaps pm{};
        CKC(c, encode_pencil_maps(f, f, L.n_alloc, &pm));
        CUtensorMap* m = &maps[((size_t)xb * W + r) * 3];
        m[0] = pm.xwe;
        m[1] = pm.xsn;
        m[2] = pm.xcor;
        d.rbase[(size_t)xb * W + r] = f;
      }
    auto upload = [&](void** dst, const void* h, size_t bytes) -> mg_status {
      if (!*dst) {
        CKC(c, cudaMalloc(dst, bytes));
        c->allocs.push_back(*dst);
      }
      CKC(c, cudaMemcpy(*dst, h, bytes, cudaMemcpyHostToDevice));
      return MG_OK;
    };
    CKS(upload((void**)&d.pid, pid.data(), pid.size() * sizeof(int32_t)));
    CKS(upload((void**)&d.rmaps, maps.data(), maps.size() * sizeof(CUtensorMap)));
    d.rworld = W;
    d.fused = true;
  }
  return MG_OK;
}

mg_status fill_copy_tables(mg_ctx* c) {
  const size_t bb = (size_t)c->lay.BV;
  for (int l = 0; l < c->lay.L; ++l) {
    const LevelLayout& L = c->lay.lv[l];
    DevLevel& d = c->dl[l];
    if (d.ncruns == 0) continue;
    std::vector<CopyRun> h((size_t)d.ncruns * 4, CopyRun{nullptr, nullptr, 0});
    d.cmax = 0;
    // x and b: only the ghost cells within the exchange depth of the owned region (the cells the
    // sweeps up to the next exchange read: a sub-box per ghost region, from its direction); the
    // coefficients (exchanged once) whole
    for (int fv = 0; fv < 4; ++fv) {  // x[0], x[1], b, coefficients
      const int field = fv < 2 ? 0 : fv - 1, xbuf = fv < 2 ? fv : 0;
      double* f = field_ptr(c, l, field, xbuf);
      if (!f) continue;
      for (int i = 0; i < d.ncruns; ++i) {
        const Run& r = L.recvs[(size_t)i];
        mg_ctx* src = c->group ? c->group->r[r.peer] : c;
        const double* sf = field_ptr(src, l, field, xbuf);
        if (c->use_peer)  // the sender's field at the same workspace offset, through its IPC mapping
          sf = (const double*)(c->peer_ws[(size_t)r.peer] + ((const char*)f - (const char*)c->peer_ws[(size_t)c->lay.rank]));
        CopyRun cr{sf + r.remote * bb, f + r.local * bb, (int64_t)r.count * (int64_t)bb};
        const int64_t cells = fv < 3 ? exch_box(c->lay, l, r, &cr.box) : (int64_t)bb;
        h[(size_t)fv * d.ncruns + i] = cr;
        d.cmax = std::max<int64_t>(d.cmax, (int64_t)r.count * cells);
      }
    }
    CKC(c, cudaMemcpy(d.cruns, h.data(), h.size() * sizeof(CopyRun), cudaMemcpyHostToDevice));
  }
  return fill_fused_tables(c);
}

// ------------------------------------------------------------- executor
// part: for OP_SWEEP2, which units of the range's pencil plan (LevelLayout::PairTable::part)
// paper_stage (the paper's kernel set, in-place smooth): 0 = applyOp then smooth, 1 = applyOp only,
// 2 = smooth only -- a split sweep must finish every applyOp before the first in-place smooth
mg_status sweep_range(mg_ctx* c, const Op& o, int64_t b0, int64_t b1, cudaStream_t s, int part = 0,
                      int paper_stage = 0, bool peer = false) {
  if (b1 <= b0) return MG_OK;
  DevLevel& d = c->dl[o.level];
  const int l = o.level;
  Coeffs cc = d.c;  // the smoother's step for this sweep (Chebyshev variant) or the level's Jacobi step
  if (o.g1 > 0) cc.gamma = o.g1;
  if (o.paper) {
    if (paper_stage != 2) CKC(c, launch_apply_op(d.x[o.src], d.Ax, d.adj, b0, b1 - b0, cc, s, c->lay.E));
    if (paper_stage != 1)
      CKC(c, launch_smooth(d.x[o.src], d.Ax, d.b, d.r, b0, b1 - b0, cc, (o.flags & SW_WRITE_R) != 0, s, o.c1,
                           c->lay.E));
    return MG_OK;
  }
  SweepArgs a{};
  a.x = d.x[o.src];
  a.xo = d.x[o.dst];
  a.b = d.b;
  a.r = d.r;
  a.adj = d.adj;
  a.parent = d.parent;
  if (l + 1 < c->lay.L) {
    a.bc = c->dl[l + 1].b;
    a.xc = c->dl[l + 1].x[o.cbuf];
  }
  a.brick0 = b0;
  a.nbricks = b1 - b0;
  a.c = cc;
  a.gamma2 = o.g2 > 0 ? o.g2 : d.c.gamma;
  a.colour = o.c1;
  a.colour2 = o.c2;
  a.E = c->lay.E;
  unsigned fl = o.flags;
  if (d.cf) {  // variable coefficients (reading A23): the column kernel's variant where a plan exists
    a.cf = d.cf;
    a.vc_g = 0.5 * (d.h * d.h);
    fl |= SW_VARCOEF;
    if (c->use_col && col_supports(o.flags) && c->lay.E == 8)
      for (const auto& col : d.cols)
        if (col.b0 == b0 && col.b1 == b1) {
          CKC(c, launch_sweep_col(a, col.args, d.fmaps[o.src], fl, s, &d.cfmaps));
          return MG_OK;
        }
    CKC(c, launch_sweep(a, fl, s));
    return MG_OK;
  }
  if (o.kind == OP_SWEEP2) {  // two sweeps in one pass: the builder only emits it where a plan exists
    for (const auto& pr : d.pairs) {
      if (pr.b0 == b0 && pr.b1 == b1 && pr.part == part) {
        if (pr.args.kind == 3 && peer) {  // the exchange fused into the pass: ghost x from the owners
          PairArgs pa = pr.args;
          pa.pid = d.pid;
          pa.rmaps = d.rmaps + (size_t)o.src * d.rworld * 3;
          PairMaps pm = d.nmaps[o.src];
          for (int r = 0; r < d.rworld; ++r) pm.rbase[r] = d.rbase[(size_t)o.src * d.rworld + r];
          CKC(c, launch_sweep2p(a, pa, pm, o.flags | SW_PEER, s, o.fused == 2));
        } else if (pr.args.kind == 3) {
          // MG_PEN_PDL=<l0> (A/B runs): pencil passes of levels >= l0 launched with PDL
          static const int pen_pdl = getenv("MG_PEN_PDL") ? atoi(getenv("MG_PEN_PDL")) : 1 << 30;
          CKC(c, launch_sweep2p(a, pr.args, d.nmaps[o.src], o.flags | (o.zero ? SW_ZERO_X : 0u), s, l >= pen_pdl));
        }
        else
          CKC(c, launch_sweep2(a, pr.args, d.pmaps[o.src], o.flags, s));
        return MG_OK;
      }
    }
    return set_err(MG_ERR_STATE, "no two-sweep plan for this brick range");
  }
  if (c->use_col && col_supports(o.flags)) {
    for (const auto& col : d.cols) {
      if (col.b0 == b0 && col.b1 == b1) {
        CKC(c, launch_sweep_col(a, col.args, d.fmaps[o.src], o.flags, s));
        return MG_OK;
      }
    }
  }
  CKC(c, launch_sweep(a, o.flags, s));
  return MG_OK;
}

mg_status timer_begin(mg_ctx* c, cudaStream_t s, cudaEvent_t* ev) {
  if (!c->timing) return MG_OK;
  *ev = pool_event(c);
  CKC(c, cudaEventRecord(*ev, s));
  return MG_OK;
}
mg_status timer_end(mg_ctx* c, cudaStream_t s, cudaEvent_t a, int level, int op) {
  if (!c->timing) return MG_OK;
  cudaEvent_t b = pool_event(c);
  CKC(c, cudaEventRecord(b, s));
  c->trec.push_back({level * MG_NUM_OPS + op, a, b});
  return MG_OK;
}

mg_status exec_op(mg_ctx* c, const Op& o, cudaStream_t s) {
  const LevelLayout& L = c->lay.lv[o.level];
  DevLevel& d = c->dl[o.level];
  cudaEvent_t t0 = nullptr;
  switch (o.kind) {
    case OP_SWEEP:
    case OP_SWEEP2: {
      const int64_t end = o.ghosts ? L.n_stored : L.n_owned;
      if (o.fused) {  // the exchange fused into the pencil pass (fill_fused_tables)
        CKS(timer_begin(c, s, &t0));
        if (o.fused == 2) CKC(c, launch_peer_handshake(c->ps_nb, s));
        CKS(sweep_range(c, o, 0, end, s, 0, 0, true));
        CKS(timer_end(c, s, t0, o.level, o.timer));
        return MG_OK;
      }
      if (o.exch_before) {
        // pencil passes: the units that read no ghost brick overlap the exchange, the rest follow
        bool pen_split = false;
        if (o.kind == OP_SWEEP2 && c->lay.p.overlap && c->pencil_overlap)
          for (const auto& pr : d.pairs) pen_split |= pr.b0 == 0 && pr.b1 == end && pr.part == 1;
        if (pen_split) {
          CKS(timer_begin(c, s, &t0));
          CKC(c, cudaEventRecord(c->ev_fork, s));
          CKC(c, cudaStreamWaitEvent(c->comm, c->ev_fork, 0));
          CKS(do_exchange(c, o.level, 0, o.src, c->comm));
          CKC(c, cudaEventRecord(c->ev_join, c->comm));
          CKS(sweep_range(c, o, 0, end, s, 1));
          CKC(c, cudaStreamWaitEvent(s, c->ev_join, 0));
          CKS(sweep_range(c, o, 0, end, s, 2));
          CKS(timer_end(c, s, t0, o.level, o.timer));
          return MG_OK;
        }
        const bool split = c->lay.p.overlap && L.n_interior > 0 && !o.nosplit;
        if (split) {
          CKS(timer_begin(c, s, &t0));
          CKC(c, cudaEventRecord(c->ev_fork, s));
          CKC(c, cudaStreamWaitEvent(c->comm, c->ev_fork, 0));
          CKS(do_exchange(c, o.level, 0, o.src, c->comm));
          CKC(c, cudaEventRecord(c->ev_join, c->comm));
          if (o.paper) {  // in-place smooth: the surface bricks' applyOp must read the interior's old x
            CKS(sweep_range(c, o, 0, L.n_interior, s, 0, 1));
            CKC(c, cudaStreamWaitEvent(s, c->ev_join, 0));
            CKS(sweep_range(c, o, L.n_interior, end, s, 0, 1));
            CKS(sweep_range(c, o, 0, end, s, 0, 2));
          } else {
            CKS(sweep_range(c, o, 0, L.n_interior, s));
            CKC(c, cudaStreamWaitEvent(s, c->ev_join, 0));
            CKS(sweep_range(c, o, L.n_interior, end, s));
          }
          CKS(timer_end(c, s, t0, o.level, o.timer));
          return MG_OK;
        }
        CKS(timer_begin(c, s, &t0));
        CKS(do_exchange(c, o.level, 0, o.src, s));
        CKS(timer_end(c, s, t0, o.level, MG_OP_EXCHANGE));
      }
      CKS(timer_begin(c, s, &t0));
      CKS(sweep_range(c, o, 0, end, s));
      CKS(timer_end(c, s, t0, o.level, o.timer));
      return MG_OK;
    }
    case OP_RESTRICT:
      CKS(timer_begin(c, s, &t0));
      CKC(c, launch_restrict(d.r, c->dl[o.level + 1].b, d.parent, L.n_owned, s, c->lay.E));
      CKS(timer_end(c, s, t0, o.level, o.timer));
      return MG_OK;
    case OP_INTERP:
      CKS(timer_begin(c, s, &t0));
      CKC(c, launch_interp(d.x[o.src], c->dl[o.level + 1].x[o.cbuf], d.parent, L.n_owned, s, c->lay.E));
      CKS(timer_end(c, s, t0, o.level, o.timer));
      return MG_OK;
    case OP_ZERO:
      CKS(timer_begin(c, s, &t0));
      CKC(c, launch_zero(d.x[o.src], 0, L.n_stored, s, c->lay.E));
      CKS(timer_end(c, s, t0, o.level, o.timer));
      return MG_OK;
    case OP_EXCH:
      CKS(timer_begin(c, s, &t0));
      CKS(do_exchange(c, o.level, o.field, o.src, s));
      CKS(timer_end(c, s, t0, o.level, o.timer));
      return MG_OK;
    case OP_COARSE: {
      if (c->lay.p.bottom_mode == MG_BOTTOM_GRID) {
        GridCoarseArgs a{};
        a.nlev = c->lay.L - o.level;
        for (int l = o.level; l < c->lay.L; ++l) {
          const DevLevel& dl = c->dl[l];
          a.lv[l - o.level] = {c->lay.lv[l].n_owned, dl.adj, dl.parent, {dl.x[0], dl.x[1]}, dl.b, dl.c, dl.h};
        }
        const mg_params& P = c->lay.p;
        a.cheb = P.smoother == 1;
        for (int k = 0; a.cheb && k < P.pre_smooths; ++k) a.nu_pre[k] = cheb_nu(P.pre_smooths, k, P.cheby_ratio);
        for (int k = 0; a.cheb && k < P.post_smooths; ++k) a.nu_post[k] = cheb_nu(P.post_smooths, k, P.cheby_ratio);
        a.pre = P.pre_smooths;
        a.post = P.post_smooths;
        a.bottom = P.bottom_smooths;
        a.bar = reinterpret_cast<unsigned*>(c->acc + 8);  // zeroed at setup; consistent after every launch
        CKS(timer_begin(c, s, &t0));
        CKC(c, launch_coarse_grid(a, s));
        CKS(timer_end(c, s, t0, o.level, o.timer));
        return MG_OK;
      }
      CoarseArgs a{};
      a.nlev = c->lay.L - o.level;
      for (int l = o.level; l < c->lay.L; ++l) {
        const DevLevel& dl = c->dl[l];
        a.lv[l - o.level] = {(int)c->lay.lv[l].n_owned, dl.adj, dl.parent, dl.c, dl.h};
      }
      const mg_params& P = c->lay.p;
      a.cheb = P.smoother == 1;
      for (int k = 0; a.cheb && k < P.pre_smooths; ++k) a.nu_pre[k] = cheb_nu(P.pre_smooths, k, P.cheby_ratio);
      for (int k = 0; a.cheb && k < P.post_smooths; ++k) a.nu_post[k] = cheb_nu(P.post_smooths, k, P.cheby_ratio);
      a.b0 = d.b;
      a.x0 = d.x[o.dst];
      a.pre = c->lay.p.pre_smooths;
      a.post = c->lay.p.post_smooths;
      a.bottom = c->lay.p.bottom_smooths;
      CKS(timer_begin(c, s, &t0));
      CKC(c, launch_coarse(a, s));
      CKS(timer_end(c, s, t0, o.level, o.timer));
      return MG_OK;
    }
    case OP_BOTTOM_REPL: {
      const Layout& lay = c->lay;
      const int64_t ng = lay.gb.n_owned;
      CKS(timer_begin(c, s, &t0));
      if (c->rp.allgather)
        CKN(c, ncclAllGather(d.b, c->rp.gbuf, (size_t)L.n_owned * c->lay.BV, ncclFloat64, c->nccl, s));
      if (c->use_peer)
        CKC(c, launch_peer_copy(c->rp.gather, (int)ng, c->lay.BV, c->ps_all, s));
      else
        CKC(c, launch_copy_runs(c->rp.gather, (int)ng, c->lay.BV, s));
      if (lay.p.bottom_solver == 1) {
        CKC(c, launch_bottom_cg(c->rp.x[1], c->rp.b, c->rp.adj, c->rp.coord, (int)ng, lay.gb.n[0], lay.gb.n[1], o.n,
                                d.c, s));
      } else if (ng <= kResidentMaxBricks && !cluster_bottom_small()) {
        CKC(c, launch_bottom_resident(c->rp.x[0], c->rp.x[1], c->rp.b, c->rp.adj, (int)ng, o.n, true, d.c, s));
      } else if (ng <= kClusterBottomMaxBricks && cluster_bottom_enabled()) {
        CKC(c, launch_bottom_cluster(c->rp.x[0], c->rp.x[1], c->rp.b, c->rp.adj, (int)ng, o.n, true, d.c, s));
      } else {
        CoarseArgs a{};
        a.nlev = 1;
        a.lv[0] = {(int)ng, c->rp.adj, nullptr, d.c, d.h};
        a.b0 = c->rp.b;
        a.x0 = c->rp.x[1];
        a.pre = a.post = 0;
        a.bottom = o.n;
        CKC(c, launch_coarse(a, s));
      }
      CKC(c, launch_copy_runs(c->rp.scatter + (size_t)o.dst * L.n_owned, (int)L.n_owned, c->lay.BV, s));
      CKS(timer_end(c, s, t0, o.level, o.timer));
      return MG_OK;
    }
    case OP_BOTTOM_CG:
      CKS(timer_begin(c, s, &t0));
      CKC(c, launch_bottom_cg(d.x[o.dst], d.b, d.adj, d.coord, (int)L.n_owned, L.n[0], L.n[1], o.n, d.c, s));
      CKS(timer_end(c, s, t0, o.level, o.timer));
      return MG_OK;
    case OP_BOTTOM_RES:
      CKS(timer_begin(c, s, &t0));
      if (!L.radj.empty()) {  // non-periodic bc, one rank: owned bricks, domain faces as images
        auto f = L.n_owned <= kResidentMaxBricks && !cluster_bottom_small() ? launch_bottom_resident : launch_bottom_cluster;
        CKC(c, f(d.x[o.src], d.x[o.dst], d.b, d.radj, (int)L.n_owned, o.n, o.zero, d.c, s, d.mirror_sign));
      } else {
        auto f = L.n_stored <= kResidentMaxBricks && !cluster_bottom_small() ? launch_bottom_resident : launch_bottom_cluster;
        CKC(c, f(d.x[o.src], d.x[o.dst], d.b, d.adj, (int)L.n_stored, o.n, o.zero, d.c, s, 0.0));
      }
      CKS(timer_end(c, s, t0, o.level, o.timer));
      return MG_OK;
  }
  return set_err(MG_ERR_STATE, "unknown op");
}

Plan make_plan(const Builder& b, const Layout& lay, bool pencil_overlap, bool local_exchange,
               const mg_ctx* c = nullptr) {
  Plan p;
  p.ops = b.ops;
  if (c)  // pencil passes after an x exchange over the owned range of a fused-exchange level
    for (Op& o : p.ops) {
      const DevLevel& d = c->dl[o.level];
      if (o.kind == OP_SWEEP2 && o.exch_before && !o.ghosts && !o.zero && d.fused &&
          pencil_supports(o.flags) && !(lay.p.overlap && c->pencil_overlap)) {
        bool plan = false;
        for (const auto& pr : d.pairs)
          plan |= pr.b0 == 0 && pr.b1 == lay.lv[o.level].n_owned && pr.part == 0 && pr.args.kind == 3;
        if (plan) o.fused = (c->use_peer && lay.world > 1) ? 2 : 1;
      }
    }
  for (int l = 0; l < MG_MAX_LEVELS; ++l) p.final_st[l] = b.st[l];
  for (const Op& o : p.ops) p.launches += op_launches(o, lay, lay.p.overlap != 0, pencil_overlap, local_exchange);
  return p;
}

// execute a plan on one context or, in lockstep, on every rank of a group
mg_status run_plan(mg_ctx* c, mg_group* g, const Plan& p, cudaStream_t s) {
  for (const Op& o : p.ops) {
    if (g) {
      for (mg_ctx* r : g->r) CKS(exec_op(r, o, s));
    } else {
      CKS(exec_op(c, o, s));
    }
  }
  return MG_OK;
}

mg_status collect_timings(mg_ctx* c) {
  if (!c->timing) return MG_OK;
  CKC(c, cudaStreamSynchronize(c->stream));
  for (const TimerRec& t : c->trec) {
    float ms = 0;
    CKC(c, cudaEventElapsedTime(&ms, t.a, t.b));
    if (t.slot >= 0 && t.slot < (int)c->tm.size()) c->tm[t.slot] += ms;
    c->recs.push_back({t.slot, (double)ms});
  }
  c->trec.clear();
  c->evnext = 0;
  return MG_OK;
}

mg_status check_ctx(mg_ctx* c) {
  if (!c) return set_err(MG_ERR_INVALID_ARG, "null context");
  if (c->poisoned) return set_err(MG_ERR_STATE, "context poisoned by an earlier CUDA/NCCL error");
  if (cudaSetDevice(c->device) != cudaSuccess) return set_err(MG_ERR_CUDA, "cudaSetDevice failed");
  g_launch_pdl = c->lay.p.launch_pdl != 2;  // kernels enqueued or captured by this call
  return MG_OK;
}

mg_status build_and_run(mg_ctx* c, mg_group* g, bool vcycle_graph, Builder& b) {
  const Plan p = make_plan(b, c->lay, c->pencil_overlap, !c->use_nccl, c);  // (peer: one copy kernel too)
  CKS(prepare_plan(c, g, p.ops));
  CKS(run_plan(c, g, p, g ? g->stream : c->stream));
  if (g) {
    for (mg_ctx* r : g->r)
      for (int l = 0; l < MG_MAX_LEVELS; ++l) r->st[l] = p.final_st[l];
  } else {
    for (int l = 0; l < MG_MAX_LEVELS; ++l) c->st[l] = p.final_st[l];
  }
  c->last_launches = p.launches * (g ? (int64_t)g->r.size() : 1);
  (void)vcycle_graph;
  return MG_OK;
}

// V-cycle for a single context or a lockstep group, via a cached CUDA graph
mg_status vcycle_impl(mg_ctx* c, mg_group* g) {
  mg_ctx* c0 = g ? g->r[0] : c;
  if (c0->lay.p.var_coef && !c0->coef_ready)
    return set_err(MG_ERR_STATE, "var_coef: set the coefficients (mg_set_coefficients) first");
  cudaStream_t s = g ? g->stream : c->stream;
  const int key = c0->st[0].cur & 1;
  const bool graph = c0->lay.p.use_graph && !c0->timing;
  cudaGraphExec_t* gexec = g ? g->gexec : c->gexec;
  Plan* gplan = g ? g->gplan : c->gplan;
  bool* gvalid = g ? g->gvalid : c->gvalid;
  if (!graph || !gvalid[key]) {
    Builder b(c0->lay);
    for (int l = 0; l < MG_MAX_LEVELS; ++l) b.st[l] = c0->st[l];
    b.vcycle();
    Plan p = make_plan(b, c0->lay, c0->pencil_overlap, !c0->use_nccl, c0);
    CKS(prepare_plan(c0, g, p.ops));
    if (graph) {
      // capture on a private non-blocking stream; the graph is then launched on the caller's stream
      cudaStream_t cs = g ? g->cap : c->cap;
      CKC(c0, cudaStreamBeginCapture(cs, cudaStreamCaptureModeThreadLocal));
      mg_status rs = run_plan(c0, g, p, cs);
      cudaGraph_t gr = nullptr;
      cudaError_t ce = cudaStreamEndCapture(cs, &gr);
      if (rs != MG_OK) return rs;
      CKC(c0, ce);
      CKC(c0, cudaGraphInstantiate(&gexec[key], gr, 0));
      cudaGraphDestroy(gr);
      gplan[key] = p;
      gvalid[key] = true;
    } else {
      CKS(run_plan(c0, g, p, s));
      if (g) {
        for (mg_ctx* r : g->r) {
          for (int l = 0; l < MG_MAX_LEVELS; ++l) r->st[l] = p.final_st[l];
          CKS(collect_timings(r));
        }
      } else {
        for (int l = 0; l < MG_MAX_LEVELS; ++l) c->st[l] = p.final_st[l];
        CKS(collect_timings(c));
      }
      c0->last_launches = p.launches * (g ? (int64_t)g->r.size() : 1);
      return MG_OK;
    }
  }
  CKC(c0, cudaGraphLaunch(gexec[key], s));
  const Plan& p = gplan[key];
  if (g) {
    for (mg_ctx* r : g->r)
      for (int l = 0; l < MG_MAX_LEVELS; ++l) r->st[l] = p.final_st[l];
  } else {
    for (int l = 0; l < MG_MAX_LEVELS; ++l) c->st[l] = p.final_st[l];
  }
  c0->last_launches = p.launches * (g ? (int64_t)g->r.size() : 1);
  return MG_OK;
}

// Pencil passes with the exchange overlapped (the units that read no ghost brick swept while the exchange
// runs, the rest after it): off by default -- measured on one B200 with the 2x2x2 halo pattern (peer
// kernel or local copies), the split costs 1.0-1.2 ms per 512^3 cycle (two launches per pass, part 1 on
// fewer CTAs, part 2's tail), more than the 12 depth-limited level-0 exchanges it could hide (~0.5 ms
// over NVLink).  MG_PENCIL_OVERLAP=1 turns it on.
bool pencil_overlap_on() {
  const char* e = getenv("MG_PENCIL_OVERLAP");
  return e && atoi(e) != 0;
}

// MG_POISON_GHOSTS=1 (tests): every ghost cell of every field starts as NaN (and x's ghosts again after
// mg_set_solution(NULL)), so a kernel reading a ghost cell the exchange did not refresh -- a cell
// beyond the exchange depth, or one stale since the last exchange -- poisons the owned results
bool poison_ghosts_on() {
  const char* e = getenv("MG_POISON_GHOSTS");
  return e && atoi(e) != 0;
}
cudaError_t poison_ghosts(mg_ctx* c, int l, bool x_only, cudaStream_t s) {
  const LevelLayout& L = c->lay.lv[(size_t)l];
  const DevLevel& d = c->dl[(size_t)l];
  if (L.n_ghost == 0) return cudaSuccess;
  const size_t off = (size_t)L.n_owned * c->lay.BV, bytes = (size_t)L.n_ghost * c->lay.BV * sizeof(double);
  double* f[6] = {d.x[0], d.x[1], d.b, d.r, d.Ax, d.cf};
  for (int k = 0; k < (x_only ? 2 : 6); ++k) {
    if (!f[k]) continue;
    cudaError_t e = cudaMemsetAsync(f[k] + off, 0xff, bytes, s);  // all-ones: a NaN
    if (e != cudaSuccess) return e;
  }
  return cudaSuccess;
}

mg_status init_ctx(mg_ctx* c, const mg_params& p, int rank, int world, int device, cudaStream_t stream,
                   void* workspace, size_t ws_bytes, bool tables_only_upload) {
  std::string msg;
  mg_status s = build_layout(p, rank, world, c->lay, msg);
  if (s != MG_OK) return set_err(s, msg);
  c->device = device;
  c->stream = stream;
  c->use_col = p.sweep_kernel != 1;
  c->pencil_overlap = pencil_overlap_on();
  const size_t need = carve(c->lay, nullptr, nullptr, nullptr, nullptr);
  if (!workspace || ws_bytes < need)
    return set_err(MG_ERR_OOM, "workspace too small: need " + std::to_string(need) + " bytes");
  if (((uintptr_t)workspace & 255) != 0) return set_err(MG_ERR_INVALID_ARG, "workspace must be 256-byte aligned");
  carve(c->lay, (char*)workspace, &c->dl, c->stage, &c->acc, &c->rp, &c->pa);
  c->peer_ws.assign((size_t)world, nullptr);
  c->peer_ws[(size_t)rank] = (char*)workspace;
  (void)tables_only_upload;
  CKC(c, cudaMemsetAsync(workspace, 0, need, stream));
  if (poison_ghosts_on())
    for (int l = 0; l < c->lay.L; ++l) CKC(c, poison_ghosts(c, l, false, stream));
  for (int l = 0; l < c->lay.L; ++l) {
    const LevelLayout& L = c->lay.lv[l];
    DevLevel& d = c->dl[l];
    CKC(c, cudaMemcpyAsync(d.adj, L.adj.data(), L.adj.size() * sizeof(int32_t), cudaMemcpyHostToDevice, stream));
    std::vector<int32_t> par = L.parent;
    par.resize((size_t)L.n_alloc, -1);
    CKC(c, cudaMemcpyAsync(d.parent, par.data(), par.size() * sizeof(int32_t), cudaMemcpyHostToDevice, stream));
    CKC(c, cudaMemcpyAsync(d.coord, L.coord.data(), L.coord.size() * sizeof(int32_t), cudaMemcpyHostToDevice,
                           stream));
    if (!L.mirror.empty())
      CKC(c, cudaMemcpyAsync(d.mirror, L.mirror.data(), L.mirror.size() * sizeof(int32_t), cudaMemcpyHostToDevice,
                             stream));
    if (!L.radj.empty())
      CKC(c, cudaMemcpyAsync(d.radj, L.radj.data(), L.radj.size() * sizeof(int32_t), cudaMemcpyHostToDevice, stream));
    for (size_t k = 0; k < L.cols.size(); ++k) {
      const auto& ct = L.cols[k];
      const ColArgs& ca = d.cols[k].args;
      CKC(c, cudaMemcpyAsync((void*)ca.bricks, ct.bricks.data(), ct.bricks.size() * 4, cudaMemcpyHostToDevice, stream));
      CKC(c, cudaMemcpyAsync((void*)ca.side, ct.side.data(), ct.side.size() * 4, cudaMemcpyHostToDevice, stream));
      CKC(c, cudaMemcpyAsync((void*)ca.segs, ct.segs.data(), ct.segs.size() * 4, cudaMemcpyHostToDevice, stream));
    }
    if (!L.cols.empty()) {
      for (int xb = 0; xb < 2; ++xb) CKC(c, encode_face_maps(d.x[xb], L.n_alloc, &d.fmaps[xb]));
      if (d.cf) CKC(c, encode_face_maps(d.cf, L.n_alloc, &d.cfmaps));
    }
    for (size_t k = 0; k < L.pairs.size(); ++k) {
      const auto& pt = L.pairs[k];
      const PairArgs& pa = d.pairs[k].args;
      CKC(c, cudaMemcpyAsync((void*)pa.meta, pt.meta.data(), pt.meta.size() * 4, cudaMemcpyHostToDevice, stream));
      CKC(c, cudaMemcpyAsync((void*)pa.ctas, pt.ctas.data(), pt.ctas.size() * 4, cudaMemcpyHostToDevice, stream));
    }
    if (!L.pairs.empty())
      for (int xb = 0; xb < 2; ++xb) {
        CKC(c, encode_pair_maps(d.x[xb], d.b, L.n_alloc, &d.pmaps[xb]));
        CKC(c, encode_pencil_maps(d.x[xb], d.b, L.n_alloc, &d.nmaps[xb]));
      }
  }
  if (c->lay.repl) {
    CKC(c, cudaMemcpyAsync(c->rp.adj, c->lay.gb.adj.data(), c->lay.gb.adj.size() * sizeof(int32_t),
                           cudaMemcpyHostToDevice, stream));
    CKC(c, cudaMemcpyAsync(c->rp.coord, c->lay.gb.coord.data(), c->lay.gb.coord.size() * sizeof(int32_t),
                           cudaMemcpyHostToDevice, stream));
  }
  CKC(c, cudaStreamSynchronize(stream));  // host vectors above are temporaries
  CKC(c, cudaStreamCreateWithFlags(&c->comm, cudaStreamNonBlocking));
  CKC(c, cudaStreamCreateWithFlags(&c->cap, cudaStreamNonBlocking));
  CKC(c, cudaEventCreateWithFlags(&c->ev_fork, cudaEventDisableTiming));
  CKC(c, cudaEventCreateWithFlags(&c->ev_join, cudaEventDisableTiming));
  CKC(c, cudaStreamCreateWithFlags(&c->h2d, cudaStreamNonBlocking));
  for (int k = 0; k < 2; ++k) {
    CKC(c, cudaEventCreateWithFlags(&c->ev_h2d[k], cudaEventDisableTiming));
    CKC(c, cudaEventCreateWithFlags(&c->ev_free[k], cudaEventDisableTiming));
  }
  CKC(c, cudaEventCreateWithFlags(&c->ev_norm, cudaEventDisableTiming));
  CKC(c, cudaMallocHost((void**)&c->h_pinned, 64));
  c->tm.assign((size_t)c->lay.L * MG_NUM_OPS, 0.0);
  for (int l = 0; l < MG_MAX_LEVELS; ++l) c->st[l] = LevelState();
  c->st[0].db = 0;
  return MG_OK;
}

void free_ctx(mg_ctx* c) {
  if (!c) return;
  for (int k = 0; k < 2; ++k)
    if (c->gexec[k]) cudaGraphExecDestroy(c->gexec[k]);
  if (c->nccl) ncclCommDestroy(c->nccl);
  if (c->comm) cudaStreamDestroy(c->comm);
  if (c->cap) cudaStreamDestroy(c->cap);
  if (c->h2d) {
    cudaStreamSynchronize(c->h2d);
    cudaStreamDestroy(c->h2d);
  }
  for (int k = 0; k < 2; ++k) {
    if (c->ev_h2d[k]) cudaEventDestroy(c->ev_h2d[k]);
    if (c->ev_free[k]) cudaEventDestroy(c->ev_free[k]);
  }
  if (c->ev_norm) cudaEventDestroy(c->ev_norm);
  if (c->ev_fork) cudaEventDestroy(c->ev_fork);
  if (c->ev_join) cudaEventDestroy(c->ev_join);
  for (cudaEvent_t e : c->evpool) cudaEventDestroy(e);
  if (c->h_pinned) cudaFreeHost(c->h_pinned);
  for (void* a : c->allocs) cudaFree(a);
  for (void* a : c->peer_open) cudaIpcCloseMemHandle(a);
  delete c;
}

mg_status set_level_field(mg_ctx* c, int l, int field, const double* src, bool exchange_b) {
  if (l < 0 || l >= c->lay.L) return set_err(MG_ERR_INVALID_ARG, "level out of range");
  if (((uintptr_t)src & 15) != 0) return set_err(MG_ERR_INVALID_ARG, "field pointer must be 16-byte aligned");
  DevLevel& d = c->dl[l];
  const LevelLayout& L = c->lay.lv[l];
  double* dst = field == MG_FIELD_X ? d.x[c->st[l].cur] : field == MG_FIELD_B ? d.b : d.r;
  CKC(c, launch_lex_to_brick(src, dst, d.coord, L.n_owned, L.n[0], L.n[1], c->stream, c->lay.E));
  if (field == MG_FIELD_X) {
    c->st[l].dx = 0;
    c->st[l].since = 1 << 20;
  }
  if (field == MG_FIELD_B) {
    c->st[l].db = 0;
    if (exchange_b && L.n_ghost > 0) {
      CKS(do_exchange(c, l, 1, 0, c->stream));
      c->st[l].db = exch_depth(c, l);
    }
  }
  return MG_OK;
}

}  // namespace

// =====================================================================================
extern "C" {

void mg_params_default(mg_params* p) {
  if (!p) return;
  std::memset(p, 0, sizeof(*p));
  for (int a = 0; a < 3; ++a) {
    p->n_local[a] = 256;
    p->proc_grid[a] = 1;
  }
  p->num_levels = 6;  // -l 6
  p->pre_smooths = 12;
  p->post_smooths = 12;
  p->bottom_smooths = 100;
  p->use_graph = 1;
  p->overlap = 1;
  p->temporal_blocking = 3;
  p->h0 = 0.0;
}

mg_status mg_workspace_bytes(const mg_params* p, int32_t rank, int32_t world_size, size_t* out_bytes) {
  if (!p || !out_bytes) return set_err(MG_ERR_INVALID_ARG, "null argument");
  Layout lay;
  std::string msg;
  const mg_params q = normalized(p);
  CKS(check_params(q));
  mg_status s = build_layout(q, rank, world_size, lay, msg);
  if (s != MG_OK) return set_err(s, msg);
  *out_bytes = carve(lay, nullptr, nullptr, nullptr, nullptr);
  return MG_OK;
}

mg_status mg_nccl_unique_id(uint8_t out_id[128]) {
  if (!out_id) return set_err(MG_ERR_INVALID_ARG, "null argument");
  ncclUniqueId id;
  ncclResult_t r = ncclGetUniqueId(&id);
  if (r != ncclSuccess) return set_err(MG_ERR_NCCL, std::string("ncclGetUniqueId: ") + ncclGetErrorString(r));
  static_assert(sizeof(id) == 128, "ncclUniqueId size");
  std::memcpy(out_id, &id, 128);
  return MG_OK;
}

static mg_status peer_connect_impl(mg_ctx* c, const uint8_t* blobs);

mg_status mg_setup(const mg_params* p, int32_t rank, int32_t world_size, const uint8_t* nccl_id, int32_t device,
                   void* cuda_stream, void* workspace, size_t ws_bytes, mg_ctx** out) {
  if (!p || !out) return set_err(MG_ERR_INVALID_ARG, "null argument");
  *out = nullptr;
  const mg_params q = normalized(p);
  CKS(check_params(q));
  int ndev = 0;
  cudaError_t ce = cudaGetDeviceCount(&ndev);
  if (ce != cudaSuccess || ndev == 0)
    return set_err(MG_ERR_CUDA, std::string("no CUDA device (no CPU fallback): ") + cudaGetErrorString(ce));
  if (device < 0 || device >= ndev) return set_err(MG_ERR_INVALID_ARG, "device out of range");
  ce = cudaSetDevice(device);
  if (ce != cudaSuccess) return set_err(MG_ERR_CUDA, std::string("cudaSetDevice: ") + cudaGetErrorString(ce));
  ce = kernels_init();
  if (ce != cudaSuccess) return set_err(MG_ERR_CUDA, std::string("kernels_init: ") + cudaGetErrorString(ce));
  mg_ctx* c = new mg_ctx();
  mg_status s = init_ctx(c, q, rank, world_size, device, (cudaStream_t)cuda_stream, workspace, ws_bytes, false);
  if (s != MG_OK) {
    free_ctx(c);
    return s;
  }
  bool any_ghost = false;
  for (const auto& L : c->lay.lv) any_ghost |= L.n_ghost > 0;
  // between processes: peer memory by default (MG_TRANSPORT_AUTO / PEER), NCCL when asked for
  c->use_peer = (world_size > 1 && q.transport == MG_TRANSPORT_AUTO) || q.transport == MG_TRANSPORT_PEER;
  const bool want_nccl = q.transport == MG_TRANSPORT_NCCL;
  if (world_size > 1 && q.transport == MG_TRANSPORT_LOCAL) {
    free_ctx(c);
    return set_err(MG_ERR_INVALID_ARG, "multi-process runs need the NCCL transport (use mg_group_* for loopback)");
  }
  if (want_nccl) {
    ncclUniqueId id;
    if (nccl_id) {
      std::memcpy(&id, nccl_id, 128);
    } else if (world_size == 1) {
      ncclResult_t r = ncclGetUniqueId(&id);
      if (r != ncclSuccess) {
        free_ctx(c);
        return set_err(MG_ERR_NCCL, std::string("ncclGetUniqueId: ") + ncclGetErrorString(r));
      }
    } else {
      free_ctx(c);
      return set_err(MG_ERR_INVALID_ARG, "world_size > 1 needs an NCCL unique id");
    }
    ncclResult_t r = ncclCommInitRank(&c->nccl, world_size, id, rank);
    if (r != ncclSuccess) {
      c->nccl = nullptr;
      free_ctx(c);
      return set_err(MG_ERR_NCCL, std::string("ncclCommInitRank: ") + ncclGetErrorString(r));
    }
    c->use_nccl = true;
  }
  (void)any_ghost;
  if (!c->use_nccl && !c->use_peer) {  // (peer: at mg_peer_connect, once the mappings exist)
    s = fill_copy_tables(c);
    if (s != MG_OK) {
      free_ctx(c);
      return s;
    }
  }
  if (!c->use_peer) {
    s = fill_repl_tables(c);
    if (s != MG_OK) {
      free_ctx(c);
      return s;
    }
  } else if (world_size == 1) {  // a one-rank self-exchange through the peer kernel (no participants)
    s = peer_connect_impl(c, nullptr);
    if (s != MG_OK) {
      free_ctx(c);
      return s;
    }
  }
  *out = c;
  return MG_OK;
}

mg_status mg_set_rhs(mg_ctx* c, const double* b_dev) {
  CKS(check_ctx(c));
  if (!b_dev) return set_err(MG_ERR_INVALID_ARG, "null b");
  return set_level_field(c, 0, MG_FIELD_B, b_dev, c->group == nullptr);
}

mg_status mg_set_rhs_host(mg_ctx* c, const double* b_host) {
  CKS(check_ctx(c));
  if (!b_host) return set_err(MG_ERR_INVALID_ARG, "null b");
  CKS(ensure_stage(c));
  const size_t bytes = (size_t)c->lay.lv[0].n_owned * c->lay.BV * sizeof(double);
  // Upload on the copy stream into staging field k (free once its previous conversion ran), so
  // the transfer overlaps whatever the caller's stream is still executing (the V-cycle of the
  // previous right-hand side); the conversion into bricks is ordered on the caller's stream.
  const int k = c->stage_k;
  c->stage_k ^= 1;
  CKC(c, cudaStreamWaitEvent(c->h2d, c->ev_free[k], 0));
  CKC(c, cudaMemcpyAsync(c->stage[k], b_host, bytes, cudaMemcpyHostToDevice, c->h2d));
  CKC(c, cudaEventRecord(c->ev_h2d[k], c->h2d));
  CKC(c, cudaStreamWaitEvent(c->stream, c->ev_h2d[k], 0));
  CKS(set_level_field(c, 0, MG_FIELD_B, c->stage[k], c->group == nullptr));
  CKC(c, cudaEventRecord(c->ev_free[k], c->stream));
  return MG_OK;
}

// Variable coefficients (reading A23): level-0 c from a local lexicographic array, coarse c = the
// restriction of the level above (restrict_kernel: the canonical volume average), then (one rank) the
// ghost bricks of every level by exchange / mirror (c is reflected evenly).  Group members restrict
// locally; mg_group_commit_coefficients exchanges once every rank has its c.
static mg_status set_coefficients_impl(mg_ctx* c, const double* c_dev, cudaStream_t s) {
  if (!c->lay.p.var_coef) return set_err(MG_ERR_STATE, "var_coef is 0: this context has the paper's constant operator");
  if (!c_dev || ((uintptr_t)c_dev & 15)) return set_err(MG_ERR_INVALID_ARG, "c must be a 16-byte aligned device pointer");
  const LevelLayout& L0 = c->lay.lv[0];
  CKC(c, launch_lex_to_brick(c_dev, c->dl[0].cf, c->dl[0].coord, L0.n_owned, L0.n[0], L0.n[1], s, c->lay.E));
  for (int l = 0; l + 1 < c->lay.L; ++l)
    CKC(c, launch_restrict(c->dl[l].cf, c->dl[l + 1].cf, c->dl[l].parent, c->lay.lv[l].n_owned, s, c->lay.E));
  return MG_OK;
}

static mg_status exchange_coefficients(mg_ctx* c, cudaStream_t s) {
  for (int l = 0; l < c->lay.L; ++l)
    if (c->lay.lv[l].n_ghost > 0) CKS(do_exchange(c, l, 2, 0, s));
  c->coef_ready = true;
  return MG_OK;
}

mg_status mg_set_coefficients(mg_ctx* c, const double* c_dev) {
  CKS(check_ctx(c));
  if (c->group) return set_err(MG_ERR_STATE, "group member: use mg_group_set_coefficients");
  CKS(set_coefficients_impl(c, c_dev, c->stream));
  return exchange_coefficients(c, c->stream);
}

mg_status mg_set_solution(mg_ctx* c, const double* x_dev) {
  CKS(check_ctx(c));
  if (!x_dev) {
    const LevelLayout& L = c->lay.lv[0];
    CKC(c, cudaMemsetAsync(c->dl[0].x[c->st[0].cur], 0, (size_t)L.n_stored * c->lay.BV * sizeof(double), c->stream));
    if (poison_ghosts_on()) CKC(c, poison_ghosts(c, 0, true, c->stream));
    c->st[0].dx = 0;
    return MG_OK;
  }
  return set_level_field(c, 0, MG_FIELD_X, x_dev, false);
}

mg_status mg_get_solution(mg_ctx* c, double* x_dev) {
  CKS(check_ctx(c));
  if (!x_dev || ((uintptr_t)x_dev & 15)) return set_err(MG_ERR_INVALID_ARG, "x must be a 16-byte aligned pointer");
  const LevelLayout& L = c->lay.lv[0];
  CKC(c, launch_brick_to_lex(c->dl[0].x[c->st[0].cur], x_dev, c->dl[0].coord, L.n_owned, L.n[0], L.n[1], c->stream, c->lay.E));
  return MG_OK;
}

mg_status mg_get_solution_host(mg_ctx* c, double* x_host) {
  CKS(check_ctx(c));
  if (!x_host) return set_err(MG_ERR_INVALID_ARG, "null x");
  CKS(ensure_stage(c));
  const int k = c->stage_k;  // every upload into it is already ordered before its conversion
  CKS(mg_get_solution(c, c->stage[k]));
  const size_t bytes = (size_t)c->lay.lv[0].n_owned * c->lay.BV * sizeof(double);
  CKC(c, cudaMemcpyAsync(x_host, c->stage[k], bytes, cudaMemcpyDeviceToHost, c->stream));
  CKC(c, cudaEventRecord(c->ev_free[k], c->stream));
  CKC(c, cudaStreamSynchronize(c->stream));
  return MG_OK;
}

mg_status mg_vcycle(mg_ctx* c) {
  CKS(check_ctx(c));
  if (c->group) return set_err(MG_ERR_STATE, "group member: use mg_group_vcycle");
  return vcycle_impl(c, nullptr);
}

// max |b - Ax| of level 0's owned cells -> atomicMax on *acc: the TMA column kernel (16 B/pt at its
// streaming rate) where level 0 has a column plan over the owned range, else the one-brick kernel
static mg_status norm_launch(mg_ctx* c, unsigned long long* acc, cudaStream_t s) {
  const LevelLayout& L = c->lay.lv[0];
  DevLevel& d = c->dl[0];
  const int cur = c->st[0].cur;
  if (c->use_col && c->lay.E == 8) {
    for (const auto& col : d.cols) {
      if (col.b0 == 0 && col.b1 == L.n_owned) {
        SweepArgs a{};
        a.x = d.x[cur];
        a.b = d.b;
        a.adj = d.adj;
        a.brick0 = 0;
        a.nbricks = L.n_owned;
        a.c = d.c;
        a.acc = acc;
        a.cf = d.cf;  // (variable coefficients: the column kernel's coefficient variant)
        a.vc_g = 0.5 * (d.h * d.h);
        CKC(c, launch_sweep_col(a, col.args, d.fmaps[cur], SW_NORM | (d.cf ? SW_VARCOEF : 0u), s, &d.cfmaps));
        return MG_OK;
      }
    }
  }
  CKC(c, launch_norm(d.x[cur], d.b, d.adj, L.n_owned, d.c, acc, s, d.cf, c->lay.E));
  return MG_OK;
}

mg_status mg_residual_norm_async(mg_ctx* c) {
  CKS(check_ctx(c));
  if (c->group) return set_err(MG_ERR_STATE, "group member: use mg_group_residual_norm");
  if (c->norm_pending) return set_err(MG_ERR_STATE, "a residual norm is already pending: call mg_residual_norm_wait");
  if (c->lay.p.var_coef && !c->coef_ready)
    return set_err(MG_ERR_STATE, "var_coef: set the coefficients (mg_set_coefficients) first");
  const LevelLayout& L = c->lay.lv[0];
  DevLevel& d = c->dl[0];
  if (L.n_ghost > 0) {
    CKS(do_exchange(c, 0, 0, c->st[0].cur, c->stream));
    c->st[0].dx = exch_depth(c, 0);
    c->st[0].since = 0;
  }
  CKC(c, cudaMemsetAsync(c->acc, 0, sizeof(unsigned long long), c->stream));
  CKS(norm_launch(c, c->acc, c->stream));
  if (c->use_nccl && c->lay.world > 1)
    CKN(c, ncclAllReduce(c->acc, c->acc, 1, ncclUint64, ncclMax, c->nccl, c->stream));
  if (c->use_peer && c->lay.world > 1) {
    if (!c->peer_ready) return set_err(MG_ERR_STATE, "peer transport: call mg_peer_connect first");
    CKC(c, launch_peer_allmax(c->acc, c->ps_all, c->d_remote_vals, c->pa.vals, c->lay.rank, c->lay.world, c->stream));
  }
  CKC(c, cudaMemcpyAsync(c->h_pinned, c->acc, sizeof(unsigned long long), cudaMemcpyDeviceToHost, c->stream));
  CKC(c, cudaEventRecord(c->ev_norm, c->stream));
  c->norm_pending = true;
  return MG_OK;
}

mg_status mg_residual_norm_wait(mg_ctx* c, double* out) {
  CKS(check_ctx(c));
  if (!out) return set_err(MG_ERR_INVALID_ARG, "null out");
  if (!c->norm_pending) return set_err(MG_ERR_STATE, "no residual norm pending: call mg_residual_norm_async");
  c->norm_pending = false;
  CKC(c, cudaEventSynchronize(c->ev_norm));
  std::memcpy(out, c->h_pinned, sizeof(double));
  return MG_OK;
}

mg_status mg_residual_norm(mg_ctx* c, double* out) {
  CKS(check_ctx(c));
  if (!out) return set_err(MG_ERR_INVALID_ARG, "null out");
  CKS(mg_residual_norm_async(c));
  return mg_residual_norm_wait(c, out);
}

mg_status mg_solve(mg_ctx* c, double tol, int32_t max_cycles, int32_t* cycles_done, double* final_norm) {
  CKS(check_ctx(c));
  double nr = 0;
  CKS(mg_residual_norm(c, &nr));
  int k = 0;
  while (nr > tol && k < max_cycles) {
    CKS(mg_vcycle(c));
    CKS(mg_residual_norm(c, &nr));
    ++k;
  }
  if (cycles_done) *cycles_done = k;
  if (final_norm) *final_norm = nr;
  // a NaN norm fails `nr > tol` as well as `nr <= tol`: the loop stops at once and the solve reports
  // that it did not converge (a diverged iteration must never look converged)
  if (!std::isfinite(nr)) return set_err(MG_NOT_CONVERGED, "residual norm is not finite: the iteration diverged");
  return nr <= tol ? MG_OK : MG_NOT_CONVERGED;
}

mg_status mg_set_timing(mg_ctx* c, int32_t enabled) {
  CKS(check_ctx(c));
  c->timing = enabled != 0;
  std::fill(c->tm.begin(), c->tm.end(), 0.0);
  c->recs.clear();
  return MG_OK;
}

mg_status mg_get_timing_records(mg_ctx* c, int32_t* slots, double* ms, int32_t cap, int32_t* count) {
  CKS(check_ctx(c));
  if (!count || (cap > 0 && (!slots || !ms))) return set_err(MG_ERR_INVALID_ARG, "null out");
  CKS(collect_timings(c));
  const int n = std::min<int>(cap, (int)c->recs.size());
  for (int i = 0; i < n; ++i) {
    slots[i] = c->recs[(size_t)i].first;
    ms[i] = c->recs[(size_t)i].second;
  }
  *count = (int32_t)c->recs.size();
  return MG_OK;
}

mg_status mg_get_timings(mg_ctx* c, double* out, int32_t cap) {
  CKS(check_ctx(c));
  if (!out) return set_err(MG_ERR_INVALID_ARG, "null out");
  CKS(collect_timings(c));
  const int n = std::min<int>(cap, (int)c->tm.size());
  for (int i = 0; i < n; ++i) out[i] = c->tm[i];
  return MG_OK;
}

mg_status mg_vcycle_launches(mg_ctx* c, int64_t* out) {
  CKS(check_ctx(c));
  if (!out) return set_err(MG_ERR_INVALID_ARG, "null out");
  Builder b(c->lay);
  for (int l = 0; l < MG_MAX_LEVELS; ++l) b.st[l] = c->st[l];
  b.vcycle();
  *out = make_plan(b, c->lay, c->pencil_overlap, !c->use_nccl, c).launches;
  return MG_OK;
}

mg_status mg_exchange_stats(mg_ctx* c, int64_t* bytes_per_cycle, int64_t* messages_per_cycle) {
  CKS(check_ctx(c));
  Builder b(c->lay);
  for (int l = 0; l < MG_MAX_LEVELS; ++l) b.st[l] = c->st[l];
  b.vcycle();
  int64_t bytes = 0, msgs = 0;
  for (const Op& o : b.ops) {
    const bool ex = o.kind == OP_EXCH || ((o.kind == OP_SWEEP || o.kind == OP_SWEEP2) && o.exch_before);
    if (!ex) continue;
    for (const Run& r : c->lay.lv[o.level].sends) {
      int32_t box;
      bytes += r.count * exch_box(c->lay, o.level, r, &box) * (int64_t)sizeof(double);
      ++msgs;
    }
  }
  if (bytes_per_cycle) *bytes_per_cycle = bytes;
  if (messages_per_cycle) *messages_per_cycle = msgs;
  return MG_OK;
}

// per level: exchanges in the cycle the builder compiles from state st (NULL: a fresh context's), and
// the bytes one exchange of x sends
static void exchange_plan_of(const Layout& lay, const LevelState* st, int64_t* exchanges, int64_t* bytes) {
  Builder b(lay);
  if (st)
    for (int l = 0; l < MG_MAX_LEVELS; ++l) b.st[l] = st[l];
  b.vcycle();
  for (int l = 0; l < lay.L; ++l) {
    exchanges[l] = 0;
    bytes[l] = 0;
    int32_t box;
    for (const Run& r : lay.lv[l].sends) bytes[l] += r.count * exch_box(lay, l, r, &box) * (int64_t)sizeof(double);
  }
  for (const Op& o : b.ops)
    if (o.kind == OP_EXCH || ((o.kind == OP_SWEEP || o.kind == OP_SWEEP2) && o.exch_before)) ++exchanges[o.level];
}

mg_status mg_exchange_plan(mg_ctx* c, int32_t cap, int64_t* exchanges, int64_t* bytes) {
  CKS(check_ctx(c));
  if (cap < c->lay.L || !exchanges || !bytes) return set_err(MG_ERR_INVALID_ARG, "need cap >= num_levels and outputs");
  exchange_plan_of(c->lay, c->st, exchanges, bytes);
  return MG_OK;
}

mg_status mg_exchange_fused(mg_ctx* c, int32_t cap, int64_t* fused) {
  CKS(check_ctx(c));
  if (cap < c->lay.L || !fused) return set_err(MG_ERR_INVALID_ARG, "need cap >= num_levels and an output");
  Builder b(c->lay);
  for (int l = 0; l < MG_MAX_LEVELS; ++l) b.st[l] = c->st[l];
  b.vcycle();
  const Plan p = make_plan(b, c->lay, c->pencil_overlap, !c->use_nccl, c);
  for (int l = 0; l < c->lay.L; ++l) fused[l] = 0;
  for (const Op& o : p.ops)
    if (o.fused) ++fused[o.level];
  return MG_OK;
}

mg_status mg_exchange_time(mg_ctx* c, int32_t level, int32_t reps, double* ms_per_exchange) {
  CKS(check_ctx(c));
  if (c->group) return set_err(MG_ERR_STATE, "group member: not supported");
  if (!ms_per_exchange || reps < 1 || level < 0 || level >= c->lay.L)
    return set_err(MG_ERR_INVALID_ARG, "bad level / reps / output");
  *ms_per_exchange = 0.0;
  if (c->lay.lv[level].n_ghost == 0) return MG_OK;
  // x of the level (its ghosts are refreshed: harmless for the V-cycle state, whose ghost validity
  // only ever grows by an exchange)
  const int xb = c->st[level].cur;
  CKS(do_exchange(c, level, 0, xb, c->stream));  // warm-up (NCCL connection setup on first use)
  cudaEvent_t e0 = pool_event(c), e1 = pool_event(c);
  CKC(c, cudaEventRecord(e0, c->stream));
  for (int i = 0; i < reps; ++i) CKS(do_exchange(c, level, 0, xb, c->stream));
  CKC(c, cudaEventRecord(e1, c->stream));
  CKC(c, cudaEventSynchronize(e1));
  float ms = 0.f;
  CKC(c, cudaEventElapsedTime(&ms, e0, e1));
  c->evnext = 0;
  *ms_per_exchange = (double)ms / reps;
  return MG_OK;
}

namespace {
struct PeerBlob {  // MG_PEER_BLOB_BYTES: what one rank publishes for the others to map it
  cudaIpcMemHandle_t handle;  // of the allocation holding the workspace
  int64_t ws_off;             // workspace pointer - allocation base
  int32_t world, rank;
  int64_t ws_bytes;
};
static_assert(sizeof(PeerBlob) <= MG_PEER_BLOB_BYTES, "peer blob");
}  // namespace

mg_status mg_peer_blob(mg_ctx* c, uint8_t* out) {
  CKS(check_ctx(c));
  if (!out) return set_err(MG_ERR_INVALID_ARG, "null out");
  if (!c->use_peer) return set_err(MG_ERR_STATE, "not a peer-transport context");
  static PFN_cuMemGetAddressRange_v3020 range = nullptr;
  if (!range) {
    void* fn = nullptr;
    cudaDriverEntryPointQueryResult qr;
    CKC(c, cudaGetDriverEntryPoint("cuMemGetAddressRange", &fn, cudaEnableDefault, &qr));
    if (qr != cudaDriverEntryPointSuccess || !fn) return set_err(MG_ERR_CUDA, "cuMemGetAddressRange unavailable");
    range = reinterpret_cast<PFN_cuMemGetAddressRange_v3020>(fn);
  }
  char* ws = c->peer_ws.empty() ? nullptr : c->peer_ws[(size_t)c->lay.rank];
  CUdeviceptr base = 0;
  size_t size = 0;
  if (range(&base, &size, (CUdeviceptr)ws) != CUDA_SUCCESS) return set_err(MG_ERR_CUDA, "cuMemGetAddressRange failed");
  PeerBlob b{};
  CKC(c, cudaIpcGetMemHandle(&b.handle, (void*)base));
  b.ws_off = (int64_t)((CUdeviceptr)ws - base);
  b.world = c->lay.world;
  b.rank = c->lay.rank;
  b.ws_bytes = (int64_t)size;
  std::memset(out, 0, MG_PEER_BLOB_BYTES);
  std::memcpy(out, &b, sizeof(b));
  return MG_OK;
}

static mg_status peer_connect_impl(mg_ctx* c, const uint8_t* blobs) {
  const int W = c->lay.world, me = c->lay.rank;
  char* mine = c->peer_ws[(size_t)me];
  for (int r = 0; r < W && W > 1; ++r) {
    PeerBlob b;
    std::memcpy(&b, blobs + (size_t)r * MG_PEER_BLOB_BYTES, sizeof(b));
    if (b.world != W || b.rank != r) return set_err(MG_ERR_INVALID_ARG, "peer blobs out of order or from another run");
    if (r == me) continue;
    void* p = nullptr;
    CKC(c, cudaIpcOpenMemHandle(&p, b.handle, cudaIpcMemLazyEnablePeerAccess));
    c->peer_open.push_back(p);
    c->peer_ws[(size_t)r] = (char*)p + b.ws_off;
  }
  // every rank carves the same workspace layout (same local geometry): rank r's object at offset o
  // of its workspace is the object at offset o of this rank's
  auto at = [&](int r, const void* local) { return c->peer_ws[(size_t)r] + ((const char*)local - mine); };
  std::vector<unsigned long long*> remote((size_t)W * 2, nullptr), rvals((size_t)W, nullptr);
  for (int r = 0; r < W; ++r) {
    for (int k = 0; k < 2; ++k)  // THIS rank's slot (me, k) in rank r's flag array
      remote[(size_t)r * 2 + k] = (unsigned long long*)at(r, c->pa.flags + ((size_t)me * 2 + k) * kPeerSlotU64);
    rvals[(size_t)r] = (unsigned long long*)at(r, c->pa.vals);
  }
  std::vector<int> nb, all;
  for (int r = 0; r < W; ++r)
    if (r != me) all.push_back(r);
  for (const auto& L : c->lay.lv)
    for (const Run& r : L.recvs)
      if (r.peer != me && std::find(nb.begin(), nb.end(), r.peer) == nb.end()) nb.push_back(r.peer);
  std::sort(nb.begin(), nb.end());
  // small device tables (library-owned)
  auto upload = [&](const void* h, size_t bytes) -> void* {
    void* d = nullptr;
    if (cudaMalloc(&d, bytes) != cudaSuccess) return nullptr;
    c->allocs.push_back(d);
    if (cudaMemcpy(d, h, bytes, cudaMemcpyHostToDevice) != cudaSuccess) return nullptr;
    return d;
  };
  void* d_remote = upload(remote.data(), remote.size() * sizeof(void*));
  void* d_rvals = upload(rvals.data(), rvals.size() * sizeof(void*));
  const int npart_nb = (int)nb.size(), npart_all = (int)all.size();
  nb.push_back(0);  // (never read past npart: keeps the device arrays non-empty on one rank)
  all.push_back(0);
  void* d_nb = upload(nb.data(), nb.size() * sizeof(int));
  void* d_all = upload(all.data(), all.size() * sizeof(int));
  if (!d_remote || !d_rvals || !d_nb || !d_all) return set_err(MG_ERR_CUDA, "peer tables: cudaMalloc / cudaMemcpy failed");
  c->d_remote_vals = (unsigned long long**)d_rvals;
  PeerSync base{};
  base.flags = c->pa.flags;
  base.remote = (unsigned long long* const*)d_remote;
  base.epoch = c->pa.epoch;
  base.done = c->pa.done;
  base.dummy_run = c->pa.dummy;
  c->ps_nb = base;
  c->ps_nb.part = (const int*)d_nb;
  c->ps_nb.npart = npart_nb;
  c->ps_all = base;
  c->ps_all.part = (const int*)d_all;
  c->ps_all.npart = npart_all;
  c->peer_ready = true;
  CKS(fill_copy_tables(c));
  CKS(fill_repl_tables(c));
  CKC(c, cudaDeviceSynchronize());
  return MG_OK;
}

mg_status mg_peer_connect(mg_ctx* c, const uint8_t* blobs) {
  CKS(check_ctx(c));
  if (!blobs) return set_err(MG_ERR_INVALID_ARG, "null blobs");
  if (!c->use_peer) return set_err(MG_ERR_STATE, "not a peer-transport context");
  if (c->peer_ready) return set_err(MG_ERR_STATE, "already connected");
  return peer_connect_impl(c, blobs);
}

mg_status mg_destroy(mg_ctx* c) {
  if (!c) return MG_OK;
  if (c->group) return set_err(MG_ERR_STATE, "group member: use mg_group_destroy");
  cudaSetDevice(c->device);
  free_ctx(c);
  return MG_OK;
}

const char* mg_last_error(void) { return g_err.c_str(); }

// ---------------------------------------------------------------- per-op
mg_status mg_level_set(mg_ctx* c, int32_t level, int32_t field, const double* src_dev) {
  CKS(check_ctx(c));
  if (!src_dev || field < 0 || field > MG_FIELD_R) return set_err(MG_ERR_INVALID_ARG, "bad field/pointer");
  return set_level_field(c, level, field, src_dev, c->group == nullptr);
}

mg_status mg_level_get(mg_ctx* c, int32_t level, int32_t field, double* dst_dev) {
  CKS(check_ctx(c));
  if (!dst_dev || field < 0 || field > MG_FIELD_R || ((uintptr_t)dst_dev & 15))
    return set_err(MG_ERR_INVALID_ARG, "bad field/pointer");
  if (level < 0 || level >= c->lay.L) return set_err(MG_ERR_INVALID_ARG, "level out of range");
  DevLevel& d = c->dl[level];
  const LevelLayout& L = c->lay.lv[level];
  const double* src = field == MG_FIELD_X ? d.x[c->st[level].cur] : field == MG_FIELD_B ? d.b : d.r;
  CKC(c, launch_brick_to_lex(src, dst_dev, d.coord, L.n_owned, L.n[0], L.n[1], c->stream, c->lay.E));
  return MG_OK;
}

static mg_status single_only(mg_ctx* c) {
  if (c->group) return set_err(MG_ERR_STATE, "per-op entry points are for single contexts");
  return MG_OK;
}

mg_status mg_op_smooth(mg_ctx* c, int32_t level, int32_t n, int32_t write_r, int32_t fusion) {
  CKS(check_ctx(c));
  CKS(single_only(c));
  if (level < 0 || level >= c->lay.L || n < 0 || fusion < 0 || fusion > MG_FUSION_FULL)
    return set_err(MG_ERR_INVALID_ARG, "bad level/n/fusion");
  Builder b(c->lay);
  for (int l = 0; l < MG_MAX_LEVELS; ++l) b.st[l] = c->st[l];
  b.fusion_override[level] = fusion == MG_FUSION_PAPER ? MG_FUSION_PAPER : MG_FUSION_SWEEP;
  b.phase(level, n, false, write_r ? 1 : 0, false, MG_OP_SWEEP);
  return build_and_run(c, nullptr, false, b);
}

mg_status mg_op_restrict(mg_ctx* c, int32_t level) {
  CKS(check_ctx(c));
  CKS(single_only(c));
  if (level < 0 || level + 1 >= c->lay.L) return set_err(MG_ERR_INVALID_ARG, "restriction needs level+1 < L");
  Builder b(c->lay);
  for (int l = 0; l < MG_MAX_LEVELS; ++l) b.st[l] = c->st[l];
  b.restrict_op(level);
  return build_and_run(c, nullptr, false, b);
}

mg_status mg_op_interp(mg_ctx* c, int32_t level) {
  CKS(check_ctx(c));
  CKS(single_only(c));
  if (level < 0 || level + 1 >= c->lay.L) return set_err(MG_ERR_INVALID_ARG, "interpolation needs level+1 < L");
  Builder b(c->lay);
  for (int l = 0; l < MG_MAX_LEVELS; ++l) b.st[l] = c->st[l];
  b.interp_op(level);
  return build_and_run(c, nullptr, false, b);
}

mg_status mg_op_bottom(mg_ctx* c, int32_t level, int32_t n) {
  CKS(check_ctx(c));
  CKS(single_only(c));
  if (level < 0 || level >= c->lay.L || n < 0) return set_err(MG_ERR_INVALID_ARG, "bad level/n");
  Builder b(c->lay);
  for (int l = 0; l < MG_MAX_LEVELS; ++l) b.st[l] = c->st[l];
  b.bottom(level, n, false);
  return build_and_run(c, nullptr, false, b);
}

mg_status mg_sync(mg_ctx* c) {
  CKS(check_ctx(c));
  CKC(c, cudaStreamSynchronize(c->stream));
  return MG_OK;
}

// ---------------------------------------------------------------- loopback group
mg_status mg_group_setup(const mg_params* p, int32_t world_size, int32_t device, void* cuda_stream, void* workspace,
                         size_t ws_bytes, mg_group** out) {
  if (!p || !out || world_size < 1) return set_err(MG_ERR_INVALID_ARG, "bad argument");
  *out = nullptr;
  const mg_params q = normalized(p);
  CKS(check_params(q));
  int ndev = 0;
  cudaError_t ce = cudaGetDeviceCount(&ndev);
  if (ce != cudaSuccess || ndev == 0)
    return set_err(MG_ERR_CUDA, std::string("no CUDA device (no CPU fallback): ") + cudaGetErrorString(ce));
  ce = cudaSetDevice(device);
  if (ce != cudaSuccess) return set_err(MG_ERR_CUDA, std::string("cudaSetDevice: ") + cudaGetErrorString(ce));
  ce = kernels_init();
  if (ce != cudaSuccess) return set_err(MG_ERR_CUDA, std::string("kernels_init: ") + cudaGetErrorString(ce));
  size_t per = 0;
  CKS(mg_workspace_bytes(&q, 0, world_size, &per));
  per = align256(per);
  if (!workspace || ws_bytes < per * (size_t)world_size)
    return set_err(MG_ERR_OOM, "group workspace too small: need " + std::to_string(per * (size_t)world_size));
  mg_group* g = new mg_group();
  g->stream = (cudaStream_t)cuda_stream;
  if (cudaStreamCreateWithFlags(&g->cap, cudaStreamNonBlocking) != cudaSuccess) {
    delete g;
    return set_err(MG_ERR_CUDA, "cudaStreamCreate failed");
  }
  for (int r = 0; r < world_size; ++r) {
    mg_ctx* c = new mg_ctx();
    mg_status s = init_ctx(c, q, r, world_size, device, g->stream, (char*)workspace + per * (size_t)r, per, false);
    c->group = g;
    c->grank = r;
    g->r.push_back(c);
    if (s != MG_OK) {
      mg_group_destroy(g);
      return s;
    }
  }
  for (mg_ctx* c : g->r) {  // every rank's fields exist now: the cross-rank copy tables
    mg_status s = fill_copy_tables(c);
    if (s == MG_OK) s = fill_repl_tables(c);
    if (s != MG_OK) {
      mg_group_destroy(g);
      return s;
    }
  }
  *out = g;
  return MG_OK;
}

mg_status mg_group_ctx(mg_group* g, int32_t rank, mg_ctx** out) {
  if (!g || !out || rank < 0 || rank >= (int)g->r.size()) return set_err(MG_ERR_INVALID_ARG, "bad rank");
  *out = g->r[rank];
  return MG_OK;
}

mg_status mg_group_set_rhs(mg_group* g, int32_t rank, const double* b_dev) {
  mg_ctx* c = nullptr;
  CKS(mg_group_ctx(g, rank, &c));
  return mg_set_rhs(c, b_dev);
}

mg_status mg_group_set_solution(mg_group* g, int32_t rank, const double* x_dev) {
  mg_ctx* c = nullptr;
  CKS(mg_group_ctx(g, rank, &c));
  return mg_set_solution(c, x_dev);
}

mg_status mg_group_set_coefficients(mg_group* g, int32_t rank, const double* c_dev) {
  mg_ctx* c = nullptr;
  CKS(mg_group_ctx(g, rank, &c));
  return set_coefficients_impl(c, c_dev, g->stream);
}

mg_status mg_group_commit_coefficients(mg_group* g) {
  if (!g) return set_err(MG_ERR_INVALID_ARG, "null group");
  for (mg_ctx* c : g->r) {
    CKS(check_ctx(c));
    CKS(exchange_coefficients(c, g->stream));
  }
  return MG_OK;
}

mg_status mg_group_commit_rhs(mg_group* g) {
  if (!g) return set_err(MG_ERR_INVALID_ARG, "null group");
  for (mg_ctx* c : g->r) {
    CKS(check_ctx(c));
    if (c->lay.lv[0].n_ghost > 0) CKS(do_exchange(c, 0, 1, 0, g->stream));
    c->st[0].db = exch_depth(c, 0);
  }
  return MG_OK;
}

mg_status mg_group_vcycle(mg_group* g) {
  if (!g) return set_err(MG_ERR_INVALID_ARG, "null group");
  CKS(check_ctx(g->r[0]));
  return vcycle_impl(g->r[0], g);
}

mg_status mg_group_residual_norm(mg_group* g, double* out) {
  if (!g || !out) return set_err(MG_ERR_INVALID_ARG, "null argument");
  mg_ctx* c0 = g->r[0];
  CKS(check_ctx(c0));
  if (c0->lay.p.var_coef && !c0->coef_ready)
    return set_err(MG_ERR_STATE, "var_coef: set the coefficients (mg_group_set_coefficients + commit) first");
  for (mg_ctx* c : g->r) {
    if (c->lay.lv[0].n_ghost > 0) {
      CKS(do_exchange(c, 0, 0, c->st[0].cur, g->stream));
    }
  }
  for (mg_ctx* c : g->r) {
    c->st[0].dx = exch_depth(c, 0);
    c->st[0].since = 0;
  }
  CKC(c0, cudaMemsetAsync(c0->acc, 0, sizeof(unsigned long long), g->stream));
  for (mg_ctx* c : g->r) {
    const LevelLayout& L = c->lay.lv[0];
    DevLevel& d = c->dl[0];
    CKC(c0, launch_norm(d.x[c->st[0].cur], d.b, d.adj, L.n_owned, d.c, c0->acc, g->stream, d.cf, c->lay.E));
  }
  CKC(c0, cudaMemcpyAsync(c0->h_pinned, c0->acc, 8, cudaMemcpyDeviceToHost, g->stream));
  CKC(c0, cudaStreamSynchronize(g->stream));
  std::memcpy(out, c0->h_pinned, sizeof(double));
  return MG_OK;
}

mg_status mg_group_destroy(mg_group* g) {
  if (!g) return MG_OK;
  for (int k = 0; k < 2; ++k)
    if (g->gexec[k]) cudaGraphExecDestroy(g->gexec[k]);
  for (mg_ctx* c : g->r) free_ctx(c);
  if (g->cap) cudaStreamDestroy(g->cap);
  delete g;
  return MG_OK;
}

// ---------------------------------------------------------------- layout queries
struct mg_layout {
  Layout lay;
};

mg_status mg_layout_create(const mg_params* p, int32_t rank, int32_t world_size, mg_layout** out) {
  if (!p || !out) return set_err(MG_ERR_INVALID_ARG, "null argument");
  mg_layout* m = new mg_layout();
  std::string msg;
  const mg_params q = normalized(p);
  mg_status s = build_layout(q, rank, world_size, m->lay, msg);
  if (s != MG_OK) {
    delete m;
    return set_err(s, msg);
  }
  *out = m;
  return MG_OK;
}

static mg_status lay_level(const mg_layout* m, int32_t level, const LevelLayout** L) {
  if (!m || level < 0 || level >= m->lay.L) return set_err(MG_ERR_INVALID_ARG, "bad layout/level");
  *L = &m->lay.lv[level];
  return MG_OK;
}

mg_status mg_layout_level_info(const mg_layout* m, int32_t level, int64_t info[16]) {
  const LevelLayout* L = nullptr;
  CKS(lay_level(m, level, &L));
  for (int a = 0; a < 3; ++a) {
    info[a] = L->n[a];
    info[3 + a] = L->nb[a];
    info[6 + a] = L->g[a];
  }
  info[9] = L->n_owned;
  info[10] = L->n_interior;
  info[11] = L->n_ghost;
  info[12] = L->n_alloc;
  info[13] = (int64_t)L->sends.size();
  info[14] = (int64_t)L->recvs.size();
  info[15] = L->zero_brick;
  return MG_OK;
}

mg_status mg_layout_repl(const mg_layout* m, int64_t info[2], int32_t* gb_src, int32_t* gb_mine, int32_t* gb_adj) {
  if (!m || !info) return set_err(MG_ERR_INVALID_ARG, "null argument");
  const Layout& lay = m->lay;
  info[0] = lay.repl ? lay.gb.n_owned : 0;
  info[1] = lay.lv[(size_t)lay.L - 1].n_owned;
  if (!lay.repl) return MG_OK;
  if (gb_src) std::copy(lay.gb_src.begin(), lay.gb_src.end(), gb_src);
  if (gb_mine) std::copy(lay.gb_mine.begin(), lay.gb_mine.end(), gb_mine);
  if (gb_adj) std::copy(lay.gb.adj.begin(), lay.gb.adj.end(), gb_adj);
  return MG_OK;
}

mg_status mg_layout_adjacency(const mg_layout* m, int32_t level, int32_t* out) {
  const LevelLayout* L = nullptr;
  CKS(lay_level(m, level, &L));
  std::memcpy(out, L->adj.data(), L->adj.size() * sizeof(int32_t));
  return MG_OK;
}

mg_status mg_layout_fused_pid(const mg_layout* m, int32_t level, int64_t* count, int32_t* out) {
  const LevelLayout* L = nullptr;
  CKS(lay_level(m, level, &L));
  if (!count) return set_err(MG_ERR_INVALID_ARG, "null count");
  Builder b(m->lay);
  std::vector<int32_t> pid;
  *count = 0;
  if (!b.fused_level(level) || !fused_pid_table(*L, m->lay.world, pid)) return MG_OK;
  *count = (int64_t)pid.size();
  if (out) std::memcpy(out, pid.data(), pid.size() * sizeof(int32_t));
  return MG_OK;
}

mg_status mg_layout_coords(const mg_layout* m, int32_t level, int32_t* out) {
  const LevelLayout* L = nullptr;
  CKS(lay_level(m, level, &L));
  std::memcpy(out, L->coord.data(), L->coord.size() * sizeof(int32_t));
  return MG_OK;
}

mg_status mg_layout_parent(const mg_layout* m, int32_t level, int32_t* out) {
  const LevelLayout* L = nullptr;
  CKS(lay_level(m, level, &L));
  for (int64_t b = 0; b < L->n_stored; ++b) out[b] = L->parent.empty() ? -1 : L->parent[(size_t)b];
  return MG_OK;
}

mg_status mg_layout_plan(const mg_layout* m, int32_t level, int32_t which, int64_t* out) {
  const LevelLayout* L = nullptr;
  CKS(lay_level(m, level, &L));
  const std::vector<Run>& v = which ? L->recvs : L->sends;
  for (size_t i = 0; i < v.size(); ++i) {
    out[i * 6 + 0] = v[i].peer;
    out[i * 6 + 1] = v[i].dir;
    out[i * 6 + 2] = v[i].run;
    out[i * 6 + 3] = v[i].local;
    out[i * 6 + 4] = v[i].remote;
    out[i * 6 + 5] = v[i].count;
  }
  return MG_OK;
}

mg_status mg_layout_mirror(const mg_layout* m, int32_t level, int64_t* count, int32_t* out) {
  const LevelLayout* L = nullptr;
  CKS(lay_level(m, level, &L));
  if (!count) return set_err(MG_ERR_INVALID_ARG, "null count");
  *count = (int64_t)(L->mirror.size() / 3);
  if (out) std::memcpy(out, L->mirror.data(), L->mirror.size() * sizeof(int32_t));
  return MG_OK;
}

mg_status mg_layout_pass_plan(const mg_layout* m, int32_t level, int32_t idx, int64_t info[6], int32_t* meta,
                              int32_t* ctas) {
  const LevelLayout* L = nullptr;
  CKS(lay_level(m, level, &L));
  if (!info) return set_err(MG_ERR_INVALID_ARG, "null info");
  if (idx < 0 || idx >= (int32_t)L->pairs.size()) return set_err(MG_ERR_INVALID_ARG, "no such pass plan");
  const auto& t = L->pairs[(size_t)idx];
  info[0] = t.kind;
  info[1] = t.b0;
  info[2] = t.b1;
  info[3] = (int64_t)t.meta.size();
  info[4] = (int64_t)t.ctas.size();
  info[5] = t.part;
  if (meta) std::copy(t.meta.begin(), t.meta.end(), meta);
  if (ctas) std::copy(t.ctas.begin(), t.ctas.end(), ctas);
  return MG_OK;
}

mg_status mg_layout_vcycle_launches(const mg_layout* m, int32_t local_exchange, int64_t* out) {
  if (!m || !out) return set_err(MG_ERR_INVALID_ARG, "null argument");
  Builder b(m->lay);
  b.vcycle();  // from the state of a fresh context (every level's ghosts stale)
  const bool pencil_overlap = pencil_overlap_on();
  int64_t n = 0;
  for (const Op& o : b.ops) n += op_launches(o, m->lay, m->lay.p.overlap != 0, pencil_overlap, local_exchange != 0);
  *out = n;
  return MG_OK;
}

mg_status mg_layout_exchange_plan(const mg_layout* m, int32_t cap, int64_t* exchanges, int64_t* bytes) {
  if (!m || !exchanges || !bytes) return set_err(MG_ERR_INVALID_ARG, "null argument");
  if (cap < m->lay.L) return set_err(MG_ERR_INVALID_ARG, "need cap >= num_levels");
  exchange_plan_of(m->lay, nullptr, exchanges, bytes);
  return MG_OK;
}

mg_status mg_layout_destroy(mg_layout* m) {
  delete m;
  return MG_OK;
}

}  // extern "C"
