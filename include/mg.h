/*
 * mg.h -- C ABI of the B200-native brick geometric-multigrid V-cycle.
 *
 * The library (paper_conf_sc_antepara0jh24_b200/libmg_b200.so) implements the
 * FP64 V-cycle of Antepara, Williams, Johansen, Hall, "High-Performance,
 * Scalable Geometric Multigrid via Fine-Grain Data Blocking for GPUs"
 * (SC'24).  Citations "P:Lnn" are lines of that paper's text.
 *
 *   problem     3D periodic Poisson, 7-point operator A x = alpha x + beta *
 *               (sum of 6 neighbours), alpha = -6/h^2, beta = 1/h^2, h the
 *               spacing of the level (Fig 1)
 *   smoother    point Jacobi x := x + gamma (Ax - b), gamma = h^2/12
 *   residual    r = b - Ax from the same Ax as the smooth
 *   restriction average of the 8 fine cells of a coarse cell
 *   interp.     piecewise-constant x^h += I(x^2h)
 *   V-cycle     Alg 2; GMG loop Alg 1
 *   layout      8^3 bricks stored contiguously with an adjacency table
 *               (P:L17, L59, L61, L154); surface bricks ordered so that the
 *               ghost exchange sends contiguous brick runs with no packing,
 *               one brick-deep ghost zone shared by several smooths
 *               (communication avoiding).
 *
 * Conventions
 *   - Every function returns mg_status: 0 success, >0 warning, <0 error.  No
 *     exception or exit() crosses the ABI.  On error a thread-local message
 *     is available from mg_last_error().  A CUDA or NCCL error poisons the
 *     context: later calls on it return MG_ERR_STATE.
 *   - Field arrays passed in/out are FP64, C-contiguous, local lexicographic
 *     with x fastest: index i + n_local[0]*(j + n_local[1]*k).  "_dev"
 *     pointers are CUDA device pointers on the context's device; "_host"
 *     pointers are host memory (pinned or pageable).  The caller owns all
 *     arrays and the workspace; the workspace must outlive the context.
 *   - The library owns its host tables, streams, events, CUDA graphs and the
 *     NCCL communicator and frees them in mg_destroy / mg_group_destroy.
 *   - Collective calls (mg_setup, mg_set_rhs, mg_set_solution, mg_vcycle,
 *     mg_residual_norm, mg_solve) must be made by all ranks in the same order.
 *   - mg_vcycle, mg_set_rhs_host and mg_residual_norm_async are stream-ordered
 *     and never synchronise the host; mg_residual_norm, mg_residual_norm_wait,
 *     mg_solve and mg_get_solution_host synchronise.
 *   - One context per process and GPU; not thread-safe.
 *   - There is no CPU fallback: without a usable CUDA device mg_setup fails
 *     with MG_ERR_CUDA.
 */
#ifndef MG_B200_H
#define MG_B200_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  MG_OK = 0,
  MG_NOT_CONVERGED = 1,   /* mg_solve hit max_cycles before tol (warning) */
  MG_ERR_INVALID_ARG = -1,
  MG_ERR_CUDA = -2,
  MG_ERR_NCCL = -3,
  MG_ERR_OOM = -4,        /* workspace too small */
  MG_ERR_STATE = -5       /* context poisoned by an earlier error, or wrong call order */
} mg_status;

#define MG_MAX_LEVELS 16
#define MG_BRICK 8          /* default brick edge: 8^3 bricks; params brick_edge = 4 selects 4^3 */
#define MG_MAX_PERIOD 8     /* ghost depth in cells = brick edge; 4 with 4^3 bricks */

/* fusion[l] variants.  Every variant produces bit-identical results. */
enum {
  MG_FUSION_AUTO = 0,
  MG_FUSION_PAPER = 1,    /* the paper's kernel set: applyOp, smooth+residual, restriction,
                             initZero, interpolation+increment as separate kernels (Alg 2) */
  MG_FUSION_SWEEP = 2,    /* applyOp+smooth(+residual) fused into one ping-pong sweep kernel */
  MG_FUSION_FULL = 3      /* + restriction fused into the last pre-sweep, interpolation into the
                             first post-sweep, initZero folded into the first coarse sweep */
};

/* ghost_mode */
enum {
  MG_GHOST_AUTO = 0,      /* ghost shell only on axes with proc_grid > 1; periodic wrap
                             through the adjacency table on the others */
  MG_GHOST_ALL = 1        /* ghost shell on every axis, even when the neighbour is this rank
                             (self-exchange: measures communication avoiding on 1 GPU) */
};

/* bc: domain boundary condition of every level (variant; reading A22).
 * PERIODIC is the paper's model problem.  DIRICHLET / NEUMANN are homogeneous conditions on
 * the faces of the cell-centred grid: the neighbour across a domain face is -x_p / +x_p.  The library
 * gives every axis a one-brick ghost shell; the domain-face ghost bricks hold the reflected values
 * (filled by a "mirror exchange" wherever an exchange runs: method of images), so every kernel and
 * the communication-avoiding schedule run unchanged. */
enum { MG_BC_PERIODIC = 0, MG_BC_DIRICHLET = 1, MG_BC_NEUMANN = 2 };

/* transport */
enum { MG_TRANSPORT_AUTO = 0, MG_TRANSPORT_NCCL = 1, MG_TRANSPORT_LOCAL = 2, MG_TRANSPORT_PEER = 3 };
#define MG_PEER_BLOB_BYTES 128

/* bottom_mode.  AUTO: a bottom level of <= 8 bricks without ghosts runs all its sweeps in one
 * CTA (resident), one of 9-64 bricks in one thread-block cluster of up to 16 CTAs (bottom_cluster.cu,
 * neighbours through distributed shared memory; also the replicated global bottom of a
 * decomposition), otherwise per-sweep launches.  CLUSTER (opt-in): the deepest
 * levels without ghosts that fit (<= 64 bricks per level, <= 200 KB of fields) run as ONE
 * 8-CTA cluster launch (coarse.cu: pre-sweeps, restriction, initZero, bottom, interpolation,
 * post-sweeps of those levels); measured no faster than graph-replayed launches (DESIGN.md
 * §7.3).  All modes are bitwise identical. */
enum { MG_BOTTOM_AUTO = 0, MG_BOTTOM_SWEEPS = 1, MG_BOTTOM_RESIDENT = 2, MG_BOTTOM_CLUSTER = 3, MG_BOTTOM_GRID = 4 };

typedef struct {
  int32_t n_local[3];            /* cells per rank per axis (x,y,z); each divisible by 8*2^(num_levels-1) */
  int32_t proc_grid[3];          /* ranks per axis; product == world_size; rank = cx + px*(cy + py*cz) */
  int32_t num_levels;            /* >= 1; levels 0..L-1, bottom solve on L-1 (reading A2) */
  int32_t pre_smooths;           /* paper: 12 */
  int32_t post_smooths;          /* paper: 12 */
  int32_t bottom_smooths;        /* paper: 100 */
  int32_t ca_period[MG_MAX_LEVELS]; /* sweeps per x-exchange per level, 1..8; 0 = auto: 2 at level 0
                                       and 8 below on the copy transports (local, peer: an exchange
                                       copies only the ghost cells within the period of the owned
                                       box), 8 everywhere over NCCL (whole bricks) */
  int32_t fusion[MG_MAX_LEVELS];    /* MG_FUSION_*; 0 = auto */
  int32_t ghost_mode;            /* MG_GHOST_* */
  int32_t transport;             /* MG_TRANSPORT_*.  Between processes (world_size > 1): auto / PEER = every
                                    rank maps the others' workspaces (CUDA IPC, mg_peer_blob /
                                    mg_peer_connect) and one device kernel per exchange copies the ghost
                                    runs out of the neighbours' fields, ordered by device-side flags (no
                                    NCCL; the norm's max and the replicated bottom's gather likewise);
                                    NCCL = grouped ncclSend/ncclRecv + ncclAllReduce (needs nccl_id).  One
                                    rank: local device copies, or NCCL self send/recv with
                                    MG_TRANSPORT_NCCL (nccl_id may then be NULL).  On the copy
                                    transports (PEER, LOCAL) a level with a pencil plan over its owned
                                    bricks (periodic box, constant coefficients, <= 8 ranks) runs NO
                                    x exchange kernel: its two-sweep passes stage the ghost bricks' x
                                    straight from the owners' fields (the exchange fused into the pass,
                                    after a flag handshake between processes; mg_exchange_fused) and
                                    take CA period 2 by default */
  int32_t use_graph;             /* 1 = replay the V-cycle as one CUDA graph (default 1) */
  int32_t bottom_mode;           /* MG_BOTTOM_* (resident = one CTA runs all bottom sweeps in smem,
                                    cluster = the coarse levels run in one cluster launch, grid = the
                                    ghost-free levels of <= 512 bricks run in one launch of one CTA per
                                    SM with grid barriers between dependent steps) */
  int32_t overlap;               /* 1 = sweep interior bricks while the exchange is in flight
                                    (single-sweep levels; the two-sweep pencil passes only with
                                    MG_PENCIL_OVERLAP=1, measured slower by default: DESIGN.md §9) */
  int32_t sweep_kernel;          /* 0 = auto (streaming column kernel on levels >= 16384 bricks),
                                    1 = one-brick-per-CTA kernel only, 2 = streaming kernel on every level */
  int32_t temporal_blocking;     /* two Jacobi sweeps per HBM pass (bit-identical): 3 = over 2x2-brick pencils
                                    (sweep2p.cu, the default), 1 = one-brick CTA item streams (sweep2.cu; also
                                    the fallback of 3 on ranges that do not tile into pencils), 0 = one sweep
                                    per pass; anything else is refused */
  int32_t smoother;              /* 0 = damped Jacobi (the paper); 1 = Chebyshev: the pre / post
                                    sweeps of a level take the steps h^2/(12 nu_k) at the Chebyshev nodes nu_k of
                                    [1/cheby_ratio, 1] (variant N4, reading A19); 2 = red-black
                                    Gauss-Seidel: each pre / post sweep is a red then a black half-sweep with step
                                    h^2/6, colour (i+j+k) mod 2, r from the last (black) half-sweep (reading A20).
                                    The bottom stays damped Jacobi. */
  int32_t cheby_ratio;           /* smoothing interval mu in [mu_max/cheby_ratio, mu_max]; 0 => 6 */
  int32_t launch_pdl;            /* programmatic dependent launch of every library kernel: 0 = auto (on),
                                    1 = on, 2 = off.  A kernel's CTAs may be scheduled while the previous
                                    kernel of the stream drains; each waits for it before touching memory
                                    (griddepcontrol), so results are bitwise unchanged */
  int32_t bottom_solver;         /* 0 = `bottom_smooths` damped-Jacobi smooths (the paper);
                                    1 = `bottom_smooths` conjugate-gradient iterations from x = 0 with a
                                    fixed-order dot product (variant N4, reading A21; needs a
                                    coarsest grid of <= 8 bricks, globally when decomposed) */
  int32_t bc;                    /* MG_BC_* (variant, reading A22): not with smoother 2 (its colours do not
                                    commute with the reflection) or bottom_solver 1 (periodic null space) */
  int32_t var_coef;              /* 1 = variable coefficients A x = div(c grad x) (variant, reading A23):
                                    the cell coefficients are set with mg_set_coefficients before the first
                                    V-cycle; the one-brick kernels run every level; smoother 0 and
                                    bottom_solver 0 only */
  int32_t brick_edge;            /* 0 or 8 = 8^3 bricks (the paper's NVIDIA / AMD choice); 4 = 4^3
                                    bricks (the paper's Sunspot choice, variant N4): the one-brick kernel
                                    family of generic.cu, per-sweep bottoms, ca_period <= 4, n_local a
                                    multiple of 4*2^(num_levels-1) */
  double h0;                     /* finest spacing; <= 0 => 1 / max_d(global N_d) (reading A7) */
} mg_params;

typedef struct mg_ctx mg_ctx;      /* one rank (process, GPU) */
typedef struct mg_group mg_group;  /* several ranks driven by one process on one GPU (loopback) */
typedef struct mg_layout mg_layout;/* host-only layout tables (no GPU needed) */

/* Fill *p with the paper's defaults (12/12/100, L=6, 1 rank, auto everything). */
void mg_params_default(mg_params* p);

/* Bytes of device workspace one rank needs (fields of every level + tables). */
mg_status mg_workspace_bytes(const mg_params* p, int32_t rank, int32_t world_size, size_t* out_bytes);

/* rank 0 creates the NCCL unique id (128 bytes) and broadcasts it itself
 * (torch.distributed in the Python harness). */
mg_status mg_nccl_unique_id(uint8_t out_id[128]);

/* Collective.  nccl_id may be NULL when world_size == 1 and no NCCL is wanted.
 * cuda_stream: the cudaStream_t every call enqueues on (NULL = legacy default).
 * workspace: device memory of >= mg_workspace_bytes, 256-byte aligned. */
mg_status mg_setup(const mg_params* p, int32_t rank, int32_t world_size, const uint8_t* nccl_id,
                   int32_t device, void* cuda_stream, void* workspace, size_t ws_bytes, mg_ctx** out);

/* Peer-memory transport (MG_TRANSPORT_PEER / AUTO with world_size > 1), after mg_setup and before
 * the first exchange: every rank writes its blob (the CUDA IPC handle of the allocation holding its
 * workspace, the workspace's offset in it, rank, world) with mg_peer_blob, the caller all-gathers
 * the blobs in rank order (torch.distributed in the Python harness) and passes all of them
 * (world_size * MG_PEER_BLOB_BYTES bytes) to mg_peer_connect, which maps the other workspaces
 * (cudaIpcOpenMemHandle; closed by mg_destroy) and builds the exchange tables.  Every rank must use
 * the same parameters (same workspace layout).  The workspace must come from cudaMalloc (e.g. the
 * default torch caching allocator), not from a VMM / expandable-segments allocation.  Exchanges,
 * norms and V-cycles before mg_peer_connect fail with MG_ERR_STATE. */
mg_status mg_peer_blob(mg_ctx* c, uint8_t* out_blob);
mg_status mg_peer_connect(mg_ctx* c, const uint8_t* all_blobs);

/* Right-hand side b of level 0, local lexicographic, device / host.
 * mg_set_rhs_host does not block the host: the upload runs on an internal copy
 * stream into one of two staging fields and overlaps work already enqueued on
 * the context's stream (e.g. the V-cycle of the previous right-hand side); the
 * conversion into bricks is ordered on the context's stream.  b_host must not
 * be modified until the next synchronising call returns; pinned memory gives a
 * truly asynchronous copy.  The first host-buffer call (mg_set_rhs_host or
 * mg_get_solution_host) allocates the two level-0 staging fields with cudaMalloc
 * (library-owned, freed by mg_destroy; not part of mg_workspace_bytes). */
mg_status mg_set_rhs(mg_ctx* c, const double* b_dev);
mg_status mg_set_rhs_host(mg_ctx* c, const double* b_host);
/* Variable-coefficient variant (params var_coef = 1, reading A23): the cell coefficients
 * c > 0 of level 0, local lexicographic like b (device pointer, 16-byte aligned, caller-owned, read
 * during the call's stream work only).  Coarse levels take the restriction of c (volume average, the
 * restriction operator of P:L69, L120); ghost bricks are exchanged (reflected evenly on domain faces).
 * Must be called before the first V-cycle / norm (MG_ERR_STATE otherwise); MG_ERR_STATE on a context
 * with var_coef = 0.  Loopback groups: mg_group_set_coefficients per rank, then
 * mg_group_commit_coefficients. */
mg_status mg_set_coefficients(mg_ctx* c, const double* c_dev);
/* Initial guess; NULL => x = 0 (reading A9). */
mg_status mg_set_solution(mg_ctx* c, const double* x_dev);
mg_status mg_get_solution(mg_ctx* c, double* x_dev);
mg_status mg_get_solution_host(mg_ctx* c, double* x_host);

/* One V-cycle (Alg 2).  Collective, stream-ordered, asynchronous. */
mg_status mg_vcycle(mg_ctx* c);

/* Global max_p |b_p - (A x)_p| at level 0 with a fresh applyOp (Alg 1
 * "maxNormRes").  Collective; synchronises the stream. */
mg_status mg_residual_norm(mg_ctx* c, double* out_max_abs);
/* The same split in two: _async enqueues the norm (and its 8-byte read-back)
 * on the stream and returns; _wait blocks until it is done and returns the
 * value.  At most one norm may be pending (MG_ERR_STATE otherwise).
 * mg_residual_norm == _async + _wait. */
mg_status mg_residual_norm_async(mg_ctx* c);
mg_status mg_residual_norm_wait(mg_ctx* c, double* out_max_abs);

/* Alg 1: while norm > tol and cycles < max_cycles: V-cycle.
 * Returns MG_OK when the final norm is <= tol, MG_NOT_CONVERGED (1) if the cap was
 * hit or the norm is not finite (a NaN stops the loop at once; mg_last_error says
 * "not finite"). */
mg_status mg_solve(mg_ctx* c, double tol, int32_t max_cycles, int32_t* cycles_done, double* final_norm);

/* Per (level, op) device times in ms of the last mg_vcycle run with
 * timing enabled (mg_set_timing(c, 1) disables graph replay and brackets each
 * op with CUDA events).  out[l*MG_NUM_OPS + op], op: MG_OP_*.  cap = capacity
 * in doubles.  Also returns counts of kernel launches in out_launches if not NULL. */
enum { MG_OP_SWEEP = 0, MG_OP_APPLYOP = 1, MG_OP_SMOOTH = 2, MG_OP_RESTRICT = 3, MG_OP_INTERP = 4,
       MG_OP_ZERO = 5, MG_OP_EXCHANGE = 6, MG_OP_BOTTOM = 7, MG_NUM_OPS = 8 };
mg_status mg_set_timing(mg_ctx* c, int32_t enabled);
mg_status mg_get_timings(mg_ctx* c, double* out, int32_t cap);
/* The individual timed ops since mg_set_timing, in issue order: slots[i] =
 * level*MG_NUM_OPS + op, ms[i] = its device time.  Writes min(cap, *count)
 * records; *count = number available (call with cap = 0 to size the buffers).
 * Input for the latency/throughput fits t = alpha + x/beta (tools/model_fit.py). */
mg_status mg_get_timing_records(mg_ctx* c, int32_t* slots, double* ms, int32_t cap, int32_t* count);

/* Number of kernel launches (own kernels) one mg_vcycle issues. */
mg_status mg_vcycle_launches(mg_ctx* c, int64_t* out);

/* Exchange statistics: bytes this rank sends per V-cycle and message count. */
mg_status mg_exchange_stats(mg_ctx* c, int64_t* bytes_per_cycle, int64_t* messages_per_cycle);

/* Per level l < cap of the V-cycle mg_vcycle would run next: exchanges[l] = ghost exchanges (x before
 * a sweep, b after the restriction), bytes[l] = bytes this rank sends in one exchange of the level
 * (0 without a ghost shell; on the copy transports only the ghost cells within the level's CA period
 * of the owned box, whole bricks over NCCL).  Host-only, no device work. */
mg_status mg_exchange_plan(mg_ctx* c, int32_t cap, int64_t* exchanges, int64_t* bytes);
/* Per level l < cap: how many of mg_exchange_plan's exchanges[l] are fused into the pencil pass that
 * follows them (DESIGN.md §9 "fused exchange"): the pass stages its ghost bricks' x straight from the
 * owners' fields (peer memory between processes, the other contexts of a loopback group, or the own
 * field for a one-rank self-exchange) instead of a separate exchange kernel; between processes a
 * flag handshake kernel (no data) precedes the pass.  Only levels with a pencil plan over the owned
 * range, a periodic box and constant coefficients, on the copy transports (not NCCL); off with
 * MG_NO_FUSED_EXCH=1.  Host-only, no device work. */
mg_status mg_exchange_fused(mg_ctx* c, int32_t cap, int64_t* fused);
/* Device time of one ghost exchange of x at `level` (the V-cycle's transport: NCCL grouped
 * send/recv of the brick runs, or the local copy kernel), averaged over `reps` back-to-back
 * exchanges on the context's stream after one warm-up exchange (CUDA events; synchronises).
 * Collective when the transport is NCCL.  0 for a level without a ghost shell.  Input of the
 * bench's exchange block and of the exchange latency / bandwidth fit t = alpha + bytes / beta. */
mg_status mg_exchange_time(mg_ctx* c, int32_t level, int32_t reps, double* ms_per_exchange);
mg_status mg_destroy(mg_ctx* c);

/* Thread-local description of the last error (never NULL). */
const char* mg_last_error(void);

/* ----------------------------------------------------------------------------
 * Per-operator entry points (tests / per-op measurement).  They act on the
 * context's level-l fields in place; "field" is MG_FIELD_*.  Level fields are
 * read/written in local lexicographic order (device pointers).
 * -------------------------------------------------------------------------- */
enum { MG_FIELD_X = 0, MG_FIELD_B = 1, MG_FIELD_R = 2 };
mg_status mg_level_set(mg_ctx* c, int32_t level, int32_t field, const double* src_dev);
mg_status mg_level_get(mg_ctx* c, int32_t level, int32_t field, double* dst_dev);
/* n sweeps of smooth+residual at level l with variant `fusion`
 * (MG_FUSION_PAPER: applyOp then smooth+residual kernels; otherwise the fused
 * sweep); write_r = 1 writes r of the last sweep.  Exchanges as the ghost
 * rule requires. */
mg_status mg_op_smooth(mg_ctx* c, int32_t level, int32_t n, int32_t write_r, int32_t fusion);
/* restriction: b_{l+1} = R r_l, fine level l. */
mg_status mg_op_restrict(mg_ctx* c, int32_t level);
/* interpolation+increment: x_l += I x_{l+1}, fine level l. */
mg_status mg_op_interp(mg_ctx* c, int32_t level);
/* bottom solve at level l: n Jacobi sweeps with the configured bottom mode. */
mg_status mg_op_bottom(mg_ctx* c, int32_t level, int32_t n);
mg_status mg_sync(mg_ctx* c);

/* ----------------------------------------------------------------------------
 * Loopback group: world_size ranks in ONE process on ONE device, exchanging
 * ghost bricks through device copies with the same exchange plan the NCCL
 * path uses.  Lets one GPU run (and test) any 3D decomposition.
 * The workspace is world_size * per-rank bytes (mg_workspace_bytes of rank 0).
 * -------------------------------------------------------------------------- */
mg_status mg_group_setup(const mg_params* p, int32_t world_size, int32_t device, void* cuda_stream,
                         void* workspace, size_t ws_bytes, mg_group** out);
mg_status mg_group_ctx(mg_group* g, int32_t rank, mg_ctx** out); /* per-rank view for set/get */
mg_status mg_group_vcycle(mg_group* g);
mg_status mg_group_residual_norm(mg_group* g, double* out_max_abs);
mg_status mg_group_set_rhs(mg_group* g, int32_t rank, const double* b_dev); /* then mg_group_commit_rhs */
mg_status mg_group_commit_rhs(mg_group* g);
mg_status mg_group_set_coefficients(mg_group* g, int32_t rank, const double* c_dev);
mg_status mg_group_commit_coefficients(mg_group* g); /* exchanges level-0 b ghosts of every rank */
mg_status mg_group_set_solution(mg_group* g, int32_t rank, const double* x_dev);
mg_status mg_group_destroy(mg_group* g);

/* ----------------------------------------------------------------------------
 * Host-only layout queries (no GPU needed; used by the CPU tests).
 * info[0..2] n_local, [3..5] bricks per axis, [6..8] ghost flags,
 * [9] owned, [10] interior, [11] ghost, [12] allocated bricks (incl. zero
 * brick), [13] send runs, [14] recv runs, [15] zero-brick index.
 * adjacency: int32 [stored][8] = W,E,S,N,B,T,self,0 (stored = owned+ghost).
 * coords: int32 [stored][3] extended brick coords (ghost: -1 or nb).
 * parent: int32 [stored] = coarse brick index*8 + octant (-1 if none).
 * plan: int64 [runs][6] = peer, direction(0..26), run index, local brick offset,
 * remote brick offset, brick count.
 * pass plan: the two-sweep (temporal blocking) plan number `idx` of a level (one per swept brick
 * range).  info[0] kind (1 one-brick CTA streams, 2 warp plane streams, 3 2x2-brick pencil chunk
 * streams), [1] b0, [2] b1 (brick range), [3] ints of meta, [4] ints of ctas, [5] part (kind 3
 * on a level with a ghost shell: 0 every unit of the range, 1 the units whose records name no
 * ghost brick -- swept while an exchange fills the ghosts --, 2 the others); MG_ERR_INVALID_ARG
 * if idx is past the last plan.  meta / ctas (may be NULL: sizes only) receive copies of the
 * tables the kernel reads; for kind 3, meta = int32 [chunks][20] = code (type << 1 | half; type 0
 * range, 1 warm-up, 2 cool-down), ids of b00, b10, b01, b11, W0, W1, E0, E1, S0, S1, N0, N1, SW,
 * NW, SE, NE, parent of b00, 0, 0; ctas = int32 [ctas][2] = first chunk, chunk count.
 * -------------------------------------------------------------------------- */
mg_status mg_layout_create(const mg_params* p, int32_t rank, int32_t world_size, mg_layout** out);
mg_status mg_layout_level_info(const mg_layout* lay, int32_t level, int64_t info[16]);
mg_status mg_layout_adjacency(const mg_layout* lay, int32_t level, int32_t* out);
mg_status mg_layout_coords(const mg_layout* lay, int32_t level, int32_t* out);
mg_status mg_layout_parent(const mg_layout* lay, int32_t level, int32_t* out);
mg_status mg_layout_plan(const mg_layout* lay, int32_t level, int32_t which /*0 send,1 recv*/, int64_t* out);
/* Mirror table of a level (non-periodic bc, reading A22): *count entries of int32 (ghost brick,
 * source brick, mask of the reflected axes, bit a = axis a) into out (3 * count int32, or NULL to
 * query the count).  The ghost brick's cell (i,j,k) is the source's cell with i -> 7-i etc. on the
 * reflected axes, negated once per reflection for Dirichlet. */
mg_status mg_layout_mirror(const mg_layout* lay, int32_t level, int64_t* count, int32_t* out);
/* The exchange fused into the level's pencil passes: per chunk record of the owned pencil
 * plan and entry e = 0..15 (the record's brick ids 1..16), -1 for a local brick or (rank << 24) | the
 * brick of rank's field that the ghost brick mirrors -- the table the pass stages its ghost x from.
 * *count = chunks * 16, 0 if the level does not fuse its exchanges; out (count int32) may be NULL. */
mg_status mg_layout_fused_pid(const mg_layout* lay, int32_t level, int64_t* count, int32_t* out);
mg_status mg_layout_pass_plan(const mg_layout* lay, int32_t level, int32_t idx, int64_t info[6], int32_t* meta,
                              int32_t* ctas);
/* Replicated bottom (the coarsest level has a ghost shell and the global coarsest grid <= 64
 * bricks): info[0] = global coarsest bricks (0: not replicated), info[1] = this rank's owned
 * coarsest bricks; gb_src int32 [info[0]] = rank * info[1] + owned index of the brick each global
 * brick is gathered from (the all-gather's rank-major order), gb_mine int32 [info[1]] = the global
 * brick of each owned brick, gb_adj int32 [info[0]][8] = the global level's adjacency (periodic
 * wrap).  Any array may be NULL. */
mg_status mg_layout_repl(const mg_layout* lay, int64_t info[2], int32_t* gb_src, int32_t* gb_mine, int32_t* gb_adj);
/* Kernel launches of this library one V-cycle issues from a fresh context's state, the count
 * mg_vcycle_launches gives on a GPU (exchanges: one copy kernel each if local_exchange, none of
 * ours over NCCL). */
mg_status mg_layout_vcycle_launches(const mg_layout* lay, int32_t local_exchange, int64_t* out);
/* mg_exchange_plan for the first V-cycle of a fresh context with this layout (host-only): per level
 * l < cap, the exchanges of the cycle and the bytes one exchange of x sends (the copy transports move
 * only the ghost cells within the level's CA period of the owned box; NCCL whole bricks). */
mg_status mg_layout_exchange_plan(const mg_layout* lay, int32_t cap, int64_t* exchanges, int64_t* bytes);
mg_status mg_layout_destroy(mg_layout* lay);

#ifdef __cplusplus
}
#endif
#endif /* MG_B200_H */
