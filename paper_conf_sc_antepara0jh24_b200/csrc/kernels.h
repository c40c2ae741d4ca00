// kernels.h -- launchers for the sm_100a brick kernels (kernels.cu).
#pragma once

#include <cuda.h>  // CUtensorMap (types only; the driver entry point is fetched at run time)
#include <cuda_runtime.h>

#include <cstdint>

namespace mgb {

// Level constants: alpha = -6/h^2, beta = 1/h^2, gamma = h^2/12.
struct Coeffs {
  double alpha, beta, gamma;
};
Coeffs level_coeffs(double h);

// Fused sweep flags (template specialisations in kernels.cu)
enum SweepFlags : unsigned {
  SW_WRITE_R = 1u,     // write r = b - Ax (smooth+residual)
  SW_RESTRICT = 2u,    // write b_coarse = R r into the parent octant instead of r
  SW_INTERP = 4u,      // read x as x_fine + x_coarse(parent) (interpolation+increment fused)
  SW_ZERO_X = 8u,      // x == 0 (initZero folded into the first coarse sweep)
  SW_NO_SMOOTH = 16u,  // do not write x' (restriction-only last sweep is never used; kept for tests)
  SW_COLOUR = 32u,     // two-sweep kernel: red-black half-sweeps (colour masks compiled in only here)
  SW_VARCOEF = 64u,    // one-brick kernel: variable coefficients div(c grad x) (reading A23), SweepArgs::cf
  SW_NORM = 128u,      // column kernel: no stores, max |b - Ax| into SweepArgs::acc (maxNormRes)
  SW_PEER = 256u,      // pencil kernel: x of ghost bricks read from their owners' fields (fused exchange)
};

struct SweepArgs {
  const double* x;       // input x (brick layout)
  double* xo;            // output x'
  const double* b;
  double* r;
  const int32_t* adj;    // [brick][8]
  const int32_t* parent; // fine brick -> coarse brick*8 + octant
  double* bc;            // coarse b (SW_RESTRICT)
  const double* xc;      // coarse x (SW_INTERP)
  int64_t brick0, nbricks;
  Coeffs c;          // c.gamma: the step of the (first) sweep
  double gamma2;     // two-sweep kernels: the step of the second sweep
  int colour = -1;   // red-black half-sweep (GSRB variant): update only cells with (i+j+k) mod 2 == colour,
  int colour2 = -1;  // keep the others (r still on every cell); -1 = every cell.  colour2: second sweep
  const double* cf = nullptr;  // SW_VARCOEF: cell coefficients c (brick layout, ghosts valid)
  double vc_g = 0.0;           // SW_VARCOEF: 0.5 * h * h (gamma_p = vc_g / sum of the face coefficients)
  int E = 8;                   // brick edge (8; 4: the generic kernels of generic.cu)
  unsigned long long* acc = nullptr;  // SW_NORM: atomicMax target (uint64 bits of a non-negative double)
};

cudaError_t launch_sweep(const SweepArgs& a, unsigned flags, cudaStream_t s);

// Streaming (column) sweep: one CTA per segment of a z-column of bricks;
// bricks of x and b arrive by TMA bulk copies into a shared-memory ring.
struct ColArgs {
  const int32_t* bricks;  // brick ids, segment after segment
  const int4* side;       // W,E,S,N neighbour ids per entry of `bricks`
  const int2* segs;       // (offset, count) per segment, count <= 16
  int64_t nseg;
};
// TMA tensor maps over one x field seen as [n_alloc*8 planes][8 j][8 i] doubles:
// `we` boxes {2 i, 8 j, 8 k} (the W / E face columns), `sn` boxes {8 i, 1 j, 8 k}
// (the S / N face rows).  One tensor copy per face per brick, no LSU gathers.
struct FaceMaps {
  CUtensorMap we;
  CUtensorMap sn;
};
// Encodes the two maps for the field at `x` with `n_alloc` bricks (driver entry
// point obtained through the runtime; no libcuda link).
cudaError_t encode_face_maps(const double* x, int64_t n_alloc, FaceMaps* out);
// One TMA tensor map over a brick field seen as [n_alloc*8 planes][8 j][8 i]
// doubles with the given box {i, j, planes}.
cudaError_t encode_box_map(const double* base, int64_t n_alloc, const unsigned box[3], CUtensorMap* out,
                           bool swizzle64 = false);  // swizzle64: 16-byte chunk c of row r lands at chunk c ^ ((r >> 1) & 3)

// Two-sweep (temporally blocked) streaming kernel, sweep2.cu.
struct PairArgs {
  int kind;             // 1: CTA item streams (sweep2.cu), 3: 2x2-brick pencil chunk streams (sweep2p.cu)
  const int32_t* meta;  // kind 1: [items][11] id, flags, W,E,S,N, SW,NW,SE,NE, parent;
                        // kind 3: [chunks][20] chunk records (mg_internal.h kPenRec)
  const int2* ctas;     // (first item / chunk, count) per CTA
  int64_t nctas;
  unsigned long long* trace = nullptr;  // sweep2p measurement (MG_PEN_TRACE): per CTA (start, end) globaltimer
  // SW_PEER (the exchange fused into the pencil pass): pid[chunk][e] for the x copies of
  // record entries e = 0..15 (ids 1..16): -1 = the local brick, else (rank << 24) | the brick of rank's
  // field that the ghost brick mirrors, staged through rank's x tensor maps rmaps[3 rank + 0..2] (xwe,
  // xsn, xcor) or, for a whole half brick, from PairMaps::rbase[rank]; b stays local (its ghosts are
  // exchanged once per level)
  const int32_t* pid = nullptr;
  const CUtensorMap* rmaps = nullptr;
};
struct PairMaps {
  CUtensorMap xwe;   // x boxes {2,8,8}: W (i=6,7) / E (i=0,1) face slabs
  CUtensorMap xsn;   // x boxes {8,2,8}: S (j=6,7) / N (j=0,1) face slabs
  CUtensorMap xcor;  // x boxes {2,1,8}: the four diagonal-corner columns
  CUtensorMap bwe;   // b boxes {2,8,8}
  CUtensorMap bsn;   // b boxes {8,1,8}
  const double* rbase[8] = {};  // SW_PEER (pencil kernel): x base pointer of the src buffer of rank r
};
cudaError_t encode_pair_maps(const double* x, const double* b, int64_t n_alloc, PairMaps* out);
// flags apply to the SECOND sweep of the pair: plain, +r, +restriction
bool pair_supports(unsigned flags);
cudaError_t launch_sweep2(const SweepArgs& a, const PairArgs& pa, const PairMaps& pm, unsigned flags,
                          cudaStream_t s);
cudaError_t pair_kernels_init();
// 2x2-brick pencil two-sweep kernel (sweep2p.cu): maps with 4-plane boxes ({2,8,4}, {8,2,4},
// {2,1,4}; b {2,8,4}, {8,1,4}) in the PairMaps fields
cudaError_t encode_pencil_maps(const double* x, const double* b, int64_t n_alloc, PairMaps* out);
bool pencil_supports(unsigned flags);
// early: launch with PDL (only after a one-CTA peer handshake, which triggers once the previous
// kernel is complete: the pass's CTAs land on a drained GPU and wait for the handshake in pdl_wait)
cudaError_t launch_sweep2p(const SweepArgs& a, const PairArgs& pa, const PairMaps& pm, unsigned flags,
                           cudaStream_t s, bool early = false);
cudaError_t pencil_kernels_init();

// true if the streaming kernel implements `flags` (plain, +r, +restriction)
bool col_supports(unsigned flags);
// flags: plain / +r / +restriction, or SW_NORM; | SW_VARCOEF with fmc = the face maps over SweepArgs::cf
cudaError_t launch_sweep_col(const SweepArgs& a, const ColArgs& c, const FaceMaps& fm, unsigned flags,
                             cudaStream_t s, const FaceMaps* fmc = nullptr);
// applyOp (paper kernel set): Ax = alpha x + beta sum6
cudaError_t launch_apply_op(const double* x, double* Ax, const int32_t* adj, int64_t brick0, int64_t nbricks,
                            Coeffs c, cudaStream_t s, int E = 8);
// smooth(+residual) pointwise (paper kernel set): x += gamma (Ax - b); r = b - Ax
cudaError_t launch_smooth(double* x, const double* Ax, const double* b, double* r, int64_t brick0, int64_t nbricks,
                          Coeffs c, bool write_r, cudaStream_t s, int colour = -1, int E = 8);
// restriction over fine bricks [0, nfine): bc[parent octant] = avg8(r)
cudaError_t launch_restrict(const double* r, double* bc, const int32_t* parent, int64_t nfine, cudaStream_t s,
                            int E = 8);
// interpolation+increment over fine bricks [0, nfine): x += xc(parent)
cudaError_t launch_interp(double* x, const double* xc, const int32_t* parent, int64_t nfine, cudaStream_t s,
                          int E = 8);
// initZero over bricks [brick0, brick0+n)
cudaError_t launch_zero(double* x, int64_t brick0, int64_t nbricks, cudaStream_t s, int E = 8);
// max |b - Ax| over bricks [0, n) -> atomicMax on *acc (uint64 bits of a non-negative double)
cudaError_t launch_norm(const double* x, const double* b, const int32_t* adj, int64_t nbricks, Coeffs c,
                        unsigned long long* acc, cudaStream_t s, const double* cf = nullptr, int E = 8);
// resident bottom solve: all `nbricks` (<= kResidentMaxBricks, no ghosts) in one CTA's shared memory
constexpr int kResidentMaxBricks = 8;
cudaError_t launch_bottom_resident(const double* x, double* xo, const double* b, const int32_t* adj, int nbricks,
                                   int sweeps, bool zero_x, Coeffs c, cudaStream_t s,
                                   double msign = 0.0);
// cluster-resident bottom solve (bottom_cluster.cu): 9 .. kClusterBottomMaxBricks bricks (no ghosts)
// over ceil(nbricks / 8) CTAs of one cluster, the resident kernel's arithmetic and arguments
constexpr int kClusterBottomMaxBricks = 64;
cudaError_t launch_bottom_cluster(const double* x, double* xo, const double* b, const int32_t* adj, int nbricks,
                                  int sweeps, bool zero_x, Coeffs c, cudaStream_t s, double msign = 0.0);
cudaError_t bottom_cluster_init();
// the bottom kernel for a level of nbricks: resident (<= 8), cluster (<= 64; MG_NO_CLUSTER_BOTTOM=1 for A/B)
bool cluster_bottom_enabled();
bool cluster_bottom_small();
// layout conversion (not part of the V-cycle): lexicographic local <-> bricks [0, nowned)
cudaError_t launch_lex_to_brick(const double* lex, double* bricks, const int32_t* coord, int64_t nowned, int nx,
                                int ny, cudaStream_t s, int E = 8);
cudaError_t launch_brick_to_lex(const double* bricks, double* lex, const int32_t* coord, int64_t nowned, int nx,
                                int ny, cudaStream_t s, int E = 8);
// Local (self / loopback) ghost exchange: every run of one exchange in ONE launch instead of one
// cudaMemcpyAsync per run (n doubles from src to dst, both 16-byte aligned, n even).  box != 0: the
// run is n / E^3 bricks of which only the cells of a sub-box are copied (copyrun.cuh copy_box).
struct CopyRun {
  const double* src;
  double* dst;
  int64_t n;
  int32_t box = 0;
  int32_t pad_ = 0;
};
cudaError_t launch_copy_runs(const CopyRun* runs, int nruns, int64_t max_n, cudaStream_t s);
// Mirror exchange (non-periodic bc, reading A22): for each entry (dst, src, mask) of the
// int32[n][3] table, brick dst = sign^popcount(mask) x brick src with the cells reversed on the axes
// of mask (bit a: axis a).  sign = -1 (Dirichlet) or +1 (Neumann).
cudaError_t launch_mirror(double* f, const int32_t* table, int n, double sign, cudaStream_t s, int E = 8);
// generic.cu: the same operations for a brick edge E != 8 (E = 4; "4x4x4 on Sunspot").
// mode 0 sweep (flags), 1 applyOp (x -> xo), 2 norm (atomicMax on *acc)
cudaError_t launch_gsweep(const SweepArgs& a, unsigned flags, int mode, unsigned long long* acc, cudaStream_t s);
cudaError_t launch_grestrict(const double* r, double* bc, const int32_t* parent, int64_t nfine, int E, cudaStream_t s);
cudaError_t launch_ginterp(double* x, const double* xc, const int32_t* parent, int64_t nfine, int E, cudaStream_t s);
cudaError_t launch_glex(const double* src, double* dst, const int32_t* coord, int64_t nowned, int nx, int ny,
                        int dir, int E, cudaStream_t s);
cudaError_t launch_gmirror(double* f, const int32_t* table, int n, double sign, int E, cudaStream_t s);
cudaError_t launch_gsmooth(double* x, const double* Ax, const double* b, double* r, int64_t brick0, int64_t nbricks,
                           Coeffs c, bool write_r, int colour, int E, cudaStream_t s);
// Exchange between processes over peer memory (peer.cu): the copy runs read other ranks' fields
// through CUDA IPC mappings; device-side flags order them (ready / done per epoch, see peer.cu).
constexpr int kPeerSlotU64 = 16;  // one flag per 128-byte slot
struct PeerSync {
  unsigned long long* flags;          // this rank's [world][2] slots (ready, done), kPeerSlotU64 apart
  unsigned long long* const* remote;  // device [world * 2]: address of THIS rank's slot (kind) at rank n
  const int* part;                    // device: the participant ranks (never this rank)
  int npart;
  unsigned long long* epoch;          // this rank's epoch counter (advanced by every peer kernel)
  unsigned* done;                     // CTA completion counter (zero between kernels)
  const CopyRun* dummy_run;           // a zero-length run (a rank without runs still takes part)
};
cudaError_t launch_peer_copy(const CopyRun* runs, int nruns, int64_t max_n, const PeerSync& s, cudaStream_t st);
// ready(e) to / from every participant, no copy (the pencil passes with SW_PEER read the neighbours' x)
cudaError_t launch_peer_handshake(const PeerSync& s, cudaStream_t st);
// global max of the uint64 bits at *acc over the participants (+ this rank): vals = this rank's
// [world] value slots, remote_vals[n] = rank n's value slots
cudaError_t launch_peer_allmax(unsigned long long* acc, const PeerSync& s, unsigned long long* const* remote_vals,
                               unsigned long long* vals, int me, int world, cudaStream_t st);
// Resident coarse solver (coarse.cu): levels l0 .. L-1 of one V-cycle (pre-sweeps + fused
// restriction, initZero, bottom, interpolation, post-sweeps) in one launch of a cluster of
// kCoarseCtas CTAs holding every field of those levels in shared memory.  No ghosts.
constexpr int kCoarseCtas = 8;
constexpr int kCoarseThreads = 512;
constexpr int kCoarseMaxLevels = 8;
constexpr size_t kCoarseMaxSmem = 200 * 1024;
constexpr int kCoarseMaxCheb = 32;  // Chebyshev smoother: pre / post sweeps the cluster solve supports
struct CoarseLevel {
  int nb;                 // bricks (owned == stored: no ghosts)
  const int32_t* adj;     // [nb][8]
  const int32_t* parent;  // [nb] coarse brick * 8 + octant (levels < last)
  Coeffs c;               // c.gamma: damped Jacobi step (bottom, and pre / post when cheb == 0)
  double h;
};
struct CoarseArgs {
  int nlev;  // levels l0 .. l0 + nlev - 1; the last one is the bottom
  CoarseLevel lv[kCoarseMaxLevels];
  const double* b0;  // b of level l0 (restricted by the level above)
  double* x0;        // out: x of level l0 after its post-sweeps
  int pre, post, bottom;
  int cheb;                                          // 1: pre / post steps h^2 / (12 nu)
  double nu_pre[kCoarseMaxCheb], nu_post[kCoarseMaxCheb];  // Chebyshev nodes in sweep order (host-computed)
};
size_t coarse_smem_bytes(const CoarseArgs& a);
// Grid-resident coarse solver (coarse_grid.cu): the same levels l0 .. L-1 in one launch of one
// kGridCoarseThreads-thread CTA per SM (cooperative: all co-resident), fields in the level buffers,
// a grid barrier between dependent steps; the bottom (<= kResidentMaxBricks bricks) in CTA 0.
// x of every level starts at 0; x of level l0 ends in lv[0].x[0].  No ghosts.
constexpr int kGridCoarseThreads = 1024;
constexpr int64_t kGridCoarseMaxBricks = 512;  // largest level handed to it (512^3: levels 3 .. 5; measured)
struct GridLevel {
  int64_t nb;             // bricks (owned == stored: no ghosts)
  const int32_t* adj;     // [nb][8]
  const int32_t* parent;  // [nb] coarse brick * 8 + octant (levels < last)
  double* x[2];           // ping-pong x (x[0] holds x at entry and, for level l0, at exit)
  double* b;              // b (level l0: restricted by the level above; deeper: written here)
  Coeffs c;
  double h;
};
struct GridCoarseArgs {
  int nlev;
  GridLevel lv[kCoarseMaxLevels];
  int pre, post, bottom;
  int cheb;
  double nu_pre[kCoarseMaxCheb], nu_post[kCoarseMaxCheb];
  unsigned* bar;  // kGridBarWords words of zeroed device memory: arrive count, generation
};
constexpr int kGridBarWords = 16;
cudaError_t launch_coarse_grid(const GridCoarseArgs& a, cudaStream_t s);
cudaError_t coarse_grid_init();

cudaError_t launch_coarse(const CoarseArgs& a, cudaStream_t s);
cudaError_t coarse_kernels_init();
cudaError_t kernels_init();  // one-time attribute setup
// CG bottom solver (cg.cu, variant: reading A21): `iters` CG iterations on A x = b from x = 0 on the
// coarsest level (no ghosts, <= kResidentMaxBricks bricks, one CTA); coord = brick coords [nb][3],
// nx, ny = cells per axis (the lexicographic order of the fixed-order dot product).
cudaError_t launch_bottom_cg(double* xo, const double* b, const int32_t* adj, const int32_t* coord, int nbricks,
                             int nx, int ny, int iters, Coeffs c, cudaStream_t s);
cudaError_t cg_kernels_init();

// Programmatic dependent launch for every kernel the library enqueues: set by the
// API from mg_params.launch_pdl before it enqueues or captures work.  The kernels begin with
// pdl_begin() (ptx.cuh), so the attribute only lets a kernel's CTAs be scheduled while the
// previous kernel of the stream drains; results are unchanged.
extern bool g_launch_pdl;
template <typename... KArgs, typename... Args>
inline cudaError_t launch_ex(bool pdl, void (*k)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t s,
                             Args... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = pdl ? 1 : 0;
  return cudaLaunchKernelEx(&cfg, k, static_cast<KArgs>(args)...);
}
// short kernels: PDL attribute when enabled
template <typename... KArgs, typename... Args>
inline cudaError_t launch_k(void (*k)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t s, Args... args) {
  return launch_ex(g_launch_pdl, k, grid, block, smem, s, args...);
}
// persistent streaming kernels: never launched early (they still wait and trigger, see ptx.cuh)
template <typename... KArgs, typename... Args>
inline cudaError_t launch_plain(void (*k)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t s,
                                Args... args) {
  return launch_ex(false, k, grid, block, smem, s, args...);
}

}  // namespace mgb
