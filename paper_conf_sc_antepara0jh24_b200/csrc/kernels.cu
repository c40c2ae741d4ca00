// kernels.cu -- sm_100a FP64 brick kernels of the GMG V-cycle.
//
// Arithmetic: every operation is a separately rounded
// binary64 op written with __dmul_rn / __dadd_rn / __dsub_rn (no FMA
// contraction; the library is also compiled with --fmad=false), in the
// canonical order of reading A8:
//   sum = ((xW + xE) + (xS + xN)) + (xB + xT)
//   a   = alpha*x + beta*sum                        applyOp
//   r   = b - a                                     residual
//   x'  = x + gamma*(a - b)                         smooth
//   bc  = 0.125*(((r000+r100)+(r010+r110)) + ((r001+r101)+(r011+r111)))  restriction
//   x  += xc(parent)                                interpolation+increment
// so the result is bit-identical to the lexicographic CPU oracle whatever the
// brick order, fusion variant, decomposition or ghost-exchange period.
//
// Brick cell (i,j,k) lives at i + 8j + 64k of its 512-double brick (A16).
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdlib>
#include <cstddef>
#include <cstdint>

#include <cudaTypedefs.h>

#include "kernels.h"
#include "copyrun.cuh"
#include "ptx.cuh"
#include "resident.cuh"

namespace mgb {

bool g_launch_pdl = true;

Coeffs level_coeffs(double h) {
  const double inv = 1.0 / (h * h);
  Coeffs c;
  c.alpha = -6.0 * inv;
  c.beta = inv;
  c.gamma = (h * h) / 12.0;
  return c;
}

// max that propagates NaN (a diverged iterate must not hide in the norm)
__device__ __forceinline__ double nan_max(double a, double b) { return (b > a || b != b) ? b : a; }

// coarse-cell offset of fine cell (i,j,k) of a fine brick with octant o
__device__ __forceinline__ int coarse_off(int oct, int i, int j, int k) {
  const int ox = oct & 1, oy = (oct >> 1) & 1, oz = oct >> 2;
  return (4 * ox + (i >> 1)) + 8 * (4 * oy + (j >> 1)) + 64 * (4 * oz + (k >> 1));
}

// ---------------------------------------------------------------------------
// Fused sweep: one CTA (256 threads) per brick, 2 cells per thread.  The brick
// is staged in shared memory (coalesced 128-bit loads), the six face halos are
// gathered from the neighbour bricks named by the adjacency table, then
//   x' = x + gamma (Ax - b)  and optionally  r = b - Ax  /  b_c = R r.
// Modes: MODE_SWEEP (x', r?), MODE_APPLY (Ax only -> xo), MODE_NORM (max|b-Ax|).
// ---------------------------------------------------------------------------
enum { MODE_SWEEP = 0, MODE_APPLY = 1, MODE_NORM = 2 };

// NT threads per CTA (256: two cells per thread; 128: four, in two cell pairs t and t + 128 -- twice
// the bricks in flight per SM for the same thread count, for the large ranges where the kernel's
// dependent load chain (adjacency -> halos) is the limit)
template <int MODE, unsigned FLAGS, int NT = 256>
__global__ void __launch_bounds__(NT) sweep_kernel(SweepArgs p, unsigned long long* acc) {
  pdl_begin();
  constexpr int HP = 256 / NT;  // cell pairs per thread
  constexpr bool WRITE_R = (FLAGS & SW_WRITE_R) != 0;
  constexpr bool RESTRICT = (FLAGS & SW_RESTRICT) != 0;
  constexpr bool INTERP = (FLAGS & SW_INTERP) != 0;
  constexpr bool ZERO_X = (FLAGS & SW_ZERO_X) != 0;
  constexpr bool VC = (FLAGS & SW_VARCOEF) != 0;  // variable coefficients (reading A23)
  __shared__ __align__(16) double xs[512];
  __shared__ double hw[64], he[64], hs[64], hn[64], hb[64], ht[64];
  __shared__ __align__(16) double rs[RESTRICT ? 512 : 1];
  // VC: the coefficient brick and its six face halos (the face coefficients need c of both cells)
  __shared__ __align__(16) double cs[VC ? 512 : 1];
  __shared__ double ch[VC ? 6 : 1][VC ? 64 : 1];

  const int t = threadIdx.x;
  const int64_t brick = p.brick0 + blockIdx.x;
  const int32_t* adj = p.adj + brick * 8;

  double2 bv[HP];
#pragma unroll
  for (int h = 0; h < HP; ++h)
    bv[h] = MODE != MODE_APPLY ? ld_stream2(p.b + brick * 512 + 2 * (t + NT * h)) : make_double2(0.0, 0.0);

  if (!ZERO_X) {
#pragma unroll
    for (int h = 0; h < HP; ++h) {
      const int tt = t + NT * h, i0 = 2 * (tt & 3), j = (tt >> 2) & 7, k = tt >> 5;
      double2 xv = ldg2(p.x + brick * 512 + 2 * tt);
      if (INTERP) {
        const int pr = __ldg(p.parent + brick);
        if (pr >= 0) {
          const double* xc = p.xc + (int64_t)(pr >> 3) * 512;
          const int co = coarse_off(pr & 7, i0, j, k);  // i0, i0+1 share a coarse cell
          const double cv = __ldg(xc + co);
          xv.x = DADD(xv.x, cv);
          xv.y = DADD(xv.y, cv);
        }
      }
      xs[2 * tt] = xv.x;
      xs[2 * tt + 1] = xv.y;
    }
    // halos: faces W,E,S,N (entries 0..255), B,T (entries 0..127)
#pragma unroll
    for (int h = 0; h < HP; ++h) {
      const int tt = t + NT * h, f = tt >> 6, m = tt & 63;
      const int nb = __ldg(adj + f);
      int ci, cj, ck;
      if (f < 2) {
        ci = f == 0 ? 7 : 0;
        cj = m & 7;
        ck = m >> 3;
      } else {
        ci = m & 7;
        cj = f == 2 ? 7 : 0;
        ck = m >> 3;
      }
      double v = __ldg(p.x + (int64_t)nb * 512 + ci + 8 * cj + 64 * ck);
      if (INTERP) {
        const int pr = __ldg(p.parent + nb);
        if (pr >= 0) v = DADD(v, __ldg(p.xc + (int64_t)(pr >> 3) * 512 + coarse_off(pr & 7, ci, cj, ck)));
      }
      double* hh = f == 0 ? hw : f == 1 ? he : f == 2 ? hs : hn;
      hh[m] = v;
    }
    if (t < 128) {
      const int f = 4 + (t >> 6), m = t & 63;
      const int nb = __ldg(adj + f);
      const int ck = f == 4 ? 7 : 0;
      double v = __ldg(p.x + (int64_t)nb * 512 + m + 64 * ck);
      if (INTERP) {
        const int pr = __ldg(p.parent + nb);
        if (pr >= 0) v = DADD(v, __ldg(p.xc + (int64_t)(pr >> 3) * 512 + coarse_off(pr & 7, m & 7, m >> 3, ck)));
      }
      (f == 4 ? hb : ht)[m] = v;
    }
    __syncthreads();
  }
  if (VC) {
#pragma unroll
    for (int h = 0; h < HP; ++h) {
      const int tt = t + NT * h;
      const double2 cv = ldg2(p.cf + brick * 512 + 2 * tt);
      cs[2 * tt] = cv.x;
      cs[2 * tt + 1] = cv.y;
      const int f = tt >> 6, m = tt & 63;
      const int nb = __ldg(adj + f);
      const int ci = f < 2 ? (f == 0 ? 7 : 0) : (m & 7), cj = f < 2 ? (m & 7) : (f == 2 ? 7 : 0), ck = m >> 3;
      ch[f][m] = __ldg(p.cf + (int64_t)nb * 512 + ci + 8 * cj + 64 * ck);
    }
    if (t < 128) {
      const int f = 4 + (t >> 6), m = t & 63;
      ch[f][m] = __ldg(p.cf + (int64_t)__ldg(adj + f) * 512 + m + 64 * (f == 4 ? 7 : 0));
    }
    __syncthreads();
  }

  double out[HP][2], res[HP][2];
  double mx = 0.0;
#pragma unroll
  for (int h = 0; h < HP; ++h) {
    const int tt = t + NT * h, i0 = 2 * (tt & 3), j = (tt >> 2) & 7, k = tt >> 5;
#pragma unroll
    for (int ii = 0; ii < 2; ++ii) {
      const int i = i0 + ii;
      const int o = i + 8 * j + 64 * k;
      double c, w, e, s, n, bt, tp;
      if (ZERO_X) {
        c = w = e = s = n = bt = tp = 0.0;
      } else {
        c = xs[o];
        w = i > 0 ? xs[o - 1] : hw[j + 8 * k];
        e = i < 7 ? xs[o + 1] : he[j + 8 * k];
        s = j > 0 ? xs[o - 8] : hs[i + 8 * k];
        n = j < 7 ? xs[o + 8] : hn[i + 8 * k];
        bt = k > 0 ? xs[o - 64] : hb[i + 8 * j];
        tp = k < 7 ? xs[o + 64] : ht[i + 8 * j];
      }
      double a, gam = p.c.gamma;
      if (VC) {
        // (A x)_p = inv * sum_n ((c_p + c_n) * 0.5) * (x_n - x_p), gamma_p = (0.5 h h) / sum_n face coefficient
        const double cp = cs[o];
        const double cw = i > 0 ? cs[o - 1] : ch[0][j + 8 * k], ce = i < 7 ? cs[o + 1] : ch[1][j + 8 * k];
        const double cS = j > 0 ? cs[o - 8] : ch[2][i + 8 * k], cN = j < 7 ? cs[o + 8] : ch[3][i + 8 * k];
        const double cB = k > 0 ? cs[o - 64] : ch[4][i + 8 * j], cT = k < 7 ? cs[o + 64] : ch[5][i + 8 * j];
        const double fw = DMUL(DADD(cp, cw), 0.5), fe = DMUL(DADD(cp, ce), 0.5), fs = DMUL(DADD(cp, cS), 0.5);
        const double fn = DMUL(DADD(cp, cN), 0.5), fb = DMUL(DADD(cp, cB), 0.5), ft = DMUL(DADD(cp, cT), 0.5);
        const double sum = DADD(DADD(DADD(DMUL(fw, DSUB(w, c)), DMUL(fe, DSUB(e, c))),
                                     DADD(DMUL(fs, DSUB(s, c)), DMUL(fn, DSUB(n, c)))),
                                DADD(DMUL(fb, DSUB(bt, c)), DMUL(ft, DSUB(tp, c))));
        a = DMUL(p.c.beta, sum);
        gam = __ddiv_rn(p.vc_g, DADD(DADD(DADD(fw, fe), DADD(fs, fn)), DADD(fb, ft)));
      } else {
        a = stencil_a(c, w, e, s, n, bt, tp, p.c.alpha, p.c.beta);
      }
      const double bb = ii ? bv[h].y : bv[h].x;
      if (MODE == MODE_APPLY) {
        out[h][ii] = a;
      } else if (MODE == MODE_NORM) {
        mx = nan_max(mx, fabs(DSUB(bb, a)));
      } else {
        res[h][ii] = DSUB(bb, a);
        out[h][ii] = keep_cell(p.colour, i, j, k) ? c : DADD(c, DMUL(gam, DSUB(a, bb)));
      }
    }
  }

  if (MODE == MODE_NORM) {
    // exact max: compare as doubles, publish the bit pattern (monotone for >= 0)
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) mx = nan_max(mx, __shfl_xor_sync(0xffffffffu, mx, off));
    __shared__ double wm[NT / 32];
    if ((t & 31) == 0) wm[t >> 5] = mx;
    __syncthreads();
    if (t == 0) {
      double m = wm[0];
      for (int w = 1; w < NT / 32; ++w) m = nan_max(m, wm[w]);
      atomicMax(acc, (unsigned long long)__double_as_longlong(m));
    }
    return;
  }
#pragma unroll
  for (int h = 0; h < HP; ++h) {
    const int tt = t + NT * h;
    st_stream2(p.xo + brick * 512 + 2 * tt, make_double2(out[h][0], out[h][1]));
    if (MODE == MODE_SWEEP && WRITE_R) st_stream2(p.r + brick * 512 + 2 * tt, make_double2(res[h][0], res[h][1]));
  }
  if (MODE == MODE_SWEEP && RESTRICT) {
#pragma unroll
    for (int h = 0; h < HP; ++h) {
      const int tt = t + NT * h;
      rs[2 * tt] = res[h][0];
      rs[2 * tt + 1] = res[h][1];
    }
    __syncthreads();
    if (t < 64) {
      const int I = t & 3, J = (t >> 2) & 3, K = t >> 4;
      const int f = 2 * I + 8 * (2 * J) + 64 * (2 * K);
      const double r000 = rs[f], r100 = rs[f + 1], r010 = rs[f + 8], r110 = rs[f + 9];
      const double r001 = rs[f + 64], r101 = rs[f + 65], r011 = rs[f + 72], r111 = rs[f + 73];
      const double v =
          DMUL(0.125, DADD(DADD(DADD(r000, r100), DADD(r010, r110)), DADD(DADD(r001, r101), DADD(r011, r111))));
      const int pr = __ldg(p.parent + brick);
      const int oct = pr & 7;
      const int ox = oct & 1, oy = (oct >> 1) & 1, oz = oct >> 2;
      p.bc[(int64_t)(pr >> 3) * 512 + (4 * ox + I) + 8 * (4 * oy + J) + 64 * (4 * oz + K)] = v;
    }
  }
}

// ranges of at least this many bricks run the 128-thread variant (more bricks in flight per SM)
constexpr int64_t kSweep128Bricks = 4096;

template <unsigned FLAGS>
static cudaError_t launch_sweep_t(const SweepArgs& a, cudaStream_t s) {
  if (a.nbricks <= 0) return cudaSuccess;
  static const bool nt256 = getenv("MG_SWEEP_NT256") != nullptr;  // (A/B: the 256-thread variant everywhere)
  if (a.nbricks >= kSweep128Bricks && !nt256)
    launch_k(sweep_kernel<MODE_SWEEP, FLAGS, 128>, (unsigned)a.nbricks, 128, 0, s, a, nullptr);
  else
    launch_k(sweep_kernel<MODE_SWEEP, FLAGS>, (unsigned)a.nbricks, 256, 0, s, a, nullptr);
  return cudaGetLastError();
}

cudaError_t launch_sweep(const SweepArgs& a, unsigned flags, cudaStream_t s) {
  if (a.E != 8) return launch_gsweep(a, flags, 0, nullptr, s);
  if (flags & SW_VARCOEF) {
    switch (flags & (SW_WRITE_R | SW_RESTRICT | SW_INTERP | SW_ZERO_X)) {
#define VC_CASE(F) \
  case (F): return launch_sweep_t<(F) | SW_VARCOEF>(a, s);
      VC_CASE(0) VC_CASE(SW_WRITE_R) VC_CASE(SW_RESTRICT) VC_CASE(SW_INTERP) VC_CASE(SW_INTERP | SW_WRITE_R)
      VC_CASE(SW_INTERP | SW_RESTRICT) VC_CASE(SW_ZERO_X) VC_CASE(SW_ZERO_X | SW_WRITE_R)
      VC_CASE(SW_ZERO_X | SW_RESTRICT)
#undef VC_CASE
      default: return cudaErrorInvalidValue;
    }
  }
  switch (flags & (SW_WRITE_R | SW_RESTRICT | SW_INTERP | SW_ZERO_X)) {
    case 0: return launch_sweep_t<0>(a, s);
    case SW_WRITE_R: return launch_sweep_t<SW_WRITE_R>(a, s);
    case SW_RESTRICT: return launch_sweep_t<SW_RESTRICT>(a, s);
    case SW_INTERP: return launch_sweep_t<SW_INTERP>(a, s);
    case SW_INTERP | SW_WRITE_R: return launch_sweep_t<SW_INTERP | SW_WRITE_R>(a, s);
    case SW_INTERP | SW_RESTRICT: return launch_sweep_t<SW_INTERP | SW_RESTRICT>(a, s);
    case SW_ZERO_X: return launch_sweep_t<SW_ZERO_X>(a, s);
    case SW_ZERO_X | SW_WRITE_R: return launch_sweep_t<SW_ZERO_X | SW_WRITE_R>(a, s);
    case SW_ZERO_X | SW_RESTRICT: return launch_sweep_t<SW_ZERO_X | SW_RESTRICT>(a, s);
    default: return cudaErrorInvalidValue;
  }
}

// ---------------------------------------------------------------------------
// Streaming column sweep (the level-0 hot kernel).
//
// One CTA of 4 warps streams a segment of <= 16 consecutive bricks of one
// z-column (7 CTAs per SM).  Warp w owns planes 2w, 2w+1 of every brick; lane l
// owns the cell pair (2(l&3), l>>2) of a plane and walks its planes in k,
// keeping planes k-1, k, k+1 of x in registers.
// In-plane neighbours: i+-1 by warp shuffles, j+-1 by 128-bit shared loads of
// the neighbouring rows.  The x and b bricks arrive by TMA bulk copies
// (cp.async.bulk, 4 KiB each, lane 0) into a 3-stage shared-memory ring
// completed on mbarriers, two bricks ahead; the 256 W/E/S/N face-halo values of
// a brick (neighbour columns, through L2) arrive by 8-byte cp.async into the
// same stage, tracked by the same mbarrier (cp.async.mbarrier.arrive.noinc).
// The k-halo is the previous brick's plane 7 (a 512-byte carry buffer) and the
// next brick's plane 0 (ring); one 512-byte plane below / above the segment.  Stores of x'
// (and r) are coalesced 128-bit streaming stores.  DRAM traffic per point:
// read x, b; write x' (+ r): the algorithmic 24 (32) bytes.
// ---------------------------------------------------------------------------
constexpr int COL_NST = 3;  // ring stages: current, next (plane 0 = k-halo), one in flight
constexpr int COL_MAXSEG = 16;

template <bool VC>
struct alignas(128) ColStage {  // (every stage and its TMA destinations 128-byte aligned)
  double x[512];
  double b[512];
  double fwe[2][64][2];  // W box (i=6,7 of the W brick) and E box (i=0,1 of the E brick), [k][j][2]
  double fsn[2][64];     // S row (j=7 of the S brick) and N row (j=0 of the N brick), [k][i]
  // variable coefficients (reading A23): the c brick and its face halos, boxes as for x
  double c[VC ? 512 : 1];
  double cwe[VC ? 2 : 1][VC ? 64 : 1][2];
  double csn[VC ? 2 : 1][VC ? 64 : 1];
};
constexpr uint32_t kStageBytes = 8192 + 2 * 1024 + 2 * 512;  // TMA bytes landing in one full stage
constexpr uint32_t kStageBytesC = 4096 + 2 * 1024 + 2 * 512;  // ... and the c brick + halos (VC)
static_assert(offsetof(ColStage<false>, fsn) % 128 == 0 && offsetof(ColStage<true>, c) % 128 == 0 &&
                  offsetof(ColStage<true>, cwe) % 128 == 0 && offsetof(ColStage<true>, csn) % 128 == 0 &&
                  sizeof(ColStage<false>) % 128 == 0 && sizeof(ColStage<true>) % 128 == 0,
              "TMA destinations 128-byte aligned");

template <bool RESTRICT, bool VC>
struct ColSmem {
  ColStage<VC> st[COL_NST];  // stage of "brick" cnt holds only plane 0 of the brick above the segment
  double carry[2][64];   // plane 7 of the previous brick (k-halo of plane 0), double-buffered;
                         // carry[1] first holds plane 7 of the brick below the segment
  double ccarry[VC ? 2 : 1][64];  // the same for c (VC)
  double rs[RESTRICT ? 2 : 1][RESTRICT ? 512 : 2];  // residual of the current brick (fused restriction)
  uint64_t bar[COL_NST + 1];
  int sid[COL_MAXSEG];
  int spar[COL_MAXSEG];
  int4 sside[COL_MAXSEG];
};

constexpr int COL_WARPS = 4;  // warp w streams planes 2w, 2w+1 of every brick

// variable-coefficient cell (reading A23, the expression of sweep_kernel<..., SW_VARCOEF>): returns a = A x
// and sets gam = (0.5 h h) / (sum of the face coefficients)
__device__ __forceinline__ double vc_cell(double c, double w, double e, double s, double n, double bt, double tp,
                                          double cp, double cw, double ce, double cS, double cN, double cB,
                                          double cT, double beta, double vc_g, double& gam) {
  const double fw = DMUL(DADD(cp, cw), 0.5), fe = DMUL(DADD(cp, ce), 0.5), fs = DMUL(DADD(cp, cS), 0.5);
  const double fn = DMUL(DADD(cp, cN), 0.5), fb = DMUL(DADD(cp, cB), 0.5), ft = DMUL(DADD(cp, cT), 0.5);
  const double sum = DADD(DADD(DADD(DMUL(fw, DSUB(w, c)), DMUL(fe, DSUB(e, c))),
                               DADD(DMUL(fs, DSUB(s, c)), DMUL(fn, DSUB(n, c)))),
                          DADD(DMUL(fb, DSUB(bt, c)), DMUL(ft, DSUB(tp, c))));
  gam = __ddiv_rn(vc_g, DADD(DADD(DADD(fw, fe), DADD(fs, fn)), DADD(fb, ft)));
  return DMUL(beta, sum);
}

template <unsigned FLAGS>
__global__ void __launch_bounds__(COL_WARPS * 32, (FLAGS & SW_VARCOEF) ? 4 : 6)
    sweep_col_kernel(SweepArgs p, ColArgs ca, const __grid_constant__ FaceMaps fm,
                     const __grid_constant__ FaceMaps fmc) {
  pdl_wait();
  constexpr bool WRITE_R = (FLAGS & SW_WRITE_R) != 0;
  constexpr bool RESTRICT = (FLAGS & SW_RESTRICT) != 0;
  constexpr bool NORM = (FLAGS & SW_NORM) != 0;  // maxNormRes: only max |b - Ax| leaves the kernel
  constexpr bool VC = (FLAGS & SW_VARCOEF) != 0;  // variable coefficients: the c field streams too
  extern __shared__ __align__(128) unsigned char smem_raw[];
  ColSmem<RESTRICT, VC>& S = *reinterpret_cast<ColSmem<RESTRICT, VC>*>(smem_raw);
  double mx = 0.0;
  const int t = threadIdx.x, w = t >> 5, l = t & 31;
  const int i0 = 2 * (l & 3), j = l >> 2;
  const int q = 8 * j + i0;  // this lane's pair inside a plane
  const int2 sg = ca.segs[blockIdx.x];
  const int cnt = sg.y;
  if (t < cnt) {
    const int id = ca.bricks[sg.x + t];
    S.sid[t] = id;
    S.sside[t] = ca.side[sg.x + t];
    if (RESTRICT) S.spar[t] = p.parent[id];
  }
  if (t == 0) {
    for (int s = 0; s <= COL_NST; ++s) mbar_init(&S.bar[s], 1);  // thread 0's expect_tx arrive + TMA bytes
    mbar_fence_init();
  }
  __syncthreads();
  // stage brick n (thread 0): x and b bricks by 1D bulk copies, the four face halos
  // by 3D tensor copies (+ the same for c).  n == cnt stages only plane 0 of the brick above the segment.
  auto issue = [&](int n) {
    if (t != 0) return;
    const int s = n % COL_NST;
    if (n == cnt) {
      const int64_t above = __ldg(p.adj + (int64_t)S.sid[cnt - 1] * 8 + 5);
      mbar_expect_tx(&S.bar[s], VC ? 1024 : 512);
      tma_load_1d(S.st[s].x, p.x + above * 512, 512, &S.bar[s]);
      if (VC) tma_load_1d(S.st[s].c, p.cf + above * 512, 512, &S.bar[s]);
      return;
    }
    const int64_t id = S.sid[n];
    const int4 sd = S.sside[n];
    mbar_expect_tx(&S.bar[s], kStageBytes + (VC ? kStageBytesC : 0));
    tma_load_1d(S.st[s].x, p.x + id * 512, 4096, &S.bar[s]);
    tma_load_1d(S.st[s].b, p.b + id * 512, 4096, &S.bar[s]);
    tma_load_3d(S.st[s].fwe[0], &fm.we, 6, 0, sd.x * 8, &S.bar[s]);  // W brick, i = 6..7
    tma_load_3d(S.st[s].fwe[1], &fm.we, 0, 0, sd.y * 8, &S.bar[s]);  // E brick, i = 0..1
    tma_load_3d(S.st[s].fsn[0], &fm.sn, 0, 7, sd.z * 8, &S.bar[s]);  // S brick, j = 7
    tma_load_3d(S.st[s].fsn[1], &fm.sn, 0, 0, sd.w * 8, &S.bar[s]);  // N brick, j = 0
    if (VC) {
      tma_load_1d(S.st[s].c, p.cf + id * 512, 4096, &S.bar[s]);
      tma_load_3d(S.st[s].cwe[0], &fmc.we, 6, 0, sd.x * 8, &S.bar[s]);
      tma_load_3d(S.st[s].cwe[1], &fmc.we, 0, 0, sd.y * 8, &S.bar[s]);
      tma_load_3d(S.st[s].csn[0], &fmc.sn, 0, 7, sd.z * 8, &S.bar[s]);
      tma_load_3d(S.st[s].csn[1], &fmc.sn, 0, 0, sd.w * 8, &S.bar[s]);
    }
  };
  if (t == 0) {
    const int64_t below = __ldg(p.adj + (int64_t)S.sid[0] * 8 + 4);
    mbar_expect_tx(&S.bar[COL_NST], VC ? 1024 : 512);
    tma_load_1d(S.carry[1], p.x + below * 512 + 448, 512, &S.bar[COL_NST]);
    if (VC) tma_load_1d(S.ccarry[VC ? 1 : 0], p.cf + below * 512 + 448, 512, &S.bar[COL_NST]);
  }
  issue(0);
  issue(1);  // brick 1, or the plane above when cnt == 1
  if (w == 0) mbar_wait(&S.bar[COL_NST], 0);

  for (int n = 0; n < cnt; ++n) {
    if (n + 2 <= cnt) {
      fence_proxy_async();  // the generic-proxy reads of the stage being refilled are complete
      issue(n + 2);         // (its last readers finished before the barrier that ended step n-1)
    }
    const int s = n % COL_NST;
    mbar_wait(&S.bar[s], (uint32_t)((n / COL_NST) & 1));
    const ColStage<VC>& G = S.st[s];
    const double* X = G.x;
    const int k0 = 2 * w;
    double2 xm, xc, xp, cm = make_double2(0.0, 0.0), cc = cm, cpn = cm;
    if (w > 0) {
      xm = *reinterpret_cast<const double2*>(X + 64 * (k0 - 1) + q);
      if (VC) cm = *reinterpret_cast<const double2*>(G.c + 64 * (k0 - 1) + q);
    } else {
      xm = *reinterpret_cast<const double2*>(S.carry[(n + 1) & 1] + q);  // = carry[(n-1)&1]
      if (VC) cm = *reinterpret_cast<const double2*>(S.ccarry[VC ? (n + 1) & 1 : 0] + q);
    }
    xc = *reinterpret_cast<const double2*>(X + 64 * k0 + q);
    if (VC) cc = *reinterpret_cast<const double2*>(G.c + 64 * k0 + q);
    const int64_t gbase = (int64_t)S.sid[n] * 512 + q;
#pragma unroll
    for (int kk = 0; kk < 2; ++kk) {
      const int k = k0 + kk;
      if (k < 7) {
        xp = *reinterpret_cast<const double2*>(X + 64 * (k + 1) + q);
        if (VC) cpn = *reinterpret_cast<const double2*>(G.c + 64 * (k + 1) + q);
      } else {  // plane 0 of the next brick (or of the brick above the segment)
        const int s1 = (n + 1) % COL_NST;
        mbar_wait(&S.bar[s1], (uint32_t)(((n + 1) / COL_NST) & 1));
        xp = *reinterpret_cast<const double2*>(S.st[s1].x + q);
        if (VC) cpn = *reinterpret_cast<const double2*>(S.st[s1].c + q);
      }
      const double2 bb = *reinterpret_cast<const double2*>(G.b + 64 * k + q);
      const double2 rs_ = *reinterpret_cast<const double2*>(X + 64 * k + (j > 0 ? q - 8 : q));
      const double2 rn_ = *reinterpret_cast<const double2*>(X + 64 * k + (j < 7 ? q + 8 : q));
      const double fw = G.fwe[0][j + 8 * k][1];  // i = 7 of the W brick
      const double fe = G.fwe[1][j + 8 * k][0];  // i = 0 of the E brick
      const double2 fs = *reinterpret_cast<const double2*>(&G.fsn[0][i0 + 8 * k]);
      const double2 fn = *reinterpret_cast<const double2*>(&G.fsn[1][i0 + 8 * k]);
      const double wl = __shfl_up_sync(0xffffffffu, xc.y, 1);
      const double er = __shfl_down_sync(0xffffffffu, xc.x, 1);
      const double wv = i0 > 0 ? wl : fw;
      const double ev = i0 < 6 ? er : fe;
      const double2 sv = j > 0 ? rs_ : fs;
      const double2 nv = j < 7 ? rn_ : fn;
      double a0, a1, g0 = p.c.gamma, g1 = p.c.gamma;
      if (VC) {
        const double2 crs = *reinterpret_cast<const double2*>(G.c + 64 * k + (j > 0 ? q - 8 : q));
        const double2 crn = *reinterpret_cast<const double2*>(G.c + 64 * k + (j < 7 ? q + 8 : q));
        const double cfw = G.cwe[0][j + 8 * k][1], cfe = G.cwe[VC ? 1 : 0][j + 8 * k][0];
        const double2 cfs = *reinterpret_cast<const double2*>(&G.csn[0][i0 + 8 * k]);
        const double2 cfn = *reinterpret_cast<const double2*>(&G.csn[VC ? 1 : 0][i0 + 8 * k]);
        const double cwl = __shfl_up_sync(0xffffffffu, cc.y, 1);
        const double cer = __shfl_down_sync(0xffffffffu, cc.x, 1);
        const double cwv = i0 > 0 ? cwl : cfw, cev = i0 < 6 ? cer : cfe;
        const double2 csv = j > 0 ? crs : cfs, cnv = j < 7 ? crn : cfn;
        a0 = vc_cell(xc.x, wv, xc.y, sv.x, nv.x, xm.x, xp.x, cc.x, cwv, cc.y, csv.x, cnv.x, cm.x, cpn.x,
                     p.c.beta, p.vc_g, g0);
        a1 = vc_cell(xc.y, xc.x, ev, sv.y, nv.y, xm.y, xp.y, cc.y, cc.x, cev, csv.y, cnv.y, cm.y, cpn.y,
                     p.c.beta, p.vc_g, g1);
      } else {
        a0 = stencil_a(xc.x, wv, xc.y, sv.x, nv.x, xm.x, xp.x, p.c.alpha, p.c.beta);
        a1 = stencil_a(xc.y, xc.x, ev, sv.y, nv.y, xm.y, xp.y, p.c.alpha, p.c.beta);
      }
      double2 xn, rv;
      xn.x = keep_cell(p.colour, i0, j, k) ? xc.x : DADD(xc.x, DMUL(g0, DSUB(a0, bb.x)));
      xn.y = keep_cell(p.colour, i0 + 1, j, k) ? xc.y : DADD(xc.y, DMUL(g1, DSUB(a1, bb.y)));
      rv.x = DSUB(bb.x, a0);
      rv.y = DSUB(bb.y, a1);
      if (NORM) {
        mx = nan_max(mx, fabs(rv.x));
        mx = nan_max(mx, fabs(rv.y));
      } else {
        st_stream2(p.xo + gbase + 64 * k, xn);
      }
      if (WRITE_R) st_stream2(p.r + gbase + 64 * k, rv);
      if (RESTRICT) *reinterpret_cast<double2*>(S.rs[n & 1] + 64 * k + q) = rv;
      if (k == 7) {
        *reinterpret_cast<double2*>(S.carry[n & 1] + q) = xc;  // k-halo of the next brick
        if (VC) *reinterpret_cast<double2*>(S.ccarry[VC ? n & 1 : 0] + q) = cc;
      }
      xm = xc;
      xc = xp;
      cm = cc;
      cc = cpn;
    }
    __syncthreads();  // stage n-1 free for refill; carry / rs of brick n complete
    if (RESTRICT && t < 64) {
      const double* R = S.rs[n & 1];
      const int I = t & 3, J = (t >> 2) & 3, K = t >> 4;
      const int f = 2 * I + 16 * J + 128 * K;
      const double v = DMUL(0.125, DADD(DADD(DADD(R[f], R[f + 1]), DADD(R[f + 8], R[f + 9])),
                                        DADD(DADD(R[f + 64], R[f + 65]), DADD(R[f + 72], R[f + 73]))));
      const int pr = S.spar[n];
      const int oct = pr & 7;
      const int ox = oct & 1, oy = (oct >> 1) & 1, oz = oct >> 2;
      p.bc[(int64_t)(pr >> 3) * 512 + (4 * ox + I) + 8 * (4 * oy + J) + 64 * (4 * oz + K)] = v;
    }
  }
  if (NORM) {  // exact max over the CTA's cells, published as uint64 bits (monotone for >= 0)
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) mx = nan_max(mx, __shfl_xor_sync(0xffffffffu, mx, off));
    __shared__ double wm[COL_WARPS];
    if (l == 0) wm[w] = mx;
    __syncthreads();
    if (t == 0) {
      double m = wm[0];
      for (int q2 = 1; q2 < COL_WARPS; ++q2) m = nan_max(m, wm[q2]);
      atomicMax(p.acc, (unsigned long long)__double_as_longlong(m));
    }
  }
  pdl_trigger();
}

bool col_supports(unsigned flags) {
  const unsigned f = flags & (SW_WRITE_R | SW_RESTRICT | SW_INTERP | SW_ZERO_X);
  return f == 0 || f == SW_WRITE_R || f == SW_RESTRICT;
}

#define COL_FLAG_LIST(X) \
  X(0) X(SW_WRITE_R) X(SW_RESTRICT) X(SW_NORM) X(SW_VARCOEF) X(SW_VARCOEF | SW_WRITE_R) X(SW_VARCOEF | SW_RESTRICT) \
  X(SW_VARCOEF | SW_NORM)

template <unsigned F>
constexpr size_t col_smem() {
  return sizeof(ColSmem<(F & SW_RESTRICT) != 0, (F & SW_VARCOEF) != 0>);
}

cudaError_t launch_sweep_col(const SweepArgs& a, const ColArgs& c, const FaceMaps& fm, unsigned flags,
                             cudaStream_t s, const FaceMaps* fmc) {
  if (c.nseg <= 0) return cudaSuccess;
  const unsigned g = (unsigned)c.nseg, b = COL_WARPS * 32;
  const unsigned f = flags & (SW_WRITE_R | SW_RESTRICT | SW_INTERP | SW_ZERO_X | SW_NORM | SW_VARCOEF);
  if ((f & SW_VARCOEF) && (!fmc || !a.cf)) return cudaErrorInvalidValue;
  const FaceMaps& mc = fmc ? *fmc : fm;
  switch (f) {
#define COL_CASE(F)                                                        \
  case (F):                                                                \
    launch_plain(sweep_col_kernel<(F)>, g, b, col_smem<(F)>(), s, a, c, fm, mc); \
    break;
    COL_FLAG_LIST(COL_CASE)
#undef COL_CASE
    default:
      return cudaErrorInvalidValue;
  }
  return cudaGetLastError();
}

cudaError_t encode_box_map(const double* base, int64_t n_alloc, const unsigned box[3], CUtensorMap* out,
                           bool swizzle64) {
  static PFN_cuTensorMapEncodeTiled_v12000 encode = nullptr;
  if (!encode) {
    void* fn = nullptr;
    cudaDriverEntryPointQueryResult q;
    cudaError_t e = cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q);
    if (e != cudaSuccess) return e;
    if (q != cudaDriverEntryPointSuccess || !fn) return cudaErrorNotSupported;
    encode = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(fn);
  }
  const cuuint64_t dims[3] = {8, 8, (cuuint64_t)n_alloc * 8};  // i, j, planes
  const cuuint64_t strides[2] = {64, 512};                      // bytes of one j row, one plane
  const cuuint32_t estr[3] = {1, 1, 1};
  const cuuint32_t bx[3] = {box[0], box[1], box[2]};
  const CUresult r = encode(out, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 3, const_cast<double*>(base), dims, strides, bx,
                            estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                            swizzle64 ? CU_TENSOR_MAP_SWIZZLE_64B : CU_TENSOR_MAP_SWIZZLE_NONE,
                            CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return r == CUDA_SUCCESS ? cudaSuccess : cudaErrorInvalidValue;
}

cudaError_t encode_face_maps(const double* x, int64_t n_alloc, FaceMaps* out) {
  const unsigned box_we[3] = {2, 8, 8}, box_sn[3] = {8, 1, 8};
  cudaError_t e = encode_box_map(x, n_alloc, box_we, &out->we);
  if (e != cudaSuccess) return e;
  return encode_box_map(x, n_alloc, box_sn, &out->sn);
}

cudaError_t encode_pair_maps(const double* x, const double* b, int64_t n_alloc, PairMaps* out) {
  const unsigned we[3] = {2, 8, 8}, sn2[3] = {8, 2, 8}, cor[3] = {2, 1, 8}, sn1[3] = {8, 1, 8};
  cudaError_t e;
  if ((e = encode_box_map(x, n_alloc, we, &out->xwe)) != cudaSuccess) return e;
  if ((e = encode_box_map(x, n_alloc, sn2, &out->xsn)) != cudaSuccess) return e;
  if ((e = encode_box_map(x, n_alloc, cor, &out->xcor)) != cudaSuccess) return e;
  if ((e = encode_box_map(b, n_alloc, we, &out->bwe)) != cudaSuccess) return e;
  return encode_box_map(b, n_alloc, sn1, &out->bsn);
}

cudaError_t launch_apply_op(const double* x, double* Ax, const int32_t* adj, int64_t brick0, int64_t nbricks,
                            Coeffs c, cudaStream_t s, int E) {
  if (nbricks <= 0) return cudaSuccess;
  SweepArgs a{};
  a.x = x;
  a.xo = Ax;
  a.adj = adj;
  a.brick0 = brick0;
  a.nbricks = nbricks;
  a.c = c;
  a.E = E;
  if (E != 8) return launch_gsweep(a, 0, 1, nullptr, s);
  static const bool nt256 = getenv("MG_SWEEP_NT256") != nullptr;
  if (nbricks >= kSweep128Bricks && !nt256)
    launch_k(sweep_kernel<MODE_APPLY, 0, 128>, (unsigned)nbricks, 128, 0, s, a, nullptr);
  else
    launch_k(sweep_kernel<MODE_APPLY, 0>, (unsigned)nbricks, 256, 0, s, a, nullptr);
  return cudaGetLastError();
}

cudaError_t launch_norm(const double* x, const double* b, const int32_t* adj, int64_t nbricks, Coeffs c,
                        unsigned long long* acc, cudaStream_t s, const double* cf, int E) {
  if (nbricks <= 0) return cudaSuccess;
  SweepArgs a{};
  a.x = x;
  a.b = b;
  a.adj = adj;
  a.brick0 = 0;
  a.nbricks = nbricks;
  a.c = c;
  a.cf = cf;
  a.E = E;
  if (E != 8) return launch_gsweep(a, cf ? SW_VARCOEF : 0u, 2, acc, s);
  static const bool nt256 = getenv("MG_SWEEP_NT256") != nullptr;
  const bool big = nbricks >= kSweep128Bricks && !nt256;
  if (cf && big)
    launch_k(sweep_kernel<MODE_NORM, SW_VARCOEF, 128>, (unsigned)nbricks, 128, 0, s, a, acc);
  else if (cf)
    launch_k(sweep_kernel<MODE_NORM, SW_VARCOEF>, (unsigned)nbricks, 256, 0, s, a, acc);
  else if (big)
    launch_k(sweep_kernel<MODE_NORM, 0, 128>, (unsigned)nbricks, 128, 0, s, a, acc);
  else
    launch_k(sweep_kernel<MODE_NORM, 0>, (unsigned)nbricks, 256, 0, s, a, acc);
  return cudaGetLastError();
}

// ---------------------------------------------------------------------------
// smooth(+residual) of the paper's kernel set: pointwise, reads x, Ax, b.
// ---------------------------------------------------------------------------
template <bool WRITE_R>
__global__ void __launch_bounds__(256) smooth_kernel(double* __restrict__ x, const double* __restrict__ Ax,
                                                     const double* __restrict__ b, double* __restrict__ r,
                                                     int64_t base, int64_t n2, double gamma, int colour) {
  pdl_begin();
  for (int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; q < n2; q += (int64_t)gridDim.x * blockDim.x) {
    const int64_t o = base + 2 * q;
    const double2 xv = ldg2(x + o);
    const double2 av = ld_stream2(Ax + o);
    const double2 bv = ld_stream2(b + o);
    const int c = (int)(o & 511), i = c & 7, j = (c >> 3) & 7, k = c >> 6;
    double2 xn, rv;
    rv.x = DSUB(bv.x, av.x);
    rv.y = DSUB(bv.y, av.y);
    xn.x = keep_cell(colour, i, j, k) ? xv.x : DADD(xv.x, DMUL(gamma, DSUB(av.x, bv.x)));
    xn.y = keep_cell(colour, i + 1, j, k) ? xv.y : DADD(xv.y, DMUL(gamma, DSUB(av.y, bv.y)));
    st_stream2(x + o, xn);
    if (WRITE_R) st_stream2(r + o, rv);
  }
}

static int g_num_sms = 148;

static unsigned grid_for(int64_t n2) {
  const int64_t want = (n2 + 255) / 256;
  const int64_t cap = (int64_t)g_num_sms * 8;
  return (unsigned)(want < cap ? (want > 0 ? want : 1) : cap);
}

cudaError_t launch_smooth(double* x, const double* Ax, const double* b, double* r, int64_t brick0, int64_t nbricks,
                          Coeffs c, bool write_r, cudaStream_t s, int colour, int E) {
  if (nbricks <= 0) return cudaSuccess;
  if (E != 8) return launch_gsmooth(x, Ax, b, r, brick0, nbricks, c, write_r, colour, E, s);
  const int64_t n2 = nbricks * 256;
  if (write_r)
    launch_k(smooth_kernel<true>, grid_for(n2), 256, 0, s, x, Ax, b, r, brick0 * 512, n2, c.gamma, colour);
  else
    launch_k(smooth_kernel<false>, grid_for(n2), 256, 0, s, x, Ax, b, r, brick0 * 512, n2, c.gamma, colour);
  return cudaGetLastError();
}

// ---------------------------------------------------------------------------
// restriction: one CTA (128 threads) per fine brick -> 64 coarse cells of the
// parent's octant.
// ---------------------------------------------------------------------------
__global__ void __launch_bounds__(128) restrict_kernel(const double* __restrict__ r, double* __restrict__ bc,
                                                       const int32_t* __restrict__ parent) {
  pdl_begin();
  __shared__ __align__(16) double rs[512];
  const int64_t f = blockIdx.x;
  const int t = threadIdx.x;
  const double2* src = reinterpret_cast<const double2*>(r + f * 512);
  reinterpret_cast<double2*>(rs)[t] = __ldg(src + t);
  reinterpret_cast<double2*>(rs)[t + 128] = __ldg(src + t + 128);
  __syncthreads();
  if (t < 64) {
    const int I = t & 3, J = (t >> 2) & 3, K = t >> 4;
    const int o = 2 * I + 16 * J + 128 * K;
    const double v = DMUL(0.125, DADD(DADD(DADD(rs[o], rs[o + 1]), DADD(rs[o + 8], rs[o + 9])),
                                      DADD(DADD(rs[o + 64], rs[o + 65]), DADD(rs[o + 72], rs[o + 73]))));
    const int pr = __ldg(parent + f);
    const int oct = pr & 7;
    const int ox = oct & 1, oy = (oct >> 1) & 1, oz = oct >> 2;
    bc[(int64_t)(pr >> 3) * 512 + (4 * ox + I) + 8 * (4 * oy + J) + 64 * (4 * oz + K)] = v;
  }
}

cudaError_t launch_restrict(const double* r, double* bc, const int32_t* parent, int64_t nfine, cudaStream_t s,
                            int E) {
  if (nfine <= 0) return cudaSuccess;
  if (E != 8) return launch_grestrict(r, bc, parent, nfine, E, s);
  launch_k(restrict_kernel, (unsigned)nfine, 128, 0, s, r, bc, parent);
  return cudaGetLastError();
}

// interpolation+increment: one CTA (256 threads) per fine brick, 2 cells each.
__global__ void __launch_bounds__(256) interp_kernel(double* __restrict__ x, const double* __restrict__ xc,
                                                     const int32_t* __restrict__ parent) {
  pdl_begin();
  const int64_t f = blockIdx.x;
  const int t = threadIdx.x;
  const int i0 = 2 * (t & 3), j = (t >> 2) & 7, k = t >> 5;
  const int pr = __ldg(parent + f);
  const double cv = __ldg(xc + (int64_t)(pr >> 3) * 512 + coarse_off(pr & 7, i0, j, k));
  double2* px = reinterpret_cast<double2*>(x + f * 512) + t;
  double2 v = *px;
  v.x = DADD(v.x, cv);
  v.y = DADD(v.y, cv);
  *px = v;
}

// the same, four fine bricks per CTA (one per 64-thread quarter, 8 cells per thread): all loads of
// a thread (parent, coarse value, four 16-byte x pieces) are issued before its adds and stores, so
// more bytes are in flight per thread; stores stream past L1 (the next pass re-reads x from HBM)
__global__ void __launch_bounds__(256) interp4_kernel(double* __restrict__ x, const double* __restrict__ xc,
                                                      const int32_t* __restrict__ parent, int64_t nfine) {
  pdl_begin();
  const int t = threadIdx.x, qb = t >> 6, u = t & 63;
  const int64_t f = (int64_t)blockIdx.x * 4 + qb;
  if (f >= nfine) return;
  // pieces e = u + 64 m, m = 0..3: the double2 at cells 2e, 2e + 1 of the brick (one coarse cell)
  const int pr = __ldg(parent + f);
  double2* px = reinterpret_cast<double2*>(x + f * 512);
  double2 v[4];
  double cv[4];
#pragma unroll
  for (int m = 0; m < 4; ++m) {
    const int e = u + 64 * m, c = 2 * e, i0 = c & 7, j = (c >> 3) & 7, k = c >> 6;
    v[m] = px[e];
    cv[m] = __ldg(xc + (int64_t)(pr >> 3) * 512 + coarse_off(pr & 7, i0, j, k));
  }
#pragma unroll
  for (int m = 0; m < 4; ++m) {
    v[m].x = DADD(v[m].x, cv[m]);
    v[m].y = DADD(v[m].y, cv[m]);
    st_stream2(x + f * 512 + 2 * (u + 64 * m), v[m]);
  }
}

cudaError_t launch_interp(double* x, const double* xc, const int32_t* parent, int64_t nfine, cudaStream_t s,
                          int E) {
  if (nfine <= 0) return cudaSuccess;
  if (E != 8) return launch_ginterp(x, xc, parent, nfine, E, s);
  static const bool one = getenv("MG_INTERP1") != nullptr;  // (measurement switch: one brick per CTA)
  if (one)
    launch_k(interp_kernel, (unsigned)nfine, 256, 0, s, x, xc, parent);
  else
    launch_k(interp4_kernel, (unsigned)((nfine + 3) / 4), 256, 0, s, x, xc, parent, nfine);
  return cudaGetLastError();
}

__global__ void __launch_bounds__(256) zero_kernel(double* __restrict__ x, int64_t base, int64_t n2) {
  pdl_begin();
  for (int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; q < n2; q += (int64_t)gridDim.x * blockDim.x)
    reinterpret_cast<double2*>(x + base)[q] = make_double2(0.0, 0.0);
}

cudaError_t launch_zero(double* x, int64_t brick0, int64_t nbricks, cudaStream_t s, int E) {
  if (nbricks <= 0) return cudaSuccess;
  const int64_t bv = (int64_t)E * E * E, n2 = nbricks * bv / 2;
  launch_k(zero_kernel, grid_for(n2), 256, 0, s, x, brick0 * bv, n2);
  return cudaGetLastError();
}

// ---------------------------------------------------------------------------
// Resident bottom solver: all bricks of the coarsest level (no
// ghosts, <= 8 bricks) in one CTA's shared memory; `sweeps` Jacobi sweeps with
// a CTA barrier between sweeps instead of `sweeps` kernel launches.
// ---------------------------------------------------------------------------

__global__ void __launch_bounds__(1024) bottom_resident_kernel(const double* __restrict__ x, double* __restrict__ xo,
                                                               const double* __restrict__ b,
                                                               const int32_t* __restrict__ adj, int nbricks,
                                                               int sweeps, int zero_x, Coeffs c, double msign) {
  pdl_begin();
  extern __shared__ __align__(16) double sm[];
  bottom_resident_body(x, xo, b, adj, nbricks, sweeps, zero_x, c, sm, msign);
}

cudaError_t launch_bottom_resident(const double* x, double* xo, const double* b, const int32_t* adj, int nbricks,
                                   int sweeps, bool zero_x, Coeffs c, cudaStream_t s, double msign) {
  if (nbricks <= 0 || nbricks > kResidentMaxBricks) return cudaErrorInvalidValue;
  const size_t smem = (size_t)nbricks * 512 * 2 * sizeof(double);
  launch_k(bottom_resident_kernel, 1, 128 * nbricks, smem, s, x, xo, b, adj, nbricks, sweeps, zero_x ? 1 : 0, c, msign);
  return cudaGetLastError();
}

// ---------------------------------------------------------------------------
// Layout conversion (mg_set_rhs / mg_get_solution; not timed in the V-cycle).
// ---------------------------------------------------------------------------
__global__ void __launch_bounds__(256) lex_to_brick_kernel(const double* __restrict__ lex, double* __restrict__ br,
                                                           const int32_t* __restrict__ coord, int nx, int ny) {
  pdl_begin();
  const int64_t bI = blockIdx.x;
  const int t = threadIdx.x;
  const int i0 = 2 * (t & 3), j = (t >> 2) & 7, k = t >> 5;
  const int cx = coord[bI * 3], cy = coord[bI * 3 + 1], cz = coord[bI * 3 + 2];
  const int64_t li = (int64_t)(8 * cx + i0) + (int64_t)nx * ((int64_t)(8 * cy + j) + (int64_t)ny * (8 * cz + k));
  reinterpret_cast<double2*>(br + bI * 512)[t] = *reinterpret_cast<const double2*>(lex + li);
}

__global__ void __launch_bounds__(256) brick_to_lex_kernel(const double* __restrict__ br, double* __restrict__ lex,
                                                           const int32_t* __restrict__ coord, int nx, int ny) {
  pdl_begin();
  const int64_t bI = blockIdx.x;
  const int t = threadIdx.x;
  const int i0 = 2 * (t & 3), j = (t >> 2) & 7, k = t >> 5;
  const int cx = coord[bI * 3], cy = coord[bI * 3 + 1], cz = coord[bI * 3 + 2];
  const int64_t li = (int64_t)(8 * cx + i0) + (int64_t)nx * ((int64_t)(8 * cy + j) + (int64_t)ny * (8 * cz + k));
  *reinterpret_cast<double2*>(lex + li) = reinterpret_cast<const double2*>(br + bI * 512)[t];
}

cudaError_t launch_lex_to_brick(const double* lex, double* bricks, const int32_t* coord, int64_t nowned, int nx,
                                int ny, cudaStream_t s, int E) {
  if (nowned <= 0) return cudaSuccess;
  if (E != 8) return launch_glex(lex, bricks, coord, nowned, nx, ny, 0, E, s);
  launch_k(lex_to_brick_kernel, (unsigned)nowned, 256, 0, s, lex, bricks, coord, nx, ny);
  return cudaGetLastError();
}

cudaError_t launch_brick_to_lex(const double* bricks, double* lex, const int32_t* coord, int64_t nowned, int nx,
                                int ny, cudaStream_t s, int E) {
  if (nowned <= 0) return cudaSuccess;
  if (E != 8) return launch_glex(bricks, lex, coord, nowned, nx, ny, 1, E, s);
  launch_k(brick_to_lex_kernel, (unsigned)nowned, 256, 0, s, bricks, lex, coord, nx, ny);
  return cudaGetLastError();
}

// blockIdx.y = run; the x-blocks stride over its 16-byte words
// Mirror exchange (reading A22, method of images): one CTA per domain-face ghost brick, two cells per
// thread; the cell (i, j, k) of the ghost brick takes cell (i', j', k') of its source brick, i' = 7 - i
// on a reflected axis, negated once per reflection for Dirichlet (negation is exact).
__global__ void __launch_bounds__(256) mirror_kernel(double* __restrict__ f, const int32_t* __restrict__ tab,
                                                     double sign) {
  pdl_begin();
  const int e = blockIdx.x, t = threadIdx.x;
  const int dst = __ldg(tab + 3 * e), src = __ldg(tab + 3 * e + 1), mask = __ldg(tab + 3 * e + 2);
  const double s = (__popc(mask) & 1) ? sign : 1.0;
#pragma unroll
  for (int h = 0; h < 2; ++h) {
    const int c = t + 256 * h;
    const int i = c & 7, j = (c >> 3) & 7, k = c >> 6;
    const int is = (mask & 1) ? 7 - i : i, js = (mask & 2) ? 7 - j : j, ks = (mask & 4) ? 7 - k : k;
    const double v = f[(int64_t)src * 512 + is + 8 * js + 64 * ks];
    f[(int64_t)dst * 512 + c] = s < 0.0 ? -v : v;
  }
}

cudaError_t launch_mirror(double* f, const int32_t* table, int n, double sign, cudaStream_t s, int E) {
  if (n <= 0) return cudaSuccess;
  if (E != 8) return launch_gmirror(f, table, n, sign, E, s);
  launch_k(mirror_kernel, (unsigned)n, 256, 0, s, f, table, sign);
  return cudaGetLastError();
}

__global__ void __launch_bounds__(256) copy_runs_kernel(const CopyRun* __restrict__ runs) {
  pdl_begin();
  const CopyRun r = runs[blockIdx.y];
  copy_run_body<false>(r, (int64_t)blockIdx.x * blockDim.x + threadIdx.x, (int64_t)gridDim.x * blockDim.x);
}

cudaError_t launch_copy_runs(const CopyRun* runs, int nruns, int64_t max_n, cudaStream_t s) {
  if (nruns <= 0 || max_n <= 0) return cudaSuccess;
  // about 4 waves of 256-thread blocks over the whole exchange, at least one block per run
  const int64_t words = max_n / 2;
  const int64_t want = (int64_t)148 * 8 * 4 / nruns;
  const unsigned gx = (unsigned)std::max<int64_t>(1, std::min<int64_t>((words + 255) / 256, std::max<int64_t>(1, want)));
  launch_k(copy_runs_kernel, dim3(gx, (unsigned)nruns), 256, 0, s, runs);
  return cudaGetLastError();
}

cudaError_t kernels_init() {
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  e = cudaDeviceGetAttribute(&g_num_sms, cudaDevAttrMultiProcessorCount, dev);
  if (e != cudaSuccess) return e;
#define COL_ATTR(F)                                                                                        \
  e = cudaFuncSetAttribute(sweep_col_kernel<(F)>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)col_smem<(F)>()); \
  if (e != cudaSuccess) return e;                                                                           \
  e = cudaFuncSetAttribute(sweep_col_kernel<(F)>, cudaFuncAttributePreferredSharedMemoryCarveout, 100);       \
  if (e != cudaSuccess) return e;
  COL_FLAG_LIST(COL_ATTR)
#undef COL_ATTR
  e = cudaFuncSetAttribute(bottom_resident_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                           kResidentMaxBricks * 512 * 2 * (int)sizeof(double));
  if (e != cudaSuccess) return e;
  e = pair_kernels_init();
  if (e != cudaSuccess) return e;
  e = pencil_kernels_init();
  if (e != cudaSuccess) return e;
  e = coarse_kernels_init();
  if (e != cudaSuccess) return e;
  e = bottom_cluster_init();
  if (e != cudaSuccess) return e;
  e = cg_kernels_init();
  if (e != cudaSuccess) return e;
  return coarse_grid_init();
}

}  // namespace mgb
