// generic.cu -- the brick kernels for a brick edge E other than 8 (E = 4: the paper's Sunspot
// configuration, "a brick size of 4x4x4 on Sunspot"; SURVEY §8(f) N4 "4^3 bricks").
//
// The layout, exchange plans, schedule and arithmetic are those of the 8^3 path (the brick edge is a
// layout parameter, Layout::E); only the kernels that index inside a brick change.  A 4^3 brick is 64
// doubles (512 B), so one CTA of 256 threads takes BPC = 512 / E^3 = 8 bricks (two cells per thread,
// a warp per brick) instead of one: the same cells per CTA as the one-brick-per-CTA kernels of
// kernels.cu, whose structure these follow (brick + six face halos staged in shared memory through
// the adjacency table; the canonical expression DAG of reading A8 / A23, so the results are bitwise
// those of the 8^3 path and of the lexicographic reference).  The 8^3-specific kernels (TMA column sweeps, two-sweep
// pencil passes, resident / cluster / CG bottoms) are not used with E = 4 (mg_setup forces the
// one-brick kernel family and per-sweep bottoms).
#include <cuda_runtime.h>

#include <cstdint>

#include "kernels.h"
#include "ptx.cuh"

namespace mgb {

namespace {

enum { G_SWEEP = 0, G_APPLY = 1, G_NORM = 2 };

template <int E>
struct Geo {
  static constexpr int V = E * E * E;   // doubles per brick
  static constexpr int F = E * E;       // cells per face
  static constexpr int BPC = 512 / V;   // bricks per 256-thread CTA
  static constexpr int TPB = V / 2;     // threads per brick (two cells each)
  static constexpr int H = E / 2;       // coarse cells per brick octant edge
};

__device__ __forceinline__ double g_nan_max(double a, double b) { return (b > a || b != b) ? b : a; }

// offset in the coarse brick of the coarse cell over fine cell (i, j, k) of octant oct
template <int E>
__device__ __forceinline__ int g_coarse_off(int oct, int i, int j, int k) {
  constexpr int H = E / 2;
  const int ox = oct & 1, oy = (oct >> 1) & 1, oz = oct >> 2;
  return (H * ox + (i >> 1)) + E * (H * oy + (j >> 1)) + E * E * (H * oz + (k >> 1));
}

template <int E, int MODE, unsigned FLAGS>
__global__ void __launch_bounds__(256) gsweep_kernel(SweepArgs p, unsigned long long* acc) {
  using G = Geo<E>;
  pdl_begin();
  constexpr bool WRITE_R = (FLAGS & SW_WRITE_R) != 0;
  constexpr bool RESTRICT = (FLAGS & SW_RESTRICT) != 0;
  constexpr bool INTERP = (FLAGS & SW_INTERP) != 0;
  constexpr bool ZERO_X = (FLAGS & SW_ZERO_X) != 0;
  constexpr bool VC = (FLAGS & SW_VARCOEF) != 0;
  __shared__ __align__(16) double xs[G::BPC][G::V];
  __shared__ double hx[G::BPC][6][G::F];
  __shared__ __align__(16) double cs[VC ? G::BPC : 1][VC ? G::V : 2];
  __shared__ double hc[VC ? G::BPC : 1][VC ? 6 : 1][VC ? G::F : 1];
  __shared__ __align__(16) double rs[RESTRICT ? G::BPC : 1][RESTRICT ? G::V : 2];
  __shared__ double wm[8];

  const int t = threadIdx.x, qb = t / G::TPB, u = t % G::TPB;
  const int64_t brick = p.brick0 + (int64_t)blockIdx.x * G::BPC + qb;
  const bool live = brick < p.brick0 + p.nbricks;
  const int c0 = 2 * u, i0 = c0 % E, j = (c0 / E) % E, k = c0 / (E * E);
  const int32_t* adj = p.adj + brick * 8;

  // the cell of face f's neighbour brick next to halo entry e (W/E: (j, k), S/N: (i, k), B/T: (i, j))
  auto face_cell = [](int f, int e) {
    const int a = e % E, b = e / E;
    if (f < 2) return (f == 0 ? E - 1 : 0) + E * a + E * E * b;
    if (f < 4) return a + E * (f == 2 ? E - 1 : 0) + E * E * b;
    return a + E * b + E * E * (f == 4 ? E - 1 : 0);
  };

  double2 bv = make_double2(0.0, 0.0);
  if (MODE != G_APPLY && live) bv = ld_stream2(p.b + brick * G::V + c0);
  if (!ZERO_X) {
    if (live) {
      double2 xv = ldg2(p.x + brick * G::V + c0);
      if (INTERP) {
        const int pr = __ldg(p.parent + brick);
        if (pr >= 0) {
          const double cv = __ldg(p.xc + (int64_t)(pr >> 3) * G::V + g_coarse_off<E>(pr & 7, i0, j, k));
          xv.x = DADD(xv.x, cv);
          xv.y = DADD(xv.y, cv);
        }
      }
      xs[qb][c0] = xv.x;
      xs[qb][c0 + 1] = xv.y;
      for (int m = u; m < 6 * G::F; m += G::TPB) {
        const int f = m / G::F, e = m % G::F;
        const int nb = __ldg(adj + f);
        const int cc = face_cell(f, e);
        double v = __ldg(p.x + (int64_t)nb * G::V + cc);
        if (INTERP) {
          const int pr = __ldg(p.parent + nb);
          if (pr >= 0)
            v = DADD(v, __ldg(p.xc + (int64_t)(pr >> 3) * G::V +
                                  g_coarse_off<E>(pr & 7, cc % E, (cc / E) % E, cc / (E * E))));
        }
        hx[qb][f][e] = v;
      }
    }
    __syncthreads();
  }
  if (VC) {
    if (live) {
      const double2 cv = ldg2(p.cf + brick * G::V + c0);
      cs[qb][c0] = cv.x;
      cs[qb][c0 + 1] = cv.y;
      for (int m = u; m < 6 * G::F; m += G::TPB) {
        const int f = m / G::F, e = m % G::F;
        hc[qb][f][e] = __ldg(p.cf + (int64_t)__ldg(adj + f) * G::V + face_cell(f, e));
      }
    }
    __syncthreads();
  }

  double out[2], res[2];
  double mx = 0.0;
#pragma unroll
  for (int ii = 0; ii < 2; ++ii) {
    const int i = i0 + ii;
    const int o = i + E * j + E * E * k;
    double c, w, e, s, n, bt, tp;
    if (ZERO_X) {
      c = w = e = s = n = bt = tp = 0.0;
    } else {
      c = xs[qb][o];
      w = i > 0 ? xs[qb][o - 1] : hx[qb][0][j + E * k];
      e = i < E - 1 ? xs[qb][o + 1] : hx[qb][1][j + E * k];
      s = j > 0 ? xs[qb][o - E] : hx[qb][2][i + E * k];
      n = j < E - 1 ? xs[qb][o + E] : hx[qb][3][i + E * k];
      bt = k > 0 ? xs[qb][o - E * E] : hx[qb][4][i + E * j];
      tp = k < E - 1 ? xs[qb][o + E * E] : hx[qb][5][i + E * j];
    }
    double a, gam = p.c.gamma;
    if (VC) {  // reading A23 (the expression of kernels.cu sweep_kernel<..., SW_VARCOEF>)
      const double cp = cs[qb][o];
      const double cw = i > 0 ? cs[qb][o - 1] : hc[qb][0][j + E * k];
      const double ce = i < E - 1 ? cs[qb][o + 1] : hc[qb][1][j + E * k];
      const double cS = j > 0 ? cs[qb][o - E] : hc[qb][2][i + E * k];
      const double cN = j < E - 1 ? cs[qb][o + E] : hc[qb][3][i + E * k];
      const double cB = k > 0 ? cs[qb][o - E * E] : hc[qb][4][i + E * j];
      const double cT = k < E - 1 ? cs[qb][o + E * E] : hc[qb][5][i + E * j];
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
    const double bb = ii ? bv.y : bv.x;
    if (MODE == G_APPLY) {
      out[ii] = a;
    } else if (MODE == G_NORM) {
      if (live) mx = g_nan_max(mx, fabs(DSUB(bb, a)));
    } else {
      res[ii] = DSUB(bb, a);
      out[ii] = keep_cell(p.colour, i, j, k) ? c : DADD(c, DMUL(gam, DSUB(a, bb)));
    }
  }

  if (MODE == G_NORM) {
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) mx = g_nan_max(mx, __shfl_xor_sync(0xffffffffu, mx, off));
    if ((t & 31) == 0) wm[t >> 5] = mx;
    __syncthreads();
    if (t == 0) {
      double m = wm[0];
      for (int q = 1; q < 8; ++q) m = g_nan_max(m, wm[q]);
      atomicMax(acc, (unsigned long long)__double_as_longlong(m));
    }
    return;
  }
  if (live) {
    st_stream2(p.xo + brick * G::V + c0, make_double2(out[0], out[1]));
    if (MODE == G_SWEEP && WRITE_R) st_stream2(p.r + brick * G::V + c0, make_double2(res[0], res[1]));
  }
  if (MODE == G_SWEEP && RESTRICT) {
    rs[qb][c0] = res[0];
    rs[qb][c0 + 1] = res[1];
    __syncthreads();
    constexpr int NC = G::V / 8;  // coarse cells per fine brick
    for (int m = t; m < G::BPC * NC; m += 256) {
      const int q = m / NC, ec = m % NC;
      const int64_t fb = p.brick0 + (int64_t)blockIdx.x * G::BPC + q;
      if (fb >= p.brick0 + p.nbricks) continue;
      const int I = ec % G::H, J = (ec / G::H) % G::H, K = ec / (G::H * G::H);
      const int f = 2 * I + E * 2 * J + E * E * 2 * K;
      const double* R = rs[q];
      const double v = DMUL(0.125, DADD(DADD(DADD(R[f], R[f + 1]), DADD(R[f + E], R[f + E + 1])),
                                        DADD(DADD(R[f + E * E], R[f + E * E + 1]),
                                             DADD(R[f + E * E + E], R[f + E * E + E + 1]))));
      const int pr = __ldg(p.parent + fb);
      const int oct = pr & 7, ox = oct & 1, oy = (oct >> 1) & 1, oz = oct >> 2;
      p.bc[(int64_t)(pr >> 3) * G::V + (G::H * ox + I) + E * (G::H * oy + J) + E * E * (G::H * oz + K)] = v;
    }
  }
}

// restriction: one thread per coarse cell of a fine brick's octant (canonical pairwise order)
template <int E>
__global__ void __launch_bounds__(256) grestrict_kernel(const double* __restrict__ r, double* __restrict__ bc,
                                                        const int32_t* __restrict__ parent, int64_t nfine) {
  using G = Geo<E>;
  pdl_begin();
  constexpr int NC = G::V / 8;
  const int64_t m = (int64_t)blockIdx.x * 256 + threadIdx.x;
  if (m >= nfine * NC) return;
  const int64_t fb = m / NC;
  const int ec = (int)(m % NC);
  const int I = ec % G::H, J = (ec / G::H) % G::H, K = ec / (G::H * G::H);
  const double* R = r + fb * G::V + 2 * I + E * 2 * J + E * E * 2 * K;
  const double v = DMUL(0.125, DADD(DADD(DADD(R[0], R[1]), DADD(R[E], R[E + 1])),
                                    DADD(DADD(R[E * E], R[E * E + 1]), DADD(R[E * E + E], R[E * E + E + 1]))));
  const int pr = __ldg(parent + fb);
  const int oct = pr & 7, ox = oct & 1, oy = (oct >> 1) & 1, oz = oct >> 2;
  bc[(int64_t)(pr >> 3) * G::V + (G::H * ox + I) + E * (G::H * oy + J) + E * E * (G::H * oz + K)] = v;
}

// interpolation+increment: one thread per fine cell pair
template <int E>
__global__ void __launch_bounds__(256) ginterp_kernel(double* __restrict__ x, const double* __restrict__ xc,
                                                      const int32_t* __restrict__ parent, int64_t nfine) {
  using G = Geo<E>;
  pdl_begin();
  const int64_t m = (int64_t)blockIdx.x * 256 + threadIdx.x;
  if (m >= nfine * G::TPB) return;
  const int64_t fb = m / G::TPB;
  const int c0 = 2 * (int)(m % G::TPB), i0 = c0 % E, j = (c0 / E) % E, k = c0 / (E * E);
  const int pr = __ldg(parent + fb);
  const double cv = __ldg(xc + (int64_t)(pr >> 3) * G::V + g_coarse_off<E>(pr & 7, i0, j, k));
  double2* px = reinterpret_cast<double2*>(x + fb * G::V + c0);
  double2 v = *px;
  v.x = DADD(v.x, cv);
  v.y = DADD(v.y, cv);
  *px = v;
}

// lexicographic <-> bricks (one thread per cell pair); dir 0: lex -> bricks, 1: bricks -> lex
template <int E>
__global__ void __launch_bounds__(256) glex_kernel(const double* __restrict__ src, double* __restrict__ dst,
                                                   const int32_t* __restrict__ coord, int64_t nowned, int nx, int ny,
                                                   int dir) {
  using G = Geo<E>;
  pdl_begin();
  const int64_t m = (int64_t)blockIdx.x * 256 + threadIdx.x;
  if (m >= nowned * G::TPB) return;
  const int64_t bI = m / G::TPB;
  const int c0 = 2 * (int)(m % G::TPB), i0 = c0 % E, j = (c0 / E) % E, k = c0 / (E * E);
  const int cx = coord[bI * 3], cy = coord[bI * 3 + 1], cz = coord[bI * 3 + 2];
  const int64_t li = (int64_t)(E * cx + i0) + (int64_t)nx * ((int64_t)(E * cy + j) + (int64_t)ny * (E * cz + k));
  if (dir == 0)
    *reinterpret_cast<double2*>(dst + bI * G::V + c0) = *reinterpret_cast<const double2*>(src + li);
  else
    *reinterpret_cast<double2*>(dst + li) = *reinterpret_cast<const double2*>(src + bI * G::V + c0);
}

// mirror exchange (reading A22): one thread per cell of a domain-face ghost brick
template <int E>
__global__ void __launch_bounds__(256) gmirror_kernel(double* __restrict__ f, const int32_t* __restrict__ tab,
                                                      int64_t n, double sign) {
  using G = Geo<E>;
  pdl_begin();
  const int64_t m = (int64_t)blockIdx.x * 256 + threadIdx.x;
  if (m >= n * G::V) return;
  const int64_t e = m / G::V;
  const int c = (int)(m % G::V), i = c % E, j = (c / E) % E, k = c / (E * E);
  const int dst = __ldg(tab + 3 * e), src = __ldg(tab + 3 * e + 1), mask = __ldg(tab + 3 * e + 2);
  const int is = (mask & 1) ? E - 1 - i : i, js = (mask & 2) ? E - 1 - j : j, ks = (mask & 4) ? E - 1 - k : k;
  const double v = f[(int64_t)src * G::V + is + E * js + E * E * ks];
  f[(int64_t)dst * G::V + c] = ((__popc(mask) & 1) && sign < 0.0) ? -v : v;
}

// the paper's pointwise smooth(+residual) (MG_FUSION_PAPER): one thread per cell pair
template <int E, bool WRITE_R>
__global__ void __launch_bounds__(256) gsmooth_kernel(double* __restrict__ x, const double* __restrict__ Ax,
                                                      const double* __restrict__ b, double* __restrict__ r,
                                                      int64_t base, int64_t n2, double gamma, int colour) {
  using G = Geo<E>;
  pdl_begin();
  const int64_t q = (int64_t)blockIdx.x * 256 + threadIdx.x;
  if (q >= n2) return;
  const int64_t o = base + 2 * q;
  const double2 xv = ldg2(x + o), av = ld_stream2(Ax + o), bv = ld_stream2(b + o);
  const int c = (int)(o % G::V), i = c % E, j = (c / E) % E, k = c / (E * E);
  double2 xn;
  xn.x = keep_cell(colour, i, j, k) ? xv.x : DADD(xv.x, DMUL(gamma, DSUB(av.x, bv.x)));
  xn.y = keep_cell(colour, i + 1, j, k) ? xv.y : DADD(xv.y, DMUL(gamma, DSUB(av.y, bv.y)));
  st_stream2(x + o, xn);
  if (WRITE_R) st_stream2(r + o, make_double2(DSUB(bv.x, av.x), DSUB(bv.y, av.y)));
}

unsigned blocks(int64_t threads) { return (unsigned)((threads + 255) / 256); }

template <int E, int MODE, unsigned F>
cudaError_t gsweep_launch(const SweepArgs& a, unsigned long long* acc, cudaStream_t s) {
  launch_k(gsweep_kernel<E, MODE, F>, (unsigned)((a.nbricks + Geo<E>::BPC - 1) / Geo<E>::BPC), 256, 0, s, a, acc);
  return cudaGetLastError();
}

}  // namespace

cudaError_t launch_gsweep(const SweepArgs& a, unsigned flags, int mode, unsigned long long* acc, cudaStream_t s) {
  if (a.nbricks <= 0) return cudaSuccess;
  if (a.E != 4) return cudaErrorInvalidValue;
  const unsigned vc = (flags & SW_VARCOEF) ? SW_VARCOEF : 0u;
  if (mode == 1) return vc ? gsweep_launch<4, G_APPLY, SW_VARCOEF>(a, acc, s) : gsweep_launch<4, G_APPLY, 0>(a, acc, s);
  if (mode == 2) return vc ? gsweep_launch<4, G_NORM, SW_VARCOEF>(a, acc, s) : gsweep_launch<4, G_NORM, 0>(a, acc, s);
  switch ((flags & (SW_WRITE_R | SW_RESTRICT | SW_INTERP | SW_ZERO_X)) | vc) {
#define GCASE(F) \
  case (F): return gsweep_launch<4, G_SWEEP, (F)>(a, acc, s);
#define GCASES(V)                                                                                   \
  GCASE(0 | V) GCASE(SW_WRITE_R | V) GCASE(SW_RESTRICT | V) GCASE(SW_INTERP | V)                   \
  GCASE(SW_INTERP | SW_WRITE_R | V) GCASE(SW_INTERP | SW_RESTRICT | V) GCASE(SW_ZERO_X | V)         \
  GCASE(SW_ZERO_X | SW_WRITE_R | V) GCASE(SW_ZERO_X | SW_RESTRICT | V)
    GCASES(0u)
    GCASES(SW_VARCOEF)
#undef GCASES
#undef GCASE
    default:
      return cudaErrorInvalidValue;
  }
}

cudaError_t launch_grestrict(const double* r, double* bc, const int32_t* parent, int64_t nfine, int E,
                             cudaStream_t s) {
  if (nfine <= 0) return cudaSuccess;
  if (E != 4) return cudaErrorInvalidValue;
  launch_k(grestrict_kernel<4>, blocks(nfine * (Geo<4>::V / 8)), 256, 0, s, r, bc, parent, nfine);
  return cudaGetLastError();
}

cudaError_t launch_ginterp(double* x, const double* xc, const int32_t* parent, int64_t nfine, int E, cudaStream_t s) {
  if (nfine <= 0) return cudaSuccess;
  if (E != 4) return cudaErrorInvalidValue;
  launch_k(ginterp_kernel<4>, blocks(nfine * Geo<4>::TPB), 256, 0, s, x, xc, parent, nfine);
  return cudaGetLastError();
}

cudaError_t launch_glex(const double* src, double* dst, const int32_t* coord, int64_t nowned, int nx, int ny,
                        int dir, int E, cudaStream_t s) {
  if (nowned <= 0) return cudaSuccess;
  if (E != 4) return cudaErrorInvalidValue;
  launch_k(glex_kernel<4>, blocks(nowned * Geo<4>::TPB), 256, 0, s, src, dst, coord, nowned, nx, ny, dir);
  return cudaGetLastError();
}

cudaError_t launch_gmirror(double* f, const int32_t* table, int n, double sign, int E, cudaStream_t s) {
  if (n <= 0) return cudaSuccess;
  if (E != 4) return cudaErrorInvalidValue;
  launch_k(gmirror_kernel<4>, blocks((int64_t)n * Geo<4>::V), 256, 0, s, f, table, (int64_t)n, sign);
  return cudaGetLastError();
}

cudaError_t launch_gsmooth(double* x, const double* Ax, const double* b, double* r, int64_t brick0, int64_t nbricks,
                           Coeffs c, bool write_r, int colour, int E, cudaStream_t s) {
  if (nbricks <= 0) return cudaSuccess;
  if (E != 4) return cudaErrorInvalidValue;
  const int64_t n2 = nbricks * Geo<4>::TPB, base = brick0 * Geo<4>::V;
  if (write_r)
    launch_k(gsmooth_kernel<4, true>, blocks(n2), 256, 0, s, x, Ax, b, r, base, n2, c.gamma, colour);
  else
    launch_k(gsmooth_kernel<4, false>, blocks(n2), 256, 0, s, x, Ax, b, r, base, n2, c.gamma, colour);
  return cudaGetLastError();
}

}  // namespace mgb
