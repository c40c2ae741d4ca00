// sweep2.cu -- two Jacobi sweeps per HBM pass (temporal blocking).
//
// The paper deepens the ghost zone to a brick so several smooths run per
// exchange; this kernel applies the same idea on chip: x0 -> x1 -> x2
// in one pass over HBM (read x0, b; write x2: 24 B per point for TWO sweeps).
// Each sweep is exactly the canonical smooth(+residual) of kernels.cu (reading
// A8), so x2 is bit-identical to two separate sweeps.
//
// One CTA (4 warps) walks an item stream of z-chain runs (layout.cpp
// pair_table): [warm-up, bricks..., cool-down] ...  Per item m, lane 0 of each
// warp stages its share by TMA into a 4-stage shared-memory ring (mbarriers):
//   the x0 brick (1D bulk, 4 KiB); 2-cell-deep x0 slabs of the W/E/S/N
//   neighbours (3D tensor boxes {2,8,8} / {8,2,8}); the b values on those faces
//   ({2,8,8} / {8,1,8}); the x0 columns of the 4 diagonal neighbours ({2,1,8}).
// Step m runs, between two CTA barriers,
//   phase A: x1 of item m on its 512 cells (warp w = planes 2w, 2w+1, register
//            k-streaming) and -- redundantly -- on the 4 x 64 side-face cells of
//            its neighbours (warp w = face w), whose x1 the second sweep needs;
//   phase B: x2 of item m-2 from x1 (its cells, its faces, plane 7 of item m-3,
//            plane 0 of item m-1), streamed to HBM with r or the restricted
//            coarse b on the last sweep of a phase;
// with x1 in a 3-deep shared ring so the phases never touch the same buffer.
// Shared-memory operand offsets are loop invariants computed once per thread.
// b of the own cells travels in registers (128-bit loads two items ahead).
#include <cudaTypedefs.h>

#include <cstddef>

#include "kernels.h"
#include "ptx.cuh"

namespace mgb {

constexpr int P2_NST = 4;     // TMA ring: items m, m+1 read; m+2, m+3 in flight
constexpr int P2_RING = 8;    // metadata ring (items m-3 .. m+4)
constexpr int P2_META = 11;   // id, flags, W,E,S,N, SW,NW,SE,NE, parent
constexpr int P2_WARPS = 4;
constexpr int P2_THREADS = 32 * P2_WARPS;

struct P2Stage {
  double x[512];              // x0 of the item brick, cell i + 8j + 64k
  double xwe[2][8][8][2];     // x0 of the W brick (i = 6,7) / E brick (i = 0,1): [k][j][ii]
  double xsn[2][8][2][8];     // x0 of the S brick (j = 6,7) / N brick (j = 0,1): [k][jj][i]
  double bwe[2][8][8][2];     // b  of the W brick (i = 6,7) / E brick (i = 0,1)
  double bsn[2][8][8];        // b  of the S brick (j = 7) / N brick (j = 0): [k][i]
  double cor[4][8][2];        // x0 columns: SW (i=6,7 j=7), NW (i=6,7 j=0), SE (i=0,1 j=7), NE (i=0,1 j=0)
};
static_assert(sizeof(P2Stage) % 128 == 0, "stage must keep TMA destinations 128-byte aligned");
// the four warps' expect_tx byte counts below add up to the whole stage
static_assert(sizeof(P2Stage) == (4096 + 1024) + 3 * 1024 + (2048 + 512) + (512 + 512), "stage bytes");
// operand offsets (in doubles) inside a stage
constexpr int OX = 0, OXWE = 512, OXSN = 768, OBWE = 1024, OBSN = 1280, OCOR = 1408;
static_assert(offsetof(P2Stage, xwe) == OXWE * 8 && offsetof(P2Stage, xsn) == OXSN * 8 &&
                  offsetof(P2Stage, bwe) == OBWE * 8 && offsetof(P2Stage, bsn) == OBSN * 8 &&
                  offsetof(P2Stage, cor) == OCOR * 8,
              "stage layout");
__host__ __device__ constexpr int oxwe(int f, int k, int j, int ii) { return OXWE + 128 * f + 16 * k + 2 * j + ii; }
__host__ __device__ constexpr int oxsn(int f, int k, int jj, int i) { return OXSN + 128 * f + 16 * k + 8 * jj + i; }
__host__ __device__ constexpr int obwe(int f, int k, int j, int ii) { return OBWE + 128 * f + 16 * k + 2 * j + ii; }
__host__ __device__ constexpr int obsn(int f, int k, int i) { return OBSN + 64 * f + 8 * k + i; }
__host__ __device__ constexpr int ocor(int c, int k, int ii) { return OCOR + 16 * c + 2 * k + ii; }

template <bool RESTRICT>
struct P2Smem {
  P2Stage st[P2_NST];
  double A[3][512];       // x1 of items m-2, m-1, m
  double F[3][4][64];     // x1 on their side faces: W/E [k][j], S/N [k][i]
  double cx0[2][64];      // x0 plane 7 of the previous item
  double cbox[2][4][8];   // x0 plane 7 of the previous item's side-face cells (W/E by j, S/N by i)
  double cx1[2][64];      // x1 plane 7 of item m-3
  uint64_t bar[P2_NST];
  int meta[P2_RING][12];
};

__device__ __forceinline__ double2 lds2(const double* p) { return *reinterpret_cast<const double2*>(p); }

template <unsigned FLAGS>
__global__ void __launch_bounds__(P2_THREADS, 3)
    sweep2_kernel(SweepArgs p, PairArgs pa, const __grid_constant__ PairMaps mp) {
  constexpr bool WRITE_R = (FLAGS & SW_WRITE_R) != 0;
  constexpr bool RESTRICT = (FLAGS & SW_RESTRICT) != 0;
  extern __shared__ __align__(128) unsigned char smem_raw[];
  P2Smem<RESTRICT>& S = *reinterpret_cast<P2Smem<RESTRICT>*>(smem_raw);
  const int t = threadIdx.x, w = t >> 5, l = t & 31;
  const int2 cr = pa.ctas[blockIdx.x];
  const int64_t base = cr.x;
  const int cnt = cr.y;
  const double alpha = p.c.alpha, beta = p.c.beta, gamma = p.c.gamma;

  // ---- own-cell geometry: planes k0 = 2w, k1 = 2w+1; cell pair (i0, i0+1), row j ----
  const int i0 = 2 * (l & 3), j = l >> 2;
  const int q = 8 * j + i0;
  const int k0 = 2 * w;
  const int qs = j > 0 ? q - 8 : q, qn = j < 7 ? q + 8 : q;  // row loads (clamped; unused lanes)
  // ---- face-cell geometry: warp w = face f; lane = (c8, planes 2kq, 2kq+1) ----
  const int f = w, c8 = l & 7, kq = l >> 3, fk0 = 2 * kq;
  int oc[2], ow[2], oe[2], os[2], on[2], ob[2], ocm, ocp;  // stage offsets of the face operands
#pragma unroll
  for (int kk = 0; kk < 2; ++kk) {
    const int k = fk0 + kk;
    if (f == 0) {  // W brick, i = 7, (j = c8, k)
      oc[kk] = oxwe(0, k, c8, 1);
      ow[kk] = oxwe(0, k, c8, 0);
      oe[kk] = OX + 64 * k + 8 * c8;
      os[kk] = c8 > 0 ? oxwe(0, k, c8 - 1, 1) : ocor(0, k, 1);
      on[kk] = c8 < 7 ? oxwe(0, k, c8 + 1, 1) : ocor(1, k, 1);
      ob[kk] = obwe(0, k, c8, 1);
    } else if (f == 1) {  // E brick, i = 0
      oc[kk] = oxwe(1, k, c8, 0);
      oe[kk] = oxwe(1, k, c8, 1);
      ow[kk] = OX + 64 * k + 8 * c8 + 7;
      os[kk] = c8 > 0 ? oxwe(1, k, c8 - 1, 0) : ocor(2, k, 0);
      on[kk] = c8 < 7 ? oxwe(1, k, c8 + 1, 0) : ocor(3, k, 0);
      ob[kk] = obwe(1, k, c8, 0);
    } else if (f == 2) {  // S brick, j = 7, (i = c8, k)
      oc[kk] = oxsn(0, k, 1, c8);
      os[kk] = oxsn(0, k, 0, c8);
      on[kk] = OX + 64 * k + c8;
      ow[kk] = c8 > 0 ? oxsn(0, k, 1, c8 - 1) : ocor(0, k, 1);
      oe[kk] = c8 < 7 ? oxsn(0, k, 1, c8 + 1) : ocor(2, k, 0);
      ob[kk] = obsn(0, k, c8);
    } else {  // N brick, j = 0
      oc[kk] = oxsn(1, k, 0, c8);
      on[kk] = oxsn(1, k, 1, c8);
      os[kk] = OX + 64 * k + 56 + c8;
      ow[kk] = c8 > 0 ? oxsn(1, k, 0, c8 - 1) : ocor(1, k, 1);
      oe[kk] = c8 < 7 ? oxsn(1, k, 0, c8 + 1) : ocor(3, k, 0);
      ob[kk] = obsn(1, k, c8);
    }
  }
  {
    const int km = fk0 - 1, kp = fk0 + 2;  // c(k) at planes fk0-1 (kq > 0) / fk0+2 (kq < 3, else next stage plane 0)
    const int kpp = kq < 3 ? kp : 0;
    if (f == 0) {
      ocm = oxwe(0, km < 0 ? 0 : km, c8, 1);
      ocp = oxwe(0, kpp, c8, 1);
    } else if (f == 1) {
      ocm = oxwe(1, km < 0 ? 0 : km, c8, 0);
      ocp = oxwe(1, kpp, c8, 0);
    } else if (f == 2) {
      ocm = oxsn(0, km < 0 ? 0 : km, 1, c8);
      ocp = oxsn(0, kpp, 1, c8);
    } else {
      ocm = oxsn(1, km < 0 ? 0 : km, 0, c8);
      ocp = oxsn(1, kpp, 0, c8);
    }
  }

  for (int e = t; e < P2_RING * P2_META; e += P2_THREADS) {
    const int it = e / P2_META, fl = e % P2_META;
    if (it < cnt) S.meta[it][fl] = pa.meta[(base + it) * P2_META + fl];
  }
  if (t == 0) {
    for (int s = 0; s < P2_NST; ++s) mbar_init(&S.bar[s], P2_WARPS);  // one expect_tx arrive per warp
    mbar_fence_init();
  }
  __syncthreads();

  // lane 0 of every warp issues its share of item m's copies
  auto issue = [&](int m) {
    const int s = m % P2_NST;
    const int* M = S.meta[m % P2_RING];
    P2Stage& G = S.st[s];
    uint64_t* bar = &S.bar[s];
    if (w == 0) {
      mbar_expect_tx(bar, 4096 + 1024);
      tma_load_1d(G.x, p.x + (int64_t)M[0] * 512, 4096, bar);
      tma_load_3d(G.xwe[0], &mp.xwe, 6, 0, M[2] * 8, bar);  // W: i = 6,7
    } else if (w == 1) {
      mbar_expect_tx(bar, 3 * 1024);
      tma_load_3d(G.xwe[1], &mp.xwe, 0, 0, M[3] * 8, bar);  // E: i = 0,1
      tma_load_3d(G.xsn[0], &mp.xsn, 0, 6, M[4] * 8, bar);  // S: j = 6,7
      tma_load_3d(G.xsn[1], &mp.xsn, 0, 0, M[5] * 8, bar);  // N: j = 0,1
    } else if (w == 2) {
      mbar_expect_tx(bar, 2048 + 512);
      tma_load_3d(G.bwe[0], &mp.bwe, 6, 0, M[2] * 8, bar);
      tma_load_3d(G.bwe[1], &mp.bwe, 0, 0, M[3] * 8, bar);
      tma_load_3d(G.bsn[0], &mp.bsn, 0, 7, M[4] * 8, bar);
    } else {
      mbar_expect_tx(bar, 512 + 512);
      tma_load_3d(G.bsn[1], &mp.bsn, 0, 0, M[5] * 8, bar);
      tma_load_3d(G.cor[0], &mp.xcor, 6, 7, M[6] * 8, bar);  // SW: (i = 7, j = 7)
      tma_load_3d(G.cor[1], &mp.xcor, 6, 0, M[7] * 8, bar);  // NW: (i = 7, j = 0)
      tma_load_3d(G.cor[2], &mp.xcor, 0, 7, M[8] * 8, bar);  // SE: (i = 0, j = 7)
      tma_load_3d(G.cor[3], &mp.xcor, 0, 0, M[9] * 8, bar);  // NE: (i = 0, j = 0)
    }
  };
  // b of this thread's own cells (planes k0, k1) of item m
  auto load_b = [&](int m, double2& v0, double2& v1) {
    const double* bp = p.b + (int64_t)S.meta[m % P2_RING][0] * 512 + 64 * k0 + q;
    v0 = ld_stream2(bp);
    v1 = ld_stream2(bp + 64);
  };

  if (l == 0)
    for (int m = 0; m < 3 && m < cnt; ++m) issue(m);
  double2 bm2a = make_double2(0.0, 0.0), bm2b = bm2a, bm1a = bm2a, bm1b = bm2a, b0a, b0b, b1a, b1b;
  load_b(0, b0a, b0b);
  if (cnt > 1)
    load_b(1, b1a, b1b);
  else
    b1a = b0a, b1b = b0b;
  int mreg = 0;
  int a_cur = 0;  // m % 3 (x1 ring slot of item m)

  for (int m = 0; m <= cnt + 1; ++m) {
    const int a_m1 = a_cur == 0 ? 2 : a_cur - 1, a_m2 = a_m1 == 0 ? 2 : a_m1 - 1;
    const int cur = m & 1, prv = cur ^ 1;
    // metadata ring holds items m-3 .. m+3 during step m: store item m+4 (loaded last step)
    // into the slot of item m-4, then load item m+5 (fields spread over the warps)
    if (l < 3 && w + 4 * l < P2_META) {
      const int fl = w + 4 * l;
      if (m >= 1 && m + 4 < cnt) S.meta[(m + 4) % P2_RING][fl] = mreg;
      if (m + 5 < cnt) mreg = pa.meta[(base + m + 5) * P2_META + fl];
    }
    // stage of item m+3 = stage of item m-1, unread since the barrier that ended step m-1
    if (l == 0 && m + 3 < cnt) {
      fence_proxy_async();
      issue(m + 3);
    }
    double2 b2a = b1a, b2b = b1b;
    if (m + 2 < cnt) load_b(m + 2, b2a, b2b);

    // ---------------- phase A: x1 of item m ----------------
    if (m < cnt) {
      mbar_wait(&S.bar[m % P2_NST], (uint32_t)((m / P2_NST) & 1));
      if (m + 1 < cnt) mbar_wait(&S.bar[(m + 1) % P2_NST], (uint32_t)(((m + 1) / P2_NST) & 1));
      const double* G = reinterpret_cast<const double*>(&S.st[m % P2_NST]);
      const double* N = reinterpret_cast<const double*>(&S.st[(m + 1) % P2_NST]);  // stale if no next item
      double* Aw = S.A[a_cur];
      {  // own cells, planes k0, k1 (k-streaming in registers)
        const double2 xm = w > 0 ? lds2(G + 64 * (k0 - 1) + q) : lds2(S.cx0[prv] + q);
        const double2 x0 = lds2(G + 64 * k0 + q);
        const double2 x1 = lds2(G + 64 * (k0 + 1) + q);
        const double2 x2 = w < P2_WARPS - 1 ? lds2(G + 64 * (k0 + 2) + q) : lds2(N + q);
#pragma unroll
        for (int kk = 0; kk < 2; ++kk) {
          const int k = k0 + kk;
          const double2 xc = kk ? x1 : x0, xb = kk ? x0 : xm, xt = kk ? x2 : x1;
          const double2 bb = kk ? b0b : b0a;
          const double2 rs_ = lds2(G + 64 * k + qs), rn_ = lds2(G + 64 * k + qn);
          const double fw = G[oxwe(0, k, j, 1)], fe = G[oxwe(1, k, j, 0)];
          const double2 fs = lds2(G + oxsn(0, k, 1, i0)), fn = lds2(G + oxsn(1, k, 0, i0));
          const double wl = __shfl_up_sync(0xffffffffu, xc.y, 1);
          const double er = __shfl_down_sync(0xffffffffu, xc.x, 1);
          const double wv = i0 > 0 ? wl : fw, ev = i0 < 6 ? er : fe;
          const double2 sv = j > 0 ? rs_ : fs, nv = j < 7 ? rn_ : fn;
          const double a0 = stencil_a(xc.x, wv, xc.y, sv.x, nv.x, xb.x, xt.x, alpha, beta);
          const double a1 = stencil_a(xc.y, xc.x, ev, sv.y, nv.y, xb.y, xt.y, alpha, beta);
          double2 y;
          y.x = DADD(xc.x, DMUL(gamma, DSUB(a0, bb.x)));
          y.y = DADD(xc.y, DMUL(gamma, DSUB(a1, bb.y)));
          *reinterpret_cast<double2*>(Aw + 64 * k + q) = y;
        }
        if (w == P2_WARPS - 1) *reinterpret_cast<double2*>(S.cx0[cur] + q) = x1;  // plane 7
      }
      {  // side-face cells of the neighbours: face f = w, planes fk0, fk0+1 at in-face c8
        const double cm = kq > 0 ? G[ocm] : S.cbox[prv][f][c8];
        const double c0 = G[oc[0]], c1 = G[oc[1]];
        const double cp = kq < 3 ? G[ocp] : N[ocp];
#pragma unroll
        for (int kk = 0; kk < 2; ++kk) {
          const double c = kk ? c1 : c0, bt = kk ? c0 : cm, tp = kk ? cp : c1;
          const double av = stencil_a(c, G[ow[kk]], G[oe[kk]], G[os[kk]], G[on[kk]], bt, tp, alpha, beta);
          S.F[a_cur][f][8 * (fk0 + kk) + c8] = DADD(c, DMUL(gamma, DSUB(av, G[ob[kk]])));
        }
        if (kq == 3) S.cbox[cur][f][c8] = c1;  // plane 7
      }
    }

    // ---------------- phase B: x2 of item m-2 ----------------
    if (m >= 2 && m <= cnt) {
      const double* P = S.A[a_m2];
      const double2 x1v = lds2(P + 64 * (k0 + 1) + q);
      if (w == P2_WARPS - 1) *reinterpret_cast<double2*>(S.cx1[cur] + q) = x1v;  // x1 plane 7 of item m-2
      const bool emit = (S.meta[(m - 1) % P2_RING][1] & 1) != 0;  // item m-2 is a range brick
      if (emit) {
        const double2 xm = w > 0 ? lds2(P + 64 * (k0 - 1) + q) : lds2(S.cx1[prv] + q);  // item m-3 plane 7
        const double2 x0v = lds2(P + 64 * k0 + q);
        const double2 x2v = w < P2_WARPS - 1 ? lds2(P + 64 * (k0 + 2) + q) : lds2(S.A[a_m1] + q);  // item m-1
        const double* Fb = &S.F[a_m2][0][0];
        const int64_t g = (int64_t)S.meta[(m - 2) % P2_RING][0] * 512 + q;
        double rsum[2];
#pragma unroll
        for (int kk = 0; kk < 2; ++kk) {
          const int k = k0 + kk;
          const double2 xc = kk ? x1v : x0v, xb = kk ? x0v : xm, xt = kk ? x2v : x1v;
          const double2 bb = kk ? bm2b : bm2a;
          const double2 rs_ = lds2(P + 64 * k + qs), rn_ = lds2(P + 64 * k + qn);
          const double fw = Fb[8 * k + j], fe = Fb[64 + 8 * k + j];
          const double2 fs = lds2(Fb + 128 + 8 * k + i0), fn = lds2(Fb + 192 + 8 * k + i0);
          const double wl = __shfl_up_sync(0xffffffffu, xc.y, 1);
          const double er = __shfl_down_sync(0xffffffffu, xc.x, 1);
          const double wv = i0 > 0 ? wl : fw, ev = i0 < 6 ? er : fe;
          const double2 sv = j > 0 ? rs_ : fs, nv = j < 7 ? rn_ : fn;
          const double a0 = stencil_a(xc.x, wv, xc.y, sv.x, nv.x, xb.x, xt.x, alpha, beta);
          const double a1 = stencil_a(xc.y, xc.x, ev, sv.y, nv.y, xb.y, xt.y, alpha, beta);
          double2 y, rv;
          y.x = DADD(xc.x, DMUL(gamma, DSUB(a0, bb.x)));
          y.y = DADD(xc.y, DMUL(gamma, DSUB(a1, bb.y)));
          rv.x = DSUB(bb.x, a0);
          rv.y = DSUB(bb.y, a1);
          st_stream2(p.xo + g + 64 * k, y);
          if (WRITE_R) st_stream2(p.r + g + 64 * k, rv);
          rsum[kk] = DADD(rv.x, rv.y);  // r(2I,.,.) + r(2I+1,.,.) of this row and plane
        }
        if (RESTRICT) {
          // coarse cell (I, J, K) = (l&3, j/2, w): its 8 fine cells are this lane's and lane+4's
          // pairs on planes 2w, 2w+1 -> canonical order ((r000+r100)+(r010+r110))+((r001+r101)+(r011+r111))
          const double s0n = __shfl_down_sync(0xffffffffu, rsum[0], 4);
          const double s1n = __shfl_down_sync(0xffffffffu, rsum[1], 4);
          if ((j & 1) == 0) {
            const double v = DMUL(0.125, DADD(DADD(rsum[0], s0n), DADD(rsum[1], s1n)));
            const int pr = S.meta[(m - 2) % P2_RING][10];
            const int oct = pr & 7;
            const int ox = oct & 1, oy = (oct >> 1) & 1, oz = oct >> 2;
            p.bc[(int64_t)(pr >> 3) * 512 + (4 * ox + (l & 3)) + 8 * (4 * oy + (j >> 1)) + 64 * (4 * oz + w)] = v;
          }
        }
      }
    }
    __syncthreads();
    bm2a = bm1a, bm2b = bm1b;
    bm1a = b0a, bm1b = b0b;
    b0a = b1a, b0b = b1b;
    b1a = b2a, b1b = b2b;
    a_cur = a_cur == 2 ? 0 : a_cur + 1;
  }
}

bool pair_supports(unsigned flags) {
  const unsigned fl = flags & (SW_WRITE_R | SW_RESTRICT | SW_INTERP | SW_ZERO_X);
  return fl == 0 || fl == SW_WRITE_R || fl == SW_RESTRICT;
}

cudaError_t launch_sweep2(const SweepArgs& a, const PairArgs& pa, const PairMaps& pm, unsigned flags,
                          cudaStream_t s) {
  if (pa.nctas <= 0) return cudaSuccess;
  const unsigned g = (unsigned)pa.nctas;
  switch (flags & (SW_WRITE_R | SW_RESTRICT | SW_INTERP | SW_ZERO_X)) {
    case 0: sweep2_kernel<0><<<g, P2_THREADS, sizeof(P2Smem<false>), s>>>(a, pa, pm); break;
    case SW_WRITE_R: sweep2_kernel<SW_WRITE_R><<<g, P2_THREADS, sizeof(P2Smem<false>), s>>>(a, pa, pm); break;
    case SW_RESTRICT: sweep2_kernel<SW_RESTRICT><<<g, P2_THREADS, sizeof(P2Smem<true>), s>>>(a, pa, pm); break;
    default: return cudaErrorInvalidValue;
  }
  return cudaGetLastError();
}

cudaError_t pair_kernels_init() {
  const void* k[3] = {(const void*)sweep2_kernel<0>, (const void*)sweep2_kernel<SW_WRITE_R>,
                      (const void*)sweep2_kernel<SW_RESTRICT>};
  const int sm[3] = {(int)sizeof(P2Smem<false>), (int)sizeof(P2Smem<false>), (int)sizeof(P2Smem<true>)};
  for (int i = 0; i < 3; ++i) {
    cudaError_t e = cudaFuncSetAttribute(k[i], cudaFuncAttributeMaxDynamicSharedMemorySize, sm[i]);
    if (e != cudaSuccess) return e;
    e = cudaFuncSetAttribute(k[i], cudaFuncAttributePreferredSharedMemoryCarveout, 100);
    if (e != cudaSuccess) return e;
  }
  return cudaSuccess;
}

}  // namespace mgb
