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
// warp stages its share by TMA into a 3-stage shared-memory ring (mbarriers):
//   the x0 brick (1D bulk, 4 KiB); 2-cell-deep x0 slabs of the W/E/S/N
//   neighbours (3D tensor boxes {2,8,8} / {8,2,8}); the b values on those faces
//   ({2,8,8} / {8,1,8}); the x0 columns of the 4 diagonal neighbours ({2,1,8}).
// Warp w owns planes 2w, 2w+1 and walks them in k with planes k-1..k+1 in
// registers.  Per plane:
//   * every lane computes x1 of ONE neighbour face cell (lanes 0-7 the W face,
//     8-15 E, 16-23 S, 24-31 N) -- the redundant ring of x1 the second sweep
//     needs; in-face neighbours by shuffles, diagonal corner columns at the ends;
//   * x1 of the warp's own cells (lane = cell pair (2(l&3), l>>2)); face x0 and
//     face x1 reach the boundary lanes by warp shuffles;
//   * x1 goes to a 2-deep shared ring; x2 of the PREVIOUS item (phase B) uses it,
//     the face x1 kept in registers, plane 7 of item m-2 (carry) and plane 0 of
//     item m, and streams to HBM with r or the restricted coarse b on the last
//     sweep of a phase.
// b of the own cells travels in registers (128-bit loads one item ahead).
#include <cudaTypedefs.h>

#include <cstddef>
#include <type_traits>

#include "kernels.h"
#include "mg_internal.h"
#include "ptx.cuh"

namespace mgb {

constexpr int P2_NX = 4;      // own-brick x0 ring: items m, m+1 read; m+2, m+3 in flight
constexpr int P2_NS = 3;      // neighbour-slab ring: items m, m+1 read; m+2 in flight (issued one step
                              // later than the own brick, so the neighbour CTAs -- walking the
                              // neighbour columns in lockstep -- have already pulled those bricks to L2)
constexpr int P2_RING = 8;    // metadata ring
constexpr int P2_META = 11;   // id, flags, W,E,S,N, SW,NW,SE,NE, parent
constexpr int P2_WARPS = 4;
constexpr int P2_THREADS = 32 * P2_WARPS;

struct P2Slab {
  double xwe[2][8][8][2];     // x0 of the W brick (i = 6,7) / E brick (i = 0,1): [k][j][ii]
  double xsn[2][8][2][8];     // x0 of the S brick (j = 6,7) / N brick (j = 0,1): [k][jj][i]
  double bwe[2][8][8][2];     // b  of the W brick (i = 6,7) / E brick (i = 0,1)
  double bsn[2][8][8];        // b  of the S brick (j = 7) / N brick (j = 0): [k][i]
  double cor[4][8][2];        // x0 columns: SW (i=6,7 j=7), NW (i=6,7 j=0), SE (i=0,1 j=7), NE (i=0,1 j=0)
};
static_assert(sizeof(P2Slab) % 128 == 0, "slab stage must keep TMA destinations 128-byte aligned");
// warps 1-3's expect_tx byte counts below add up to the whole slab stage
static_assert(sizeof(P2Slab) == 3 * 1024 + 3 * 1024 + (512 + 512 + 512), "slab bytes");
constexpr int OXWE = 0, OXSN = 256, OBWE = 512, OBSN = 768, OCOR = 896;  // offsets in doubles
static_assert(offsetof(P2Slab, xwe) == OXWE * 8 && offsetof(P2Slab, xsn) == OXSN * 8 &&
                  offsetof(P2Slab, bwe) == OBWE * 8 && offsetof(P2Slab, bsn) == OBSN * 8 &&
                  offsetof(P2Slab, cor) == OCOR * 8,
              "slab layout");

struct P2Smem {
  double ownx[P2_NX][512];  // x0 of the item bricks, cell i + 8j + 64k
  P2Slab sl[P2_NS];
  double A[2][512];        // x1 of items m-1, m
  double cx0[2][64];       // x0 plane 7 of the previous item (own cells)
  double cface[2][32];     // x0 plane 7 of the previous item's face cells (one per face lane)
  double cx1[2][64];       // x1 plane 7 of item m-2
  uint64_t bx[P2_NX];      // own-brick ring barriers (1 arrive: warp 0)
  uint64_t bs[P2_NS];      // slab ring barriers (3 arrives: warps 1-3)
  int meta[P2_RING][12];
};

__device__ __forceinline__ double2 lds2(const double* p) { return *reinterpret_cast<const double2*>(p); }

template <unsigned FLAGS>
__global__ void __launch_bounds__(P2_THREADS, kPairCtasPerSm)
    sweep2_kernel(SweepArgs p, PairArgs pa, const __grid_constant__ PairMaps mp) {
  pdl_wait();
  constexpr bool WRITE_R = (FLAGS & SW_WRITE_R) != 0;
  constexpr bool RESTRICT = (FLAGS & SW_RESTRICT) != 0;
  constexpr bool COLOUR = (FLAGS & SW_COLOUR) != 0;  // red-black half-sweeps (GSRB variant)
  constexpr unsigned FULL = 0xffffffffu;
  extern __shared__ __align__(128) unsigned char smem_raw[];
  P2Smem& S = *reinterpret_cast<P2Smem*>(smem_raw);
  const int col1 = COLOUR ? p.colour : -1, col2 = COLOUR ? p.colour2 : -1;
  const int t = threadIdx.x, w = t >> 5, l = t & 31;
  const int2 cr = pa.ctas[blockIdx.x];
  const int64_t base = cr.x;
  const int cnt = cr.y;
  const double alpha = p.c.alpha, beta = p.c.beta, gamma = p.c.gamma, gamma2 = p.gamma2;
  const uint64_t pol_keep = l2_evict_last(), pol_stream = l2_evict_first();

  // ---- own-cell role: planes k0 = 2w, k0+1; cell pair (i0, i0+1) of row j ----
  const int i0 = 2 * (l & 3), j = l >> 2;
  const int q = 8 * j + i0;
  const int k0 = 2 * w;
  const bool isW = i0 == 0, isE = i0 == 6, isS = j == 0, isN = j == 7;
  const int sWE = isW ? j : 8 + j;                     // face lane holding my W / E face cell
  const int sSN = (isS ? 16 : 24) + i0;                // face lanes holding my S / N face pair
  // my W / E face x0 (row j) and S / N face x0 pair (i0, i0+1) in the slab stage at plane 0 (lanes
  // inside the brick read the same words as a boundary lane: broadcasts, no extra wavefronts)
  const int fwo = isE ? OXWE + 128 + 2 * j : OXWE + 2 * j + 1;
  const int fsno = isN ? OXSN + 128 + i0 : OXSN + 8 + i0;
  // ---- face-cell role: face ff (0 W, 1 E, 2 S, 3 N), in-face coordinate c8 ----
  const int ff = l >> 3, c8 = l & 7;
  // in-brick (i, j) of this lane's face cell in its neighbour brick (the red-black colour)
  const int fci = ff == 0 ? 7 : ff == 1 ? 0 : c8, fcj = ff == 0 || ff == 1 ? c8 : ff == 2 ? 7 : 0;
  int oc0, oo0, ob0, obk, olo, ohi;  // stage offsets (doubles) at plane 0; slabs step 16 / plane
  if (ff == 0) {         // W brick, cell (7, c8, k): o = (6, c8), own = (0, c8) of my brick
    oc0 = OXWE + 2 * c8 + 1, oo0 = OXWE + 2 * c8, ob0 = OBWE + 2 * c8 + 1, obk = 16;
    olo = OCOR + 0 * 16 + 1, ohi = OCOR + 1 * 16 + 1;  // j-1 -> SW (i=7), j+1 -> NW (i=7)
  } else if (ff == 1) {  // E brick, cell (0, c8, k): o = (1, c8), own = (7, c8)
    oc0 = OXWE + 128 + 2 * c8, oo0 = OXWE + 128 + 2 * c8 + 1, ob0 = OBWE + 128 + 2 * c8, obk = 16;
    olo = OCOR + 2 * 16 + 0, ohi = OCOR + 3 * 16 + 0;  // SE (i=0), NE (i=0)
  } else if (ff == 2) {  // S brick, cell (c8, 7, k): o = (c8, 6), own = (c8, 0)
    oc0 = OXSN + 8 + c8, oo0 = OXSN + c8, ob0 = OBSN + c8, obk = 8;
    olo = OCOR + 0 * 16 + 1, ohi = OCOR + 2 * 16 + 0;  // i-1 -> SW (i=7), i+1 -> SE (i=0)
  } else {               // N brick, cell (c8, 0, k): o = (c8, 1), own = (c8, 7)
    oc0 = OXSN + 128 + c8, oo0 = OXSN + 128 + 8 + c8, ob0 = OBSN + 64 + c8, obk = 8;
    olo = OCOR + 1 * 16 + 1, ohi = OCOR + 3 * 16 + 0;  // NW (i=7), NE (i=0)
  }
  const int ocr = c8 == 7 ? ohi : olo;  // the one diagonal-corner value this face lane needs
  // the own-brick cell next to the face cell lives in lane srcOwn's register pair
  const int srcOwn = ff == 0 ? 4 * c8 : ff == 1 ? 4 * c8 + 3 : ff == 2 ? (c8 >> 1) : 28 + (c8 >> 1);
  const bool ownY = ff == 1 || (ff >= 2 && (c8 & 1));

  for (int e = t; e < P2_RING * P2_META; e += P2_THREADS) {
    const int it = e / P2_META, fl = e % P2_META;
    if (it < cnt) S.meta[it][fl] = pa.meta[(base + it) * P2_META + fl];
  }
  if (t == 0) {
    for (int s = 0; s < P2_NX; ++s) mbar_init(&S.bx[s], 1);
    for (int s = 0; s < P2_NS; ++s) mbar_init(&S.bs[s], P2_WARPS - 1);
    mbar_fence_init();
  }
  __syncthreads();

  // lane 0 of warp 0 stages item m's own brick; lanes 0 of warps 1-3 its neighbour slabs
  auto issue_x = [&](int m) {
    const int s = m % P2_NX;
    mbar_expect_tx(&S.bx[s], 4096);
    // evict_last: the neighbour CTAs read this brick's faces shortly after
    tma_load_1d_hint(S.ownx[s], p.x + (int64_t)S.meta[m % P2_RING][0] * 512, 4096, &S.bx[s], pol_keep);
  };
  auto issue_slab = [&](int m) {
    const int s = m % P2_NS;
    const int* M = S.meta[m % P2_RING];
    P2Slab& G = S.sl[s];
    uint64_t* bar = &S.bs[s];
    if (w == 1) {
      mbar_expect_tx(bar, 3 * 1024);
      tma_load_3d(G.xwe[0], &mp.xwe, 6, 0, M[2] * 8, bar);  // W: i = 6,7
      tma_load_3d(G.xwe[1], &mp.xwe, 0, 0, M[3] * 8, bar);  // E: i = 0,1
      tma_load_3d(G.xsn[0], &mp.xsn, 0, 6, M[4] * 8, bar);  // S: j = 6,7
    } else if (w == 2) {
      mbar_expect_tx(bar, 3 * 1024);
      tma_load_3d(G.xsn[1], &mp.xsn, 0, 0, M[5] * 8, bar);  // N: j = 0,1
      tma_load_3d(G.bwe[0], &mp.bwe, 6, 0, M[2] * 8, bar);
      tma_load_3d(G.bwe[1], &mp.bwe, 0, 0, M[3] * 8, bar);
    } else {
      mbar_expect_tx(bar, 512 + 512 + 512);
      tma_load_3d(G.bsn[0], &mp.bsn, 0, 7, M[4] * 8, bar);
      tma_load_3d(G.bsn[1], &mp.bsn, 0, 0, M[5] * 8, bar);
      tma_load_3d(G.cor[0], &mp.xcor, 6, 7, M[6] * 8, bar);  // SW: (i = 7, j = 7)
      tma_load_3d(G.cor[1], &mp.xcor, 6, 0, M[7] * 8, bar);  // NW: (i = 7, j = 0)
      tma_load_3d(G.cor[2], &mp.xcor, 0, 7, M[8] * 8, bar);  // SE: (i = 0, j = 7)
      tma_load_3d(G.cor[3], &mp.xcor, 0, 0, M[9] * 8, bar);  // NE: (i = 0, j = 0)
    }
  };
  auto load_b = [&](int m, double2& v0, double2& v1) {
    const double* bp = p.b + (int64_t)S.meta[m % P2_RING][0] * 512 + 64 * k0 + q;
    v0 = ld_hint2(bp, pol_keep);  // the neighbours' b-face slabs reuse these lines from L2
    v1 = ld_hint2(bp + 64, pol_keep);
  };

  if (l == 0) {
    if (w == 0)
      for (int m = 0; m < P2_NX - 1 && m < cnt; ++m) issue_x(m);
    else
      for (int m = 0; m < P2_NS - 1 && m < cnt; ++m) issue_slab(m);
  }
  // registers indexed by item parity (the walk is unrolled by two, so every index is constant):
  //   bq[par]  b of the own cells (planes k0, k0+1) of the item with that parity
  //   fweq/fsnq[par]  face x1 delivered to this lane (W/E value, S/N pair) per plane
  double2 bq[2][2];
  double fweq[2][2];
  double2 fsnq[2][2];
  load_b(0, bq[0][0], bq[0][1]);
  bq[1][0] = bq[1][1] = make_double2(0.0, 0.0);
  int mreg = 0;

  auto step = [&](const int m, auto par) {
    constexpr int cur = decltype(par)::value, prv = cur ^ 1;
    // metadata ring holds items m-3 .. m+3 during step m: store item m+4 (loaded last step)
    // into the slot of item m-4, then load item m+5 (fields spread over the warps)
    if (l < 3 && w + 4 * l < P2_META) {
      const int fl = w + 4 * l;
      if (m >= 1 && m + 4 < cnt) S.meta[(m + 4) % P2_RING][fl] = mreg;
      if (m + 5 < cnt) mreg = pa.meta[(base + m + 5) * P2_META + fl];
    }
    // the ring slots of items m+NX-1 / m+NS-1 are item m-1's, unread since the barrier ending step m-1
    if (l == 0) {
      fence_proxy_async();
      if (w == 0) {
        if (m + P2_NX - 1 < cnt) issue_x(m + P2_NX - 1);
      } else if (m + P2_NS - 1 < cnt) {
        issue_slab(m + P2_NS - 1);
      }
    }
    double2 bna = bq[cur][0], bnb = bq[cur][1];  // b of item m+1
    if (m + 1 < cnt) load_b(m + 1, bna, bnb);

    // ---------------- phase A: x1 of item m ----------------
    {
      mbar_wait(&S.bx[m % P2_NX], (uint32_t)((m / P2_NX) & 1));
      mbar_wait(&S.bs[m % P2_NS], (uint32_t)((m / P2_NS) & 1));
      if (m + 1 < cnt) {
        mbar_wait(&S.bx[(m + 1) % P2_NX], (uint32_t)(((m + 1) / P2_NX) & 1));
        mbar_wait(&S.bs[(m + 1) % P2_NS], (uint32_t)(((m + 1) / P2_NS) & 1));
      }
      // a warm-up item contributes only its x1 plane 7 (warp 3), a cool-down item only plane 0 (warp 0)
      const int fl = S.meta[m % P2_RING][1];
      const bool idle = ((fl & 2) && w < P2_WARPS - 1) || ((fl & 4) && w > 0);
      const double* X = S.ownx[m % P2_NX];
      const double* NX = S.ownx[(m + 1) % P2_NX];  // stale if no next item (feeds only unused cells)
      const double* G = reinterpret_cast<const double*>(&S.sl[m % P2_NS]);
      const double* N = reinterpret_cast<const double*>(&S.sl[(m + 1) % P2_NS]);
      if (!idle) {
        const double2 xm = w > 0 ? lds2(X + 64 * (k0 - 1) + q) : lds2(S.cx0[prv] + q);
        const double2 x0 = lds2(X + 64 * k0 + q);
        const double2 x1 = lds2(X + 64 * (k0 + 1) + q);
        const double2 x2 = w < P2_WARPS - 1 ? lds2(X + 64 * (k0 + 2) + q) : lds2(NX + q);
        // face lane: its face cell's x0 on planes k0-1 .. k0+2
        const double cm = w > 0 ? G[oc0 + 16 * (k0 - 1)] : S.cface[prv][l];
        const double cf0 = G[oc0 + 16 * k0], cf1 = G[oc0 + 16 * (k0 + 1)];
        const double cp = w < P2_WARPS - 1 ? G[oc0 + 16 * (k0 + 2)] : N[oc0];
        double* Aw = S.A[cur];
#pragma unroll
        for (int kk = 0; kk < 2; ++kk) {
          const int k = k0 + kk;
          const double2 xc = kk ? x1 : x0, xb = kk ? x0 : xm, xt = kk ? x2 : x1;
          // -- x1 of this lane's face cell.  Its W/E (or S/N) neighbour pair is {o, own} and the
          //    other in-plane pair {lo, hi}; IEEE addition is commutative, so
          //    ((o+own)+(lo+hi))+(b+t) is bit-identical to the canonical ((w+e)+(s+n))+(b+t).
          const double c = kk ? cf1 : cf0, bt = kk ? cf0 : cm, tp = kk ? cp : cf1;
          const double o = G[oo0 + 16 * k];
          const double bf = G[ob0 + obk * k];
          const double ownx = __shfl_sync(FULL, xc.x, srcOwn), owny = __shfl_sync(FULL, xc.y, srcOwn);
          const double own = ownY ? owny : ownx;
          const double up = __shfl_up_sync(FULL, c, 1), dn = __shfl_down_sync(FULL, c, 1);
          const double corner = G[ocr + 2 * k];
          const double lo = c8 > 0 ? up : corner;
          const double hi = c8 < 7 ? dn : corner;
          const double sum = DADD(DADD(DADD(o, own), DADD(lo, hi)), DADD(bt, tp));
          const double af = DADD(DMUL(alpha, c), DMUL(beta, sum));
          const double fx1 = keep_cell(col1, fci, fcj, k) ? c : DADD(c, DMUL(gamma, DSUB(af, bf)));
          // -- face x0 next to my cells from the slab; face x1 delivered by the face lanes
          const double vwe = G[fwo + 16 * k];
          const double2 vsn = lds2(G + fsno + 16 * k);
          fweq[cur][kk] = __shfl_sync(FULL, fx1, sWE);
          fsnq[cur][kk].x = __shfl_sync(FULL, fx1, sSN);
          fsnq[cur][kk].y = __shfl_sync(FULL, fx1, sSN + 1);
          // -- x1 of the own cells
          const double2 bb = bq[cur][kk];
          double2 rs_, rn_;  // rows j-1, j+1 of the plane live in lanes l-4, l+4
          rs_.x = __shfl_up_sync(FULL, xc.x, 4), rs_.y = __shfl_up_sync(FULL, xc.y, 4);
          rn_.x = __shfl_down_sync(FULL, xc.x, 4), rn_.y = __shfl_down_sync(FULL, xc.y, 4);
          const double wl = __shfl_up_sync(FULL, xc.y, 1), er = __shfl_down_sync(FULL, xc.x, 1);
          const double wo = isW ? vwe : wl, eo = isE ? vwe : er;
          const double2 so = isS ? vsn : rs_, no = isN ? vsn : rn_;
          const double a0 = stencil_a(xc.x, wo, xc.y, so.x, no.x, xb.x, xt.x, alpha, beta);
          const double a1 = stencil_a(xc.y, xc.x, eo, so.y, no.y, xb.y, xt.y, alpha, beta);
          double2 y;
          y.x = keep_cell(col1, i0, j, k) ? xc.x : DADD(xc.x, DMUL(gamma, DSUB(a0, bb.x)));
          y.y = keep_cell(col1, i0 + 1, j, k) ? xc.y : DADD(xc.y, DMUL(gamma, DSUB(a1, bb.y)));
          *reinterpret_cast<double2*>(Aw + 64 * k + q) = y;
        }
        if (w == P2_WARPS - 1) {  // plane 7 carries for the next item's plane 0
          *reinterpret_cast<double2*>(S.cx0[cur] + q) = x1;
          S.cface[cur][l] = cf1;
        }
      }
    }
    __syncthreads();  // x1 of item m (plane 0 for phase B) and the carries are visible

    // ---------------- phase B: x2 of item m-1 ----------------
    if (m >= 1) {
      const double* P = S.A[prv];
      const double2 y0 = lds2(P + 64 * k0 + q), y1 = lds2(P + 64 * (k0 + 1) + q);
      if (w == P2_WARPS - 1) *reinterpret_cast<double2*>(S.cx1[prv] + q) = y1;  // x1 plane 7 of item m-1
      const bool emit = (S.meta[m % P2_RING][1] & 1) != 0;  // item m-1 is a range brick
      if (emit) {
        const double2 ym = w > 0 ? lds2(P + 64 * (k0 - 1) + q) : lds2(S.cx1[cur] + q);  // item m-2 plane 7
        const double2 yp = w < P2_WARPS - 1 ? lds2(P + 64 * (k0 + 2) + q) : lds2(S.A[cur] + q);  // item m
        const int64_t g = (int64_t)S.meta[(m - 1) % P2_RING][0] * 512 + q;
        double rsum[2];
#pragma unroll
        for (int kk = 0; kk < 2; ++kk) {
          const int k = k0 + kk;
          const double2 xc = kk ? y1 : y0, xb = kk ? y0 : ym, xt = kk ? yp : y1;
          const double2 bb = bq[prv][kk];
          double2 rs_, rn_;
          rs_.x = __shfl_up_sync(FULL, xc.x, 4), rs_.y = __shfl_up_sync(FULL, xc.y, 4);
          rn_.x = __shfl_down_sync(FULL, xc.x, 4), rn_.y = __shfl_down_sync(FULL, xc.y, 4);
          const double wl = __shfl_up_sync(FULL, xc.y, 1), er = __shfl_down_sync(FULL, xc.x, 1);
          const double wv = isW ? fweq[prv][kk] : wl, ev = isE ? fweq[prv][kk] : er;
          const double2 sv = isS ? fsnq[prv][kk] : rs_, nv = isN ? fsnq[prv][kk] : rn_;
          const double a0 = stencil_a(xc.x, wv, xc.y, sv.x, nv.x, xb.x, xt.x, alpha, beta);
          const double a1 = stencil_a(xc.y, xc.x, ev, sv.y, nv.y, xb.y, xt.y, alpha, beta);
          double2 y, rv;
          y.x = keep_cell(col2, i0, j, k) ? xc.x : DADD(xc.x, DMUL(gamma2, DSUB(a0, bb.x)));
          y.y = keep_cell(col2, i0 + 1, j, k) ? xc.y : DADD(xc.y, DMUL(gamma2, DSUB(a1, bb.y)));
          rv.x = DSUB(bb.x, a0);
          rv.y = DSUB(bb.y, a1);
          st_hint2(p.xo + g + 64 * k, y, pol_stream);  // never re-read by this pass
          if (WRITE_R) st_hint2(p.r + g + 64 * k, rv, pol_stream);
          rsum[kk] = DADD(rv.x, rv.y);  // r(2I,.,.) + r(2I+1,.,.) of this row and plane
        }
        if (RESTRICT) {
          // coarse cell (I, J, K) = (l&3, j/2, w): its 8 fine cells are this lane's and lane+4's
          // pairs on planes 2w, 2w+1 -> canonical order ((r000+r100)+(r010+r110))+((r001+r101)+(r011+r111))
          const double s0n = __shfl_down_sync(FULL, rsum[0], 4);
          const double s1n = __shfl_down_sync(FULL, rsum[1], 4);
          if ((j & 1) == 0) {
            const double v = DMUL(0.125, DADD(DADD(rsum[0], s0n), DADD(rsum[1], s1n)));
            const int pr = S.meta[(m - 1) % P2_RING][10];
            const int oct = pr & 7;
            const int ox = oct & 1, oy = (oct >> 1) & 1, oz = oct >> 2;
            p.bc[(int64_t)(pr >> 3) * 512 + (4 * ox + (l & 3)) + 8 * (4 * oy + (j >> 1)) + 64 * (4 * oz + w)] = v;
          }
        }
      }
    }
    __syncthreads();  // x1 ring slot of item m-1 and the carries may be overwritten next step
    bq[prv][0] = bna;  // item m+1 has parity prv; item m-1's b is consumed
    bq[prv][1] = bnb;
  };

  // the last item is always a cool-down brick: its x2 is not wanted, so step cnt-1 ends the walk
  for (int m = 0; m < cnt; m += 2) {
    step(m, std::integral_constant<int, 0>{});
    if (m + 1 < cnt) step(m + 1, std::integral_constant<int, 1>{});
  }
  pdl_trigger();
}

bool pair_supports(unsigned flags) {
  const unsigned fl = flags & (SW_WRITE_R | SW_RESTRICT | SW_INTERP | SW_ZERO_X);
  return fl == 0 || fl == SW_WRITE_R || fl == SW_RESTRICT;
}

cudaError_t launch_sweep2(const SweepArgs& a, const PairArgs& pa, const PairMaps& pm, unsigned flags,
                          cudaStream_t s) {
  if (pa.nctas <= 0) return cudaSuccess;
  const unsigned g = (unsigned)pa.nctas;
  const size_t sm = sizeof(P2Smem);
  const unsigned col = (a.colour >= 0 || a.colour2 >= 0) ? SW_COLOUR : 0u;
  switch ((flags & (SW_WRITE_R | SW_RESTRICT | SW_INTERP | SW_ZERO_X)) | col) {
    case 0: launch_plain(sweep2_kernel<0>, g, P2_THREADS, sm, s, a, pa, pm); break;
    case SW_WRITE_R: launch_plain(sweep2_kernel<SW_WRITE_R>, g, P2_THREADS, sm, s, a, pa, pm); break;
    case SW_RESTRICT: launch_plain(sweep2_kernel<SW_RESTRICT>, g, P2_THREADS, sm, s, a, pa, pm); break;
    case SW_COLOUR: launch_plain(sweep2_kernel<SW_COLOUR>, g, P2_THREADS, sm, s, a, pa, pm); break;
    case SW_WRITE_R | SW_COLOUR: launch_plain(sweep2_kernel<SW_WRITE_R | SW_COLOUR>, g, P2_THREADS, sm, s, a, pa, pm); break;
    case SW_RESTRICT | SW_COLOUR: launch_plain(sweep2_kernel<SW_RESTRICT | SW_COLOUR>, g, P2_THREADS, sm, s, a, pa, pm); break;
    default: return cudaErrorInvalidValue;
  }
  return cudaGetLastError();
}

cudaError_t pair_kernels_init() {
  const void* k[6] = {(const void*)sweep2_kernel<0>, (const void*)sweep2_kernel<SW_WRITE_R>,
                      (const void*)sweep2_kernel<SW_RESTRICT>, (const void*)sweep2_kernel<SW_COLOUR>,
                      (const void*)sweep2_kernel<SW_WRITE_R | SW_COLOUR>,
                      (const void*)sweep2_kernel<SW_RESTRICT | SW_COLOUR>};
  for (int i = 0; i < 6; ++i) {
    cudaError_t e = cudaFuncSetAttribute(k[i], cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(P2Smem));
    if (e != cudaSuccess) return e;
    e = cudaFuncSetAttribute(k[i], cudaFuncAttributePreferredSharedMemoryCarveout, 100);
    if (e != cudaSuccess) return e;
  }
  return cudaSuccess;
}

}  // namespace mgb
