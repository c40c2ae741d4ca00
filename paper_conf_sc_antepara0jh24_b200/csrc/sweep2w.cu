// sweep2w.cu -- two Jacobi sweeps per HBM pass, one warp per two plane streams
// (temporal blocking; second design).
//
// Same arithmetic as sweep2.cu (x0 -> x1 -> x2 in one pass, every sweep the
// canonical smooth(+residual) of reading A8, bit-identical to two separate
// sweeps), different data flow: the k-direction lives in registers.
//
// Each half-warp walks its own stream of z-planes (layout.cpp warp_table:
// [warm-up planes 5..7, run bricks 0..7, cool-down plane 0] per run).  A lane
// owns a 2x2 footprint of the plane -- cells (2ip+a, 2jp+c), lane = ip + 4jp --
// and keeps three planes of x0 and of x1 around the current one.  Per step
// (plane k of brick m):
//   * x0 of plane k+1 and b of plane k come from 3-slot register rings of
//     128-bit loads issued one step ahead (the lines were prefetched into L2 four
//     planes ahead);
//   * the four side neighbours' 2-deep x0 face slabs, their b faces and the four
//     diagonal corner columns arrive per brick by TMA into a 2-stage ring (item
//     m+1's slabs are issued at plane 4 of item m);
//   * lane (face ff, pair pr) computes x1 of the neighbour face cells 2pr, 2pr+1
//     of plane k (the redundant ring the second sweep needs); the adjacent own
//     cells reach it by a 3-round shuffle from the owner lanes;
//   * every lane computes x1 of its 4 cells of plane k, then x2 of the previous
//     plane (one-plane lag) from the x1 window, and streams x2 (with r, or the
//     restricted coarse b, which the 2x2 footprint sums in registers) to HBM.
// In-plane neighbours come by width-16 shuffles (2 per cell per sweep instead of
// 3 with a 2x1 footprint), face values by LDS from the slabs; x0, x1 and b make
// no shared-memory round trip and there are no CTA barriers.
#include <cudaTypedefs.h>

#include <cstddef>
#include <type_traits>

#include "kernels.h"
#include "mg_internal.h"
#include "ptx.cuh"

namespace mgb {

namespace {

struct W2Slab {
  double xwe[2][8][8][2];  // x0 of the W brick (i = 6,7) / E brick (i = 0,1): [k][j][ii]
  double xsn[2][8][2][8];  // x0 of the S brick (j = 6,7) / N brick (j = 0,1): [k][jj][i]
  double bwe[2][8][8][2];  // b of the W / E brick, same boxes
  double bsn[2][8][8];     // b of the S brick (j = 7) / N brick (j = 0): [k][i]
  double cor[4][8][2];     // x0 columns SW (i=6,7 j=7), NW (i=6,7 j=0), SE (i=0,1 j=7), NE (i=0,1 j=0)
};
static_assert(sizeof(W2Slab) == 7680 && sizeof(W2Slab) % 128 == 0, "slab stage keeps TMA destinations aligned");
constexpr int WXWE = 0, WXSN = 256, WBWE = 512, WBSN = 768, WCOR = 896;  // offsets in doubles
static_assert(offsetof(W2Slab, xsn) == WXSN * 8 && offsetof(W2Slab, bwe) == WBWE * 8 &&
                  offsetof(W2Slab, bsn) == WBSN * 8 && offsetof(W2Slab, cor) == WCOR * 8,
              "slab layout");
constexpr int kSlabD = (int)(sizeof(W2Slab) / sizeof(double));
constexpr int kMR = 8;  // meta ring slots per half: items m .. m+7

struct alignas(128) W2Smem {  // one per warp; 128-byte multiple keeps every warp's TMA stages aligned
  W2Slab sl[2][2];          // [half][stage]
  int meta[2][kMR][kW2Meta];
  uint64_t bar[2][2];       // [half][stage]
};
static_assert(sizeof(W2Smem) % 128 == 0 && sizeof(W2Smem) * kW2WarpsPerSm <= 227 * 1024, "per-SM shared memory");

__device__ __forceinline__ double2 lds2w(const double* p) { return *reinterpret_cast<const double2*>(p); }

// one of the lane's four x values: code bit0 = i offset, bit1 = j offset
__device__ __forceinline__ double sel4(int code, double2 r0, double2 r1) {
  const double2 r = (code & 2) ? r1 : r0;
  return (code & 1) ? r.y : r.x;
}

// a = A x for the lane's 2x2 footprint of one plane (c: rows 2jp, 2jp+1; m / p: planes k-1 / k+1);
// in-plane neighbours from the lanes around (width-16 shuffles) or, at the brick's side faces,
// from (we0, we1) (W or E face, rows 2jp, 2jp+1) and sn (S or N face, columns 2ip, 2ip+1)
__device__ __forceinline__ void own_a(double2 c0, double2 c1, double2 m0, double2 m1, double2 p0, double2 p1,
                                      double we0, double we1, double2 sn, bool isW, bool isE, bool isS, bool isN,
                                      double alpha, double beta, double a[4]) {
  constexpr unsigned FULL = 0xffffffffu;
  const double wl0 = __shfl_up_sync(FULL, c0.y, 1, 16), wl1 = __shfl_up_sync(FULL, c1.y, 1, 16);
  const double er0 = __shfl_down_sync(FULL, c0.x, 1, 16), er1 = __shfl_down_sync(FULL, c1.x, 1, 16);
  const double sb0 = __shfl_up_sync(FULL, c1.x, 4, 16), sb1 = __shfl_up_sync(FULL, c1.y, 4, 16);
  const double nt0 = __shfl_down_sync(FULL, c0.x, 4, 16), nt1 = __shfl_down_sync(FULL, c0.y, 4, 16);
  const double W0 = isW ? we0 : wl0, W1 = isW ? we1 : wl1;
  const double E0 = isE ? we0 : er0, E1 = isE ? we1 : er1;
  const double S0 = isS ? sn.x : sb0, S1 = isS ? sn.y : sb1;
  const double N0 = isN ? sn.x : nt0, N1 = isN ? sn.y : nt1;
  a[0] = stencil_a(c0.x, W0, c0.y, S0, c1.x, m0.x, p0.x, alpha, beta);
  a[1] = stencil_a(c0.y, c0.x, E0, S1, c1.y, m0.y, p0.y, alpha, beta);
  a[2] = stencil_a(c1.x, W1, c1.y, c0.x, N0, m1.x, p1.x, alpha, beta);
  a[3] = stencil_a(c1.y, c1.x, E1, c0.y, N1, m1.y, p1.y, alpha, beta);
}

// x1 of one neighbour face cell: its in-plane pairs are {o, own} (across the face) and {lo, hi}
// (along it); IEEE addition is commutative, so ((o+own)+(lo+hi))+(bt+tp) is bit-identical to the
// canonical ((w+e)+(s+n))+(b+t) for every face orientation
__device__ __forceinline__ double face_x1(double c, double o, double own, double lo, double hi, double bt, double tp,
                                          double bf, double alpha, double beta, double gamma) {
  const double sum = DADD(DADD(DADD(o, own), DADD(lo, hi)), DADD(bt, tp));
  const double a = DADD(DMUL(alpha, c), DMUL(beta, sum));
  return DADD(c, DMUL(gamma, DSUB(a, bf)));
}

}  // namespace

template <unsigned FLAGS>
__global__ void __launch_bounds__(32 * kW2WarpsPerSm, 1)
    sweep2w_kernel(SweepArgs p, PairArgs pa, const __grid_constant__ PairMaps mp) {
  pdl_wait();
  constexpr bool WRITE_R = (FLAGS & SW_WRITE_R) != 0;
  constexpr bool RESTRICT = (FLAGS & SW_RESTRICT) != 0;
  constexpr unsigned FULL = 0xffffffffu;
  extern __shared__ __align__(128) unsigned char smem_raw[];
  // the CTA is kW2WarpsPerSm independent warps (one CTA per SM spreads them over the four
  // sub-partitions); each warp has its own shared-memory region and never waits on the others
  const int wid = threadIdx.x >> 5;
  const int64_t gw = (int64_t)blockIdx.x * kW2WarpsPerSm + wid;
  if (gw >= pa.nwarps) return;
  W2Smem& S = reinterpret_cast<W2Smem*>(smem_raw)[wid];
  const int lane = threadIdx.x & 31, h = lane >> 4, hl = lane & 15;
  const int4 wd = pa.warps[gw];
  const int64_t it0 = h ? wd.y : wd.x;
  const int nsteps = wd.z;
  const int nitems = h ? (int)((unsigned)wd.w >> 16) : (wd.w & 0xffff);
  const int32_t* MG = pa.meta + it0 * kW2Meta;  // this half's items
  int(*MT)[kW2Meta] = S.meta[h];
  double* SLb = &S.sl[h][0].xwe[0][0][0][0];
  uint64_t* BAR = S.bar[h];
  const double alpha = p.c.alpha, beta = p.c.beta, gamma = p.c.gamma, gamma2 = p.gamma2;
  const uint64_t pol_keep = l2_evict_last(), pol_stream = l2_evict_first();

  // ---- own footprint: cells (2ip + a, 2jp + c); rows at q0 and q0 + 8 of a plane
  const int ip = hl & 3, jp = hl >> 2;
  const int q0 = 2 * ip + 16 * jp;
  const bool isW = ip == 0, isE = ip == 3, isS = jp == 0, isN = jp == 3;
  // face x0 of plane k for the lanes next to a face (lanes inside read the same words: broadcast)
  const int fo0 = isE ? WXWE + 128 + 4 * jp : WXWE + 4 * jp + 1, fo1 = fo0 + 2;  // W / E, rows 2jp, 2jp+1
  const int fsno = isN ? WXSN + 128 + 2 * ip : WXSN + 8 + 2 * ip;                 // S / N, columns 2ip, 2ip+1
  // lanes holding my W/E and S/N face x1 (face lane = 4 ff + pr)
  const int src_we = isE ? 4 + jp : jp, src_sn = isN ? 12 + ip : 8 + ip;
  // what I send in the three rounds that bring the face lanes their adjacent own cells
  // (corner lanes serve two faces; the round-A value is the cell both want)
  int cA = 0, cB = 0, cC = 0;
  if (isW && isS) cA = 0, cB = 2, cC = 1;
  else if (isE && isS) cA = 1, cB = 3, cC = 0;
  else if (isW && isN) cA = 2, cB = 0, cC = 3;
  else if (isE && isN) cA = 3, cB = 1, cC = 2;
  else if (isW) cA = 0, cB = 2;
  else if (isE) cA = 1, cB = 3;
  else if (isS) cA = 0, cC = 1;
  else if (isN) cA = 2, cC = 3;
  // ---- face role: face ff (0 W, 1 E, 2 S, 3 N), cells c8 = 2pr, 2pr+1 of the neighbour's face layer
  const int ff = hl >> 2, pr = hl & 3;
  int u0o, u1o, bo0, bks, coff, fsrc;
  if (ff == 0) {         // W brick (i = 7): U_e = (o, c) of row 2pr+e; corners SW (lo), NW (hi)
    u0o = WXWE + 4 * pr, u1o = u0o + 2, bo0 = WBWE + 4 * pr + 1, bks = 16;
    coff = pr == 3 ? WCOR + 16 + 1 : WCOR + 1, fsrc = 4 * pr;
  } else if (ff == 1) {  // E brick (i = 0): U_e = (c, o); corners SE, NE
    u0o = WXWE + 128 + 4 * pr, u1o = u0o + 2, bo0 = WBWE + 128 + 4 * pr, bks = 16;
    coff = pr == 3 ? WCOR + 48 : WCOR + 32, fsrc = 4 * pr + 3;
  } else if (ff == 2) {  // S brick (j = 7): U0 = c pair, U1 = o pair; corners SW, SE
    u0o = WXSN + 8 + 2 * pr, u1o = WXSN + 2 * pr, bo0 = WBSN + 2 * pr, bks = 8;
    coff = pr == 3 ? WCOR + 32 : WCOR + 1, fsrc = pr;
  } else {               // N brick (j = 0); corners NW, NE
    u0o = WXSN + 128 + 2 * pr, u1o = WXSN + 128 + 8 + 2 * pr, bo0 = WBSN + 64 + 2 * pr, bks = 8;
    coff = pr == 3 ? WCOR + 48 : WCOR + 16 + 1, fsrc = 12 + pr;
  }
  const int bo1 = bo0 + (bks == 16 ? 2 : 1);
  const bool fWE = ff < 2, fswap = pr == 3;
  // in-brick (i, j) of the two face cells (red-black colour): W (7, c8), E (0, c8), S (c8, 7), N (c8, 0)
  const int fi0 = ff == 0 ? 7 : ff == 1 ? 0 : 2 * pr, fj0 = ff < 2 ? 2 * pr : ff == 2 ? 7 : 0;
  const int fi1 = ff < 2 ? fi0 : fi0 + 1, fj1 = ff < 2 ? fj0 + 1 : fj0;

  // ---- meta ring (items 0..6) + the pending item 7; barriers; the first two slab stages
  for (int e = hl; e < 7 * kW2Meta / 4; e += 16)
    reinterpret_cast<int4*>(&MT[0][0])[e] = reinterpret_cast<const int4*>(MG)[e];
  int4 pend = make_int4(0, 0, 0, 0);
  if (hl < kW2Meta / 4) pend = reinterpret_cast<const int4*>(MG + 7 * kW2Meta)[hl];
  if (hl == 0) {
    mbar_init(&BAR[0], 1);
    mbar_init(&BAR[1], 1);
    mbar_fence_init();
  }
  __syncwarp();

  auto issue = [&](int m) {  // item m's slabs -> stage m & 1 (lane 0 of the half)
    const int* M = MT[m & (kMR - 1)];
    double* G = SLb + (m & 1) * kSlabD;
    uint64_t* bar = &BAR[m & 1];
    mbar_expect_tx(bar, (uint32_t)sizeof(W2Slab));
    tma_load_3d(G + WXWE, &mp.xwe, 6, 0, M[2] * 8, bar);        // W: i = 6,7
    tma_load_3d(G + WXWE + 128, &mp.xwe, 0, 0, M[3] * 8, bar);  // E: i = 0,1
    tma_load_3d(G + WXSN, &mp.xsn, 0, 6, M[4] * 8, bar);        // S: j = 6,7
    tma_load_3d(G + WXSN + 128, &mp.xsn, 0, 0, M[5] * 8, bar);  // N: j = 0,1
    tma_load_3d(G + WBWE, &mp.bwe, 6, 0, M[2] * 8, bar);
    tma_load_3d(G + WBWE + 128, &mp.bwe, 0, 0, M[3] * 8, bar);
    tma_load_3d(G + WBSN, &mp.bsn, 0, 7, M[4] * 8, bar);
    tma_load_3d(G + WBSN + 64, &mp.bsn, 0, 0, M[5] * 8, bar);
    tma_load_3d(G + WCOR, &mp.xcor, 6, 7, M[6] * 8, bar);       // SW
    tma_load_3d(G + WCOR + 16, &mp.xcor, 6, 0, M[7] * 8, bar);  // NW
    tma_load_3d(G + WCOR + 32, &mp.xcor, 0, 7, M[8] * 8, bar);  // SE
    tma_load_3d(G + WCOR + 48, &mp.xcor, 0, 0, M[9] * 8, bar);  // NE
  };
  if (hl == 0 && nitems > 0) issue(0);

  auto fl_of = [&](int m) { return MT[m & (kMR - 1)][1]; };
  auto id_of = [&](int m) { return MT[m & (kMR - 1)][0]; };
  auto adv = [&](int& m, int& k) {  // next step of the stream
    if (k + 1 < (fl_of(m) >> 16)) {
      ++k;
    } else {
      ++m;
      k = (fl_of(m) >> 8) & 255;
    }
  };
  // x0 rows of the plane after (m, k) (k+1, or plane 0 of the next item = the z-successor)
  auto load_x = [&](int m, int k, double2* x) {
    const int idn = k < 7 ? id_of(m) : id_of(m + 1);
    const double* xs = p.x + (int64_t)idn * 512 + 64 * ((k + 1) & 7) + q0;
    x[0] = ld_hint2(xs, pol_keep);
    x[1] = ld_hint2(xs + 8, pol_keep);
  };
  auto load_b = [&](int m, int k, double2* b) {  // b rows of (m, k)
    const double* bs = p.b + (int64_t)id_of(m) * 512 + 64 * k + q0;
    b[0] = ld_hint2(bs, pol_keep);
    b[1] = ld_hint2(bs + 8, pol_keep);
  };

  // stream cursor: P(s) = (m, k), P(s+1) = (m1, k1)
  int m = 0, k = (fl_of(0) >> 8) & 255;
  int m1 = m, k1 = k;
  adv(m1, k1);
  // 3-slot register rings indexed by step % 3 (the body is unrolled by three, so every index is
  // a constant and no ring ever moves):
  //   X[j]  x0 rows of the plane after P(j)  -> at step s: xp = X[s], xc = X[s-1], xm = X[s-2]
  //   B[j]  b rows of P(j)                   -> bc = B[s], b of the lagged plane = B[s-1]
  //   Y[j]  x1 rows of P(j)                  -> x2 of P(s-1) from Y[s-2], Y[s-1], Y[s]
  //   C[j], O[j]  face x0 c / o of the plane after P(j) -> c window C[s-2..s], o = O[s-1]
  //   GW[j], GS[j]  face x1 of P(j) next to my cells (W/E pair, S/N pair)
  // (garbage until a run's two priming planes have streamed through)
  const double2 z2 = make_double2(0.0, 0.0);
  double2 X[3][2] = {{z2, z2}, {z2, z2}, {z2, z2}}, B[3][2] = {{z2, z2}, {z2, z2}, {z2, z2}};
  double2 Y[3][2] = {{z2, z2}, {z2, z2}, {z2, z2}};
  double C[3][2] = {}, O[3][2] = {}, GW[3][2] = {}, GS[3][2] = {};
  load_x(m, k, X[0]);
  load_b(m, k, B[0]);
  int out_id = 0, out_k = 0, out_par = 0;
  bool out_emit = false;
  double rpart = 0;

  auto step = [&](auto rc) {
    constexpr int r = decltype(rc)::value, rp = (r + 2) % 3, rq = (r + 1) % 3;  // s, s-1, s-2 (= s+1)
    const int fl = fl_of(m);
    const int kb = (fl >> 8) & 255, ke = fl >> 16;
    const int st = m & 1;
    if (hl == 0) {
      // item m+1's slabs go into the stage item m-1 has left, at plane 4 of item m (or its first /
      // last stepped plane): late enough that the neighbours' lines are still in L2 from their own
      // reads, early enough to land before the look-ahead at plane 7
      if (k == min(max(4, kb), ke - 1) && m + 1 < nitems) {
        fence_proxy_async();
        issue(m + 1);
      }
    }
    {
      // L2 prefetch of my rows of x and b four planes ahead (plane k+4 of this brick or of the
      // next item, the z-successor inside a run): the 128-bit loads issued one step ahead then hit
      // L2, and the lines stay resident only a few steps (a brick-sized prefetch an item ahead was
      // evicted before use)
      const int kf = k + 4;
      const int64_t off = (int64_t)(kf < 8 ? id_of(m) : id_of(m + 1)) * 512 + 64 * (kf & 7) + q0;
      prefetch_l2_line(p.x + off);
      prefetch_l2_line(p.b + off);
    }
    // b of the next step into the free slot (B[s-2])
    load_b(m1, k1, B[rq]);
    if (k == kb) mbar_wait(&BAR[st], (uint32_t)((m >> 1) & 1));
    const bool look = k == 7;  // plane k+1 is plane 0 of the next item
    if (look && m + 1 < nitems) mbar_wait(&BAR[st ^ 1], (uint32_t)(((m + 1) >> 1) & 1));
    const double* SC = SLb + st * kSlabD;
    const double* SN = look ? SLb + (st ^ 1) * kSlabD : SC;
    const int kn = (k + 1) & 7;

    // ---- shared-memory reads: face x0 / o of plane k+1, face b and corner of plane k, face x0
    //      of plane k next to my cells
    const double2 U0 = lds2w(SN + u0o + 16 * kn), U1 = lds2w(SN + u1o + 16 * kn);
    const double bf0 = SC[bo0 + bks * k], bf1 = SC[bo1 + bks * k];
    const double corn = SC[coff + 2 * k];
    const double fw0 = SC[fo0 + 16 * k], fw1 = SC[fo1 + 16 * k];
    const double2 fsn = lds2w(SC + fsno + 16 * k);
    C[r][0] = ff == 0 ? U0.y : U0.x;
    C[r][1] = ff == 0 ? U1.y : (ff == 1 ? U1.x : U0.y);
    O[r][0] = ff == 0 ? U0.x : (ff == 1 ? U0.y : U1.x);
    O[r][1] = ff == 0 ? U1.x : U1.y;

    // ---- sweep 1, face ring: x1 of my two neighbour face cells of plane k
    const double2 xc0 = X[rp][0], xc1 = X[rp][1];
    const double rA = __shfl_sync(FULL, sel4(cA, xc0, xc1), fsrc, 16);
    const double rB = __shfl_sync(FULL, sel4(cB, xc0, xc1), fsrc, 16);
    const double rC = __shfl_sync(FULL, sel4(cC, xc0, xc1), fsrc, 16);
    const double r2 = fWE ? rB : rC;
    const double own0 = fswap ? r2 : rA, own1 = fswap ? rA : r2;
    const double cc0 = C[rp][0], cc1 = C[rp][1];
    const double up = __shfl_up_sync(FULL, cc1, 1, 16), dn = __shfl_down_sync(FULL, cc0, 1, 16);
    const double lo0 = pr > 0 ? up : corn, hi1 = pr < 3 ? dn : corn;
    const double fx1a0 = face_x1(cc0, O[rp][0], own0, lo0, cc1, C[rq][0], C[r][0], bf0, alpha, beta, gamma);
    const double fx1b0 = face_x1(cc1, O[rp][1], own1, cc0, hi1, C[rq][1], C[r][1], bf1, alpha, beta, gamma);
    const double fx1a = keep_cell(p.colour, fi0, fj0, k) ? cc0 : fx1a0;
    const double fx1b = keep_cell(p.colour, fi1, fj1, k) ? cc1 : fx1b0;

    // ---- sweep 1, my four cells of plane k
    double a[4];
    own_a(xc0, xc1, X[rq][0], X[rq][1], X[r][0], X[r][1], fw0, fw1, fsn, isW, isE, isS, isN, alpha, beta, a);
    // X[s-2] is dead: x0 of the plane after the next step goes there
    load_x(m1, k1, X[rq]);
    const double2 bc0 = B[r][0], bc1 = B[r][1];
    Y[r][0].x = keep_cell(p.colour, 2 * ip, 2 * jp, k) ? xc0.x : DADD(xc0.x, DMUL(gamma, DSUB(a[0], bc0.x)));
    Y[r][0].y = keep_cell(p.colour, 2 * ip + 1, 2 * jp, k) ? xc0.y : DADD(xc0.y, DMUL(gamma, DSUB(a[1], bc0.y)));
    Y[r][1].x = keep_cell(p.colour, 2 * ip, 2 * jp + 1, k) ? xc1.x : DADD(xc1.x, DMUL(gamma, DSUB(a[2], bc1.x)));
    Y[r][1].y = keep_cell(p.colour, 2 * ip + 1, 2 * jp + 1, k) ? xc1.y : DADD(xc1.y, DMUL(gamma, DSUB(a[3], bc1.y)));
    // face x1 of plane k for the lanes next to the faces (their x2 of plane k, next step)
    GW[r][0] = __shfl_sync(FULL, fx1a, src_we, 16);
    GW[r][1] = __shfl_sync(FULL, fx1b, src_we, 16);
    GS[r][0] = __shfl_sync(FULL, fx1a, src_sn, 16);
    GS[r][1] = __shfl_sync(FULL, fx1b, src_sn, 16);

    // ---- sweep 2, my four cells of the previous plane P(s-1)
    const double2 yc0 = Y[rp][0], yc1 = Y[rp][1];
    own_a(yc0, yc1, Y[rq][0], Y[rq][1], Y[r][0], Y[r][1], GW[rp][0], GW[rp][1], make_double2(GS[rp][0], GS[rp][1]),
          isW, isE, isS, isN, alpha, beta, a);
    if (out_emit) {
      const double2 bp0 = B[rp][0], bp1 = B[rp][1];
      double2 z0, z1, r0, r1;
      const int ko = out_k;
      z0.x = keep_cell(p.colour2, 2 * ip, 2 * jp, ko) ? yc0.x : DADD(yc0.x, DMUL(gamma2, DSUB(a[0], bp0.x)));
      z0.y = keep_cell(p.colour2, 2 * ip + 1, 2 * jp, ko) ? yc0.y : DADD(yc0.y, DMUL(gamma2, DSUB(a[1], bp0.y)));
      z1.x = keep_cell(p.colour2, 2 * ip, 2 * jp + 1, ko) ? yc1.x : DADD(yc1.x, DMUL(gamma2, DSUB(a[2], bp1.x)));
      z1.y = keep_cell(p.colour2, 2 * ip + 1, 2 * jp + 1, ko) ? yc1.y : DADD(yc1.y, DMUL(gamma2, DSUB(a[3], bp1.y)));
      r0.x = DSUB(bp0.x, a[0]);
      r0.y = DSUB(bp0.y, a[1]);
      r1.x = DSUB(bp1.x, a[2]);
      r1.y = DSUB(bp1.y, a[3]);
      const int64_t g = (int64_t)out_id * 512 + 64 * out_k + q0;
      st_hint2(p.xo + g, z0, pol_stream);  // never re-read by this pass
      st_hint2(p.xo + g + 8, z1, pol_stream);
      if (WRITE_R) {
        st_hint2(p.r + g, r0, pol_stream);
        st_hint2(p.r + g + 8, r1, pol_stream);
      }
      if (RESTRICT) {
        // coarse cell (ip, jp, out_k/2) of the parent octant: the footprint's 2x2 of planes 2K, 2K+1 in
        // canonical order ((r000+r100)+(r010+r110))+((r001+r101)+(r011+r111))
        const double part = DADD(DADD(r0.x, r0.y), DADD(r1.x, r1.y));
        if (out_k & 1) {
          const int oct = out_par & 7;
          const int ox = oct & 1, oy = (oct >> 1) & 1, oz = oct >> 2;
          p.bc[(int64_t)(out_par >> 3) * 512 + (4 * ox + ip) + 8 * (4 * oy + jp) + 64 * (4 * oz + (out_k >> 1))] =
              DMUL(0.125, DADD(rpart, part));
        } else {
          rpart = part;
        }
      }
    }
    out_id = id_of(m), out_k = k, out_emit = (fl & 1) != 0, out_par = MT[m & (kMR - 1)][10];

    // ---- item m ends: the meta slot of item m-1 takes item m+7
    const bool last = k + 1 >= ke;
    __syncwarp();  // every lane has consumed its reads of stage m (item m+2 may overwrite it)
    if (last) {
      if (hl < kW2Meta / 4) {
        reinterpret_cast<int4*>(MT[(m + 7) & (kMR - 1)])[hl] = pend;
        pend = reinterpret_cast<const int4*>(MG + (int64_t)(m + 8) * kW2Meta)[hl];
      }
    }
    __syncwarp();  // the new meta slot is visible
    m = m1, k = k1;
    adv(m1, k1);
  };

  for (int s = 0; s < nsteps; s += 3) {
    step(std::integral_constant<int, 0>{});
    if (s + 1 < nsteps) step(std::integral_constant<int, 1>{});
    if (s + 2 < nsteps) step(std::integral_constant<int, 2>{});
  }
  pdl_trigger();
}

cudaError_t launch_sweep2w(const SweepArgs& a, const PairArgs& pa, const PairMaps& pm, unsigned flags,
                           cudaStream_t s) {
  if (pa.nwarps <= 0) return cudaSuccess;
  const unsigned g = (unsigned)((pa.nwarps + kW2WarpsPerSm - 1) / kW2WarpsPerSm);
  const size_t sm = sizeof(W2Smem) * kW2WarpsPerSm;
  constexpr unsigned kThreads = 32 * kW2WarpsPerSm;
  switch (flags & (SW_WRITE_R | SW_RESTRICT | SW_INTERP | SW_ZERO_X)) {
    case 0: launch_plain(sweep2w_kernel<0>, g, kThreads, sm, s, a, pa, pm); break;
    case SW_WRITE_R: launch_plain(sweep2w_kernel<SW_WRITE_R>, g, kThreads, sm, s, a, pa, pm); break;
    case SW_RESTRICT: launch_plain(sweep2w_kernel<SW_RESTRICT>, g, kThreads, sm, s, a, pa, pm); break;
    default: return cudaErrorInvalidValue;
  }
  return cudaGetLastError();
}

cudaError_t pairw_kernels_init() {
  const void* k[3] = {(const void*)sweep2w_kernel<0>, (const void*)sweep2w_kernel<SW_WRITE_R>,
                      (const void*)sweep2w_kernel<SW_RESTRICT>};
  for (int i = 0; i < 3; ++i) {
    cudaError_t e = cudaFuncSetAttribute(k[i], cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         (int)(sizeof(W2Smem) * kW2WarpsPerSm));
    if (e != cudaSuccess) return e;
    e = cudaFuncSetAttribute(k[i], cudaFuncAttributePreferredSharedMemoryCarveout, 100);
    if (e != cudaSuccess) return e;
  }
  return cudaSuccess;
}

}  // namespace mgb
