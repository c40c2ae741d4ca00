// sweep2q.cu -- two Jacobi sweeps per HBM pass, one warp per 2x2-brick pencil (temporal blocking,
// SURVEY §8(f) N1; fourth design).
//
// Same chunk plan, same per-cell expressions and therefore the same bits as sweep2p.cu (two
// separate canonical sweeps, reading A8); what changes is how a cell's neighbours reach the
// registers, because the pass is bound by the SM's shared-memory / shuffle crossbar (the LSU data
// pipe), not by FLOPs or DRAM:
//   * ONE warp owns the whole 16x16-cell tile (2x2 bricks) of its pencil and streams it up z.  A lane
//     holds a 4-wide x 2-tall cell footprint (pc = lane & 3: columns 4pc..4pc+3; jr = lane >> 2:
//     rows 2jr, 2jr+1), so a cell needs 6 (not 8) crossbar words per sweep from outside its lane.
//   * The x1 of the first sweep never goes through shared memory inside the tile: the second sweep
//     takes its in-plane neighbours by shuffles (a shared-memory round trip costs a store AND a load
//     per word, a shuffle one transfer).  Only the redundant 1-cell ring around the tile (x1 that
//     the second sweep of the tile's edge cells needs) is published, to a small ring buffer.
//   * The two rows of a footprint are kept as "sets": set s of lane jr holds tile row
//     2jr + (s ^ (jr & 1)).  Every set's in-lane S/N neighbour is the other set and its outside
//     neighbour is the same set of lane jr -/+ 1, so the second sweep's outside rows come from ONE
//     shuffle per word with a per-lane source lane, and the first sweep's 128-bit loads of the own
//     rows (and of the outside rows) hit 8 different 16-byte bank groups per quarter warp (bricks
//     1 and 3 are staged 16 B off modulo 128): conflict-free.  The stencil takes (outside, other)
//     as its (s, n) operands for both sets: for an odd row that is (n, s), and since IEEE addition is
//     commutative the canonical ((w+e)+(s+n))+(b+t) comes out bit for bit.
//   * Stages are 2-plane units (the own x0 planes by 1D bulk copies, the 2-cell slabs of the 8 side
//     neighbours, their b faces and the 4 diagonal corner columns by 3D tensor boxes) in a QD_ST-deep
//     ring, one mbarrier per stage, b of the own cells with them (kept in registers for one more plane:
//     the second sweep's b); the chunk records (brick ids) are read from global memory two records
//     ahead (the issue side keeps one field per lane: lane l issues copy l).  No CTA barrier: the
//     warp synchronises with __syncwarp.
//   * initZero folded into the first sweep (SW_ZERO_X: x0 == 0, only b is staged), so the first
//     coarse-level pass pairs up too (level 1 and 2 pre-smoothing: 6 passes instead of 1 single +
//     5 passes + 1 single).
#include <cudaTypedefs.h>

#include <type_traits>

#include "kernels.h"
#include "mg_internal.h"
#include "ptx.cuh"

namespace mgb {

namespace {

constexpr int QD_ST = 2;    // stage ring depth (2-plane units): one unit (two planes) of lead
constexpr int QD_MINB = 8;  // resident one-warp CTAs per SM (27 KB of shared memory each)
// stage layout, offsets in doubles (tensor-copy destinations 128-byte aligned).  Own brick q (2
// planes x 64) of x0 at qb(q), of b at QOB + qb(q): bricks 1 and 3 sit 16 B off modulo 128 from
// bricks 0 and 2.
__host__ __device__ constexpr int qb(int q) { return 272 * (q >> 1) + 130 * (q & 1); }
constexpr int QOB = 544;                                    // own b bricks
constexpr int QXW = 1088, QXE = 1152, QXS = 1216, QXN = 1280;  // x0 slabs, 2 boxes of 32 each (W0 W1 ...)
constexpr int QBW = 1344, QBE = 1408, QBS = 1472, QBN = 1536;  // b faces, 2 boxes of 32 each
constexpr int QCOR = 1600;                                     // SW, NW, SE, NE corner columns at +16 k
constexpr int QSTAGE = 1664;
// ring buffer of the ring cells' x1, per plane parity: W column rows j at RW + j, E rows at
// RE + (j ^ 9), S row columns i at RS + i, N columns at RN + (i ^ 10).  The permutations make both
// the ring stores (W rows 0-7 with E rows 0-7 per half warp) and the edge lanes' loads (rows of one
// set, resp. the 128-bit column pairs) conflict-free.
constexpr int QRW = 0, QRE = 16, QRS = 32, QRN = 48, QRPAR = 64;
constexpr size_t QSMEM = (size_t)(QD_ST * QSTAGE + 2 * QRPAR) * 8 + QD_ST * 8;
static_assert(qb(1) >= qb(0) + 128 && qb(2) >= qb(1) + 128 && qb(3) >= qb(2) + 128 && qb(1) % 16 == 2 &&
                  qb(2) % 16 == 0 && qb(3) % 16 == 2,
              "own bricks: disjoint, bricks 1 and 3 16 B off modulo 128");
static_assert(QOB >= qb(3) + 128 && QOB % 16 == 0 && QXW >= QOB + qb(3) + 128 && QXW % 16 == 0 && QBW % 16 == 0 && QCOR % 16 == 0 && QSTAGE % 16 == 0,
              "stage layout");
static_assert(QXE == QXW + 64 && QXS == QXW + 128 && QXN == QXW + 192 && QBE == QBW + 64 && QBS == QBW + 128 &&
                  QBN == QBW + 192,
              "slab k lands at QXW + 32 k, b face k at QBW + 32 k");
static_assert(QSMEM + 1024 <= 233472 / QD_MINB, "QD_MINB CTAs per SM must fit in shared memory");
constexpr uint32_t QTX_X = 4 * 1024 + 8 * 256 + 4 * 32;           // own x0, x0 slabs, corners
constexpr uint32_t QTX_B = 4 * 1024 + 4 * 256 + 4 * 256;            // own b, b faces W/E, S/N

__device__ __forceinline__ double2 lds2(const double* p) { return *reinterpret_cast<const double2*>(p); }
__device__ __forceinline__ int ldgi(const int32_t* p) { return __ldg(p); }
__device__ __forceinline__ double shfl_d(double v, int src) { return __shfl_sync(0xffffffffu, v, src); }

}  // namespace

template <unsigned FLAGS>
__global__ void __launch_bounds__(32, QD_MINB)
    sweep2q_kernel(SweepArgs p, PairArgs pa, const __grid_constant__ PairMaps mp) {
  pdl_wait();
  constexpr bool WRITE_R = (FLAGS & SW_WRITE_R) != 0;
  constexpr bool RESTRICT = (FLAGS & SW_RESTRICT) != 0;
  constexpr bool COLOUR = (FLAGS & SW_COLOUR) != 0;  // red-black half-sweeps (GSRB variant)
  constexpr bool ZX = (FLAGS & SW_ZERO_X) != 0;      // x0 == 0: initZero folded into the first sweep
  constexpr unsigned FULL = 0xffffffffu;
  constexpr int RANGE = 0, WARM = 1;
  extern __shared__ __align__(128) unsigned char smem_raw[];
  double* const ST = reinterpret_cast<double*>(smem_raw);  // [QD_ST][QSTAGE]
  double* const RBF = ST + QD_ST * QSTAGE;                 // [2][QRPAR] ring-cell x1
  uint64_t* const BAR = reinterpret_cast<uint64_t*>(RBF + 2 * QRPAR);
  const int l = threadIdx.x;
  const int2 cr = pa.ctas[blockIdx.x];
  const int32_t* REC = pa.meta + (int64_t)cr.x * kPenRec;  // chunk records: code, 16 brick ids, parent
  const int cnt = cr.y;
  const double alpha = p.c.alpha, beta = p.c.beta, gamma = p.c.gamma, gamma2 = p.gamma2;
  const int col1 = COLOUR ? p.colour : -1, col2 = COLOUR ? p.colour2 : -1;
  const uint64_t pol_keep = l2_evict_last(), pol_stream = l2_evict_first();

  // ---- own cells: columns 4pc..4pc+3, set s = tile row 2jr + (s ^ (jr & 1)) ----
  const int pc = l & 3, jr = l >> 2, bx = pc >> 1, q = bx + 2 * (jr >> 2), ib = (4 * pc) & 7, jo = jr & 1;
  int jb[2], oOwn[2], oOut[2], sOut[2], oEd[2], rEd[2];
#pragma unroll
  for (int s = 0; s < 2; ++s) {
    const int row = 2 * jr + (s ^ jo);
    jb[s] = row & 7;
    oOwn[s] = qb(q) + 8 * jb[s] + ib;
    const int orow = (s ^ jo) == 0 ? row - 1 : row + 1;  // the row outside the footprint
    if (orow < 0) oOut[s] = QXS + 32 * bx + 8 + ib, sOut[s] = 16;        // S slab row j = 7
    else if (orow > 15) oOut[s] = QXN + 32 * bx + ib, sOut[s] = 16;      // N slab row j = 0
    else oOut[s] = qb(bx + 2 * (orow >> 3)) + 8 * (orow & 7) + ib, sOut[s] = 64;
    oEd[s] = pc == 3 ? QXE + 32 * (row >> 3) + 2 * (row & 7) : QXW + 32 * (row >> 3) + 2 * (row & 7) + 1;
    rEd[s] = pc == 3 ? QRE + (row ^ 9) : QRW + row;
  }
  const bool edW = pc == 0, edE = pc == 3, edge = edW || edE, edSN = jr == 0 || jr == 7;
  // set 0's outside row on the tile edge (jr = 0: the S ring row, jr = 7: the N ring row), two pairs
  const int rOut0 = jr == 0 ? QRS + 4 * pc : QRN + ((4 * pc) ^ 10);
  const int rOut1 = jr == 0 ? QRS + 4 * pc + 2 : QRN + ((4 * pc + 2) ^ 10);
  const int part0 = jo ? l + 4 : l - 4, part1 = jo ? l - 4 : l + 4;  // outside row's lane, per set

  // ---- ring A: x1 of one W (lanes with bit 3 clear) / E ring cell, tile row jA ----
  const int sA = (l >> 3) & 1, hA = l >> 4, jA8 = l & 7, jA = jA8 + 8 * hA, cA = sA ? 0 : 1;
  const int XA = sA ? QXE : QXW;
  const int oAc = XA + 32 * hA + 2 * jA8 + cA, oAo = oAc + (sA ? 1 : -1), oAb = (sA ? QBE : QBW) + 32 * hA + 2 * jA8 + cA;
  int oAlo, sAlo, oAhi, sAhi;
  if (jA8 > 0) oAlo = oAc - 2, sAlo = 16;
  else if (hA == 1) oAlo = XA + 14 + cA, sAlo = 16;
  else oAlo = QCOR + (sA ? 32 : 1), sAlo = 2;  // (-1,-1): SW column 1 / (16,-1): SE column 0
  if (jA8 < 7) oAhi = oAc + 2, sAhi = 16;
  else if (hA == 0) oAhi = XA + 32 + cA, sAhi = 16;
  else oAhi = QCOR + (sA ? 48 : 17), sAhi = 2;  // (-1,16): NW column 1 / (16,16): NE column 0
  const int srcA = 4 * (jA >> 1) + (sA ? 3 : 0), setA = (jA & 1) ^ ((jA >> 1) & 1);
  const int oAr = sA ? QRE + (jA ^ 9) : QRW + jA;
  const int rciA = sA ? 0 : 7;
  // ---- ring B: x1 of one S (bit 3 clear) / N ring cell, tile column iB ----
  const int sB = (l >> 3) & 1, hB = l >> 4, iB8 = l & 7, iB = iB8 + 8 * hB;
  const int oBc = sB ? QXN + 32 * hB + iB8 : QXS + 32 * hB + 8 + iB8;
  const int oBo = sB ? oBc + 8 : oBc - 8;
  const int oBb = sB ? QBN + 32 * hB + iB8 : QBS + 32 * hB + 8 + iB8;
  const int oBown = sB ? qb(2 + hB) + 56 + iB8 : qb(hB) + iB8;
  int oBlo, sBlo, oBhi, sBhi;
  if (iB8 > 0) oBlo = oBc - 1, sBlo = 16;
  else if (hB == 1) oBlo = oBc - 32 + 7, sBlo = 16;
  else oBlo = QCOR + (sB ? 17 : 1), sBlo = 2;  // (-1,16): NW column 1 / (-1,-1): SW column 1
  if (iB8 < 7) oBhi = oBc + 1, sBhi = 16;
  else if (hB == 0) oBhi = oBc + 32 - 7, sBhi = 16;
  else oBhi = QCOR + (sB ? 48 : 32), sBhi = 2;  // (16,16): NE column 0 / (16,-1): SE column 0
  const int oBr = sB ? QRN + (iB ^ 10) : QRS + iB;
  const int rcjB = sB ? 0 : 7;

  // ---- producer: lane 0 issues every copy of a unit in straight-line code (per-lane operands of
  // the TMA instructions would make the compiler loop over the issuing lanes); lane f keeps field
  // f + 1 of the record being issued (f < 17: the 16 brick ids and the parent), lane 17 the code,
  // prefetched two records ahead ----
  const int fld = l < 17 ? l + 1 : 0;
  if (l == 0) {
    for (int s = 0; s < QD_ST; ++s) mbar_init(&BAR[s], 1);
    mbar_fence_init();
  }
  __syncwarp();
  int irec = 0, isub = 0, issued = 0;
  int fcur = ldgi(REC + fld), fnext = cnt > 1 ? ldgi(REC + kPenRec + fld) : 0;
  int fnext2 = cnt > 2 ? ldgi(REC + 2 * kPenRec + fld) : 0;
  int icode = __shfl_sync(FULL, fcur, 17);
  isub = ((icode >> 1) & 3) == WARM ? 1 : 0;
  auto issue_next = [&]() {  // uniform: stage unit (irec, isub) into stage issued % QD_ST
    const int s = issued % QD_ST, pl0 = 4 * (icode & 1) + 2 * isub;
    double* D = ST + s * QSTAGE;
    int id[16];
#pragma unroll
    for (int f = 0; f < 16; ++f) id[f] = __shfl_sync(FULL, fcur, f);  // b00 b10 b01 b11 W0 W1 E0 E1 S0 S1 N0 N1 SW NW SE NE
    fence_proxy_async();  // this lane's generic reads of the stage are ordered before the refill
    __syncwarp();
    if (l == 0) {
      mbar_expect_tx(&BAR[s], ZX ? QTX_B : QTX_X + QTX_B);
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        // evict_last: the neighbour tiles' slab copies read these bricks' faces shortly after
        if (!ZX) tma_load_1d_hint(D + qb(q), p.x + (int64_t)id[q] * 512 + 64 * pl0, 1024, &BAR[s], pol_keep);
        tma_load_1d_hint(D + QOB + qb(q), p.b + (int64_t)id[q] * 512 + 64 * pl0, 1024, &BAR[s], pol_keep);
      }
#pragma unroll
      for (int k = 0; k < 8; ++k) {  // W0 W1 E0 E1 S0 S1 N0 N1: the W / S boxes sit at the neighbour's high face
        const bool xf = k < 4, low = (k & 2) == 0;
        const int kz = id[4 + k] * 8 + pl0;
        if (!ZX) tma_load_3d(D + QXW + 32 * k, xf ? &mp.xwe : &mp.xsn, xf && low ? 6 : 0, !xf && low ? 6 : 0, kz, &BAR[s]);
        tma_load_3d(D + QBW + 32 * k, xf ? &mp.bwe : &mp.bsn, xf && low ? 6 : 0, !xf && low ? 6 : 0, kz, &BAR[s]);
      }
#pragma unroll
      for (int k = 0; k < 4; ++k)  // SW (6,7), NW (6,0), SE (0,7), NE (0,0)
        if (!ZX) tma_load_3d(D + QCOR + 16 * k, &mp.xcor, k < 2 ? 6 : 0, (k & 1) ? 0 : 7, id[12 + k] * 8 + pl0, &BAR[s]);
    }
    __syncwarp();
    ++issued;
    if (((icode >> 1) & 3) == RANGE && isub == 0) {
      isub = 1;
    } else {
      ++irec;
      fcur = fnext;
      fnext = fnext2;
      fnext2 = irec + 2 < cnt ? ldgi(REC + (int64_t)(irec + 2) * kPenRec + fld) : 0;
      icode = __shfl_sync(FULL, fcur, 17);
      isub = ((icode >> 1) & 3) == WARM ? 1 : 0;
    }
  };
  int ucur = 0;  // unit holding the current plane (units are consumed in issue order)
  while (irec < cnt && issued < QD_ST) issue_next();
  auto wait_unit = [&](int u) { mbar_wait(&BAR[u % QD_ST], (uint32_t)((u / QD_ST) & 1)); };

  // ---- registers: rings indexed by plane mod 4 (the step's kk, compile-time) ----
  double2 XR[4][2][2], YR[4][2][2], BR[2][2][2];  // [plane slot (b: plane parity)][set][column pair]
  double RA[4], RBc[4];                           // ring cells' x0 windows
  double rpart[2] = {0.0, 0.0};
#pragma unroll
  for (int k = 0; k < 4; ++k) {
    RA[k] = RBc[k] = 0.0;
#pragma unroll
    for (int s = 0; s < 2; ++s)
#pragma unroll
      for (int h = 0; h < 2; ++h) XR[k][s][h] = YR[k][s][h] = BR[k & 1][s][h] = make_double2(0.0, 0.0);
  }
  // compute-side records: current, next, the one after (prefetched), previous
  int codeC = 0, idC = 0, parC = 0, codeN = 0, idN = 0, parN = 0, codeN2 = 0, idN2 = 0, parN2 = 0;
  (void)idN;
  int codeP = 0, idP = 0, parP = 0;
  auto ldrec = [&](int n, int& code, int& id, int& par) {
    if (n < cnt) {
      const int32_t* r = REC + (int64_t)n * kPenRec;
      code = ldgi(r);
      id = ldgi(r + 1 + q);
      par = RESTRICT ? ldgi(r + 17) : 0;
    }
  };
  ldrec(0, codeN, idN, parN);
  ldrec(1, codeN2, idN2, parN2);

  // one step: sweep 1 on plane g (in-chunk plane kk), the ring, sweep 2 on plane g - 1
  auto step = [&](auto kkc, const bool start, const bool sw2, const bool cool) {
    constexpr int kk = decltype(kkc)::value;
    constexpr int kp = (kk + 1) & 3, km1 = (kk + 3) & 3, km2 = (kk + 2) & 3;
    constexpr int pl0 = kk & 1, pl1 = (kk + 1) & 1;  // planes g, g + 1 within their units
    if (kk == 0 || start) wait_unit(ucur);
    if (kk & 1) wait_unit(ucur + 1);
    const double* S0 = ST + (ucur % QD_ST) * QSTAGE;
    const double* S1 = (kk & 1) ? ST + ((ucur + 1) % QD_ST) * QSTAGE : S0;
    double2(&Xm)[2][2] = XR[km1];
    double2(&X)[2][2] = XR[kk];
    double2(&Xp)[2][2] = XR[kp];
    double2(&Ym)[2][2] = YR[km2];
    double2(&Yc)[2][2] = YR[km1];
    double2(&Y)[2][2] = YR[kk];
    if (start) {  // first step of a run (warm-up plane 7 = unit plane 1): prime the windows
#pragma unroll
      for (int s = 0; s < 2; ++s)
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          Xm[s][h] = ZX ? make_double2(0.0, 0.0) : lds2(S0 + oOwn[s] + 2 * h);
          X[s][h] = ZX ? make_double2(0.0, 0.0) : lds2(S0 + oOwn[s] + 64 + 2 * h);
        }
      RA[km1] = ZX ? 0.0 : S0[oAc];
      RA[kk] = ZX ? 0.0 : S0[oAc + 16];
      RBc[km1] = ZX ? 0.0 : S0[oBc];
      RBc[kk] = ZX ? 0.0 : S0[oBc + 16];
    }
    // b of the own cells, plane g (kept for sweep 2 of the next step)
#pragma unroll
    for (int s = 0; s < 2; ++s)
#pragma unroll
      for (int h = 0; h < 2; ++h) BR[kk & 1][s][h] = lds2(S0 + QOB + oOwn[s] + 64 * pl0 + 2 * h);
    const int kz1 = 4 * (codeC & 1) + kk;  // in-brick plane of g (red-black colour)

    // ---------------- sweep 1, own cells, plane g ----------------
    {
      double2 xo[2][2];
#pragma unroll
      for (int s = 0; s < 2; ++s)
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          Xp[s][h] = ZX ? make_double2(0.0, 0.0) : lds2(S1 + oOwn[s] + 64 * pl1 + 2 * h);
          xo[s][h] = ZX ? make_double2(0.0, 0.0) : lds2(S0 + oOut[s] + sOut[s] * pl0 + 2 * h);
        }
      double ed[2] = {0.0, 0.0};
      if (!ZX && edge) {
        ed[0] = S0[oEd[0] + 16 * pl0];
        ed[1] = S0[oEd[1] + 16 * pl0];
      }
#pragma unroll
      for (int s = 0; s < 2; ++s) {
        const double wl = __shfl_up_sync(FULL, X[s][1].y, 1), er = __shfl_down_sync(FULL, X[s][0].x, 1);
        const double W = edW ? ed[s] : wl, E = edE ? ed[s] : er;
        const double c0 = X[s][0].x, c1 = X[s][0].y, c2 = X[s][1].x, c3 = X[s][1].y;
        const double2 o0 = X[s ^ 1][0], o1 = X[s ^ 1][1], b0 = BR[kk & 1][s][0], b1 = BR[kk & 1][s][1];
        // (s, n) = (outside, other set): for an odd row that is (n, s) -- same bits (a + b == b + a)
        const double a0 = stencil_a(c0, W, c1, xo[s][0].x, o0.x, Xm[s][0].x, Xp[s][0].x, alpha, beta);
        const double a1 = stencil_a(c1, c0, c2, xo[s][0].y, o0.y, Xm[s][0].y, Xp[s][0].y, alpha, beta);
        const double a2 = stencil_a(c2, c1, c3, xo[s][1].x, o1.x, Xm[s][1].x, Xp[s][1].x, alpha, beta);
        const double a3 = stencil_a(c3, c2, E, xo[s][1].y, o1.y, Xm[s][1].y, Xp[s][1].y, alpha, beta);
        Y[s][0].x = keep_cell(col1, ib, jb[s], kz1) ? c0 : DADD(c0, DMUL(gamma, DSUB(a0, b0.x)));
        Y[s][0].y = keep_cell(col1, ib + 1, jb[s], kz1) ? c1 : DADD(c1, DMUL(gamma, DSUB(a1, b0.y)));
        Y[s][1].x = keep_cell(col1, ib + 2, jb[s], kz1) ? c2 : DADD(c2, DMUL(gamma, DSUB(a2, b1.x)));
        Y[s][1].y = keep_cell(col1, ib + 3, jb[s], kz1) ? c3 : DADD(c3, DMUL(gamma, DSUB(a3, b1.y)));
      }
    }
    // ---------------- sweep 1, the two ring cells of this lane, plane g ----------------
    {
      double* R1 = RBF + (kk & 1) * QRPAR;  // parity of plane g
      // ring A's tile-edge neighbour: column 0 (W) / 15 (E) of its row, from the lane that holds it
      const double v0 = pc == 0 ? X[0][0].x : X[0][1].y, v1 = pc == 0 ? X[1][0].x : X[1][1].y;
      const double w0 = shfl_d(v0, srcA), w1 = shfl_d(v1, srcA);
      RA[kp] = ZX ? 0.0 : S1[oAc + 16 * pl1];
      RBc[kp] = ZX ? 0.0 : S1[oBc + 16 * pl1];
      {
        const double own = setA ? w1 : w0;
        const double o = ZX ? 0.0 : S0[oAo + 16 * pl0], lo = ZX ? 0.0 : S0[oAlo + sAlo * pl0];
        const double hi = ZX ? 0.0 : S0[oAhi + sAhi * pl0], bv = S0[oAb + 16 * pl0];
        // ((o + own) + (lo + hi)) + (b + t): the canonical ((w+e)+(s+n))+(b+t) up to the order of
        // the operands of single additions (IEEE addition is commutative: bit for bit equal)
        const double sum = DADD(DADD(DADD(o, own), DADD(lo, hi)), DADD(RA[km1], RA[kp]));
        const double a = DADD(DMUL(alpha, RA[kk]), DMUL(beta, sum));
        R1[oAr] = keep_cell(col1, rciA, jA8, kz1) ? RA[kk] : DADD(RA[kk], DMUL(gamma, DSUB(a, bv)));
      }
      {
        const double own = ZX ? 0.0 : S0[oBown + 64 * pl0];
        const double o = ZX ? 0.0 : S0[oBo + 16 * pl0], lo = ZX ? 0.0 : S0[oBlo + sBlo * pl0];
        const double hi = ZX ? 0.0 : S0[oBhi + sBhi * pl0], bv = S0[oBb + 16 * pl0];
        const double sum = DADD(DADD(DADD(o, own), DADD(lo, hi)), DADD(RBc[km1], RBc[kp]));
        const double a = DADD(DMUL(alpha, RBc[kk]), DMUL(beta, sum));
        R1[oBr] = keep_cell(col1, iB8, rcjB, kz1) ? RBc[kk] : DADD(RBc[kk], DMUL(gamma, DSUB(a, bv)));
      }
    }
    // (the ring x1 of plane g is read by sweep 2 of the NEXT step, after the __syncwarp below; this
    // step's sweep 2 reads the other parity)
    // ---------------- sweep 2, own cells, plane g - 1 ----------------
    {
      constexpr int par2 = (kk + 1) & 1;  // parity of plane g - 1
      const double* R2 = RBF + par2 * QRPAR;
      double2 yo[2][2];
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        yo[0][h].x = shfl_d(Yc[0][h].x, part0);
        yo[0][h].y = shfl_d(Yc[0][h].y, part0);
        yo[1][h].x = shfl_d(Yc[1][h].x, part1);
        yo[1][h].y = shfl_d(Yc[1][h].y, part1);
      }
      if (edSN) {  // set 0 of the tile's first / last row: the S / N ring row
        yo[0][0] = lds2(R2 + rOut0);
        yo[0][1] = lds2(R2 + rOut1);
      }
      double e2[2] = {0.0, 0.0};
      if (edge) {
        e2[0] = R2[rEd[0]];
        e2[1] = R2[rEd[1]];
      }
      constexpr int km = (kk + 3) & 3;  // plane g - 1 within its chunk
      const int code2 = kk > 0 ? codeC : codeP, id2 = kk > 0 ? idC : idP;
      const int kz2 = 4 * (code2 & 1) + km;
      double rs[2] = {0.0, 0.0};  // restriction: per coarse column, rows summed
#pragma unroll
      for (int s = 0; s < 2; ++s) {
        const double wl = __shfl_up_sync(FULL, Yc[s][1].y, 1), er = __shfl_down_sync(FULL, Yc[s][0].x, 1);
        const double W = edW ? e2[s] : wl, E = edE ? e2[s] : er;
        const double c0 = Yc[s][0].x, c1 = Yc[s][0].y, c2 = Yc[s][1].x, c3 = Yc[s][1].y;
        const double2 o0 = Yc[s ^ 1][0], o1 = Yc[s ^ 1][1], b0 = BR[(kk + 1) & 1][s][0], b1 = BR[(kk + 1) & 1][s][1];
        const double a0 = stencil_a(c0, W, c1, yo[s][0].x, o0.x, Ym[s][0].x, Y[s][0].x, alpha, beta);
        const double a1 = stencil_a(c1, c0, c2, yo[s][0].y, o0.y, Ym[s][0].y, Y[s][0].y, alpha, beta);
        const double a2 = stencil_a(c2, c1, c3, yo[s][1].x, o1.x, Ym[s][1].x, Y[s][1].x, alpha, beta);
        const double a3 = stencil_a(c3, c2, E, yo[s][1].y, o1.y, Ym[s][1].y, Y[s][1].y, alpha, beta);
        double2 z0, z1, r0, r1;
        z0.x = keep_cell(col2, ib, jb[s], kz2) ? c0 : DADD(c0, DMUL(gamma2, DSUB(a0, b0.x)));
        z0.y = keep_cell(col2, ib + 1, jb[s], kz2) ? c1 : DADD(c1, DMUL(gamma2, DSUB(a1, b0.y)));
        z1.x = keep_cell(col2, ib + 2, jb[s], kz2) ? c2 : DADD(c2, DMUL(gamma2, DSUB(a2, b1.x)));
        z1.y = keep_cell(col2, ib + 3, jb[s], kz2) ? c3 : DADD(c3, DMUL(gamma2, DSUB(a3, b1.y)));
        r0.x = DSUB(b0.x, a0), r0.y = DSUB(b0.y, a1), r1.x = DSUB(b1.x, a2), r1.y = DSUB(b1.y, a3);
        const int64_t go = (int64_t)id2 * 512 + 64 * kz2 + 8 * jb[s] + ib;
        if (sw2) {
          st_hint2(p.xo + go, z0, pol_stream);  // never re-read by this pass
          st_hint2(p.xo + go + 2, z1, pol_stream);
        }
        if (WRITE_R && sw2) {
          st_hint2(p.r + go, r0, pol_stream);
          st_hint2(p.r + go + 2, r1, pol_stream);
        }
        if (RESTRICT) {
          // coarse columns 2pc, 2pc+1: (r(0,j) + r(1,j)) of this row
          if (s == 0) {
            rs[0] = DADD(r0.x, r0.y);
            rs[1] = DADD(r1.x, r1.y);
          } else {
            // ((r000+r100)+(r010+r110)): the two rows' pair sums added (set order = row order or its
            // mirror: commutative, same bits)
            rs[0] = DADD(rs[0], DADD(r0.x, r0.y));
            rs[1] = DADD(rs[1], DADD(r1.x, r1.y));
          }
        }
      }
      if (RESTRICT) {
        // this lane's 4x2 footprint over two planes is two coarse cells: plane k = 0 sum + plane k = 1 sum
        if ((km & 1) == 0) {
          rpart[0] = rs[0];
          rpart[1] = rs[1];
        } else if (sw2) {
          const int pr = kk > 0 ? parC : parP;
          const int K = 4 * ((pr >> 2) & 1) + (kz2 >> 1);
          const double2 v = make_double2(DMUL(0.125, DADD(rpart[0], rs[0])), DMUL(0.125, DADD(rpart[1], rs[1])));
          *reinterpret_cast<double2*>(p.bc + (int64_t)(pr >> 3) * 512 + 2 * pc + 8 * jr + 64 * K) = v;
        }
      }
    }
    __syncwarp();  // sweep 2's ring reads done before the next step overwrites that parity
    if ((kk & 1) || cool) {  // the unit of plane g is consumed: refill its stage
      ++ucur;
      while (irec < cnt && issued < ucur + QD_ST) issue_next();
    }
  };

  for (int c = 0; c < cnt; ++c) {
    codeP = codeC, idP = idC, parP = parC;
    codeC = codeN, idC = idN, parC = parN;
    codeN = codeN2, idN = idN2, parN = parN2;
    ldrec(c + 2, codeN2, idN2, parN2);
    const int type = (codeC >> 1) & 3, typeP = c > 0 ? (codeP >> 1) & 3 : WARM;
    using I0 = std::integral_constant<int, 0>;
    using I1 = std::integral_constant<int, 1>;
    using I2 = std::integral_constant<int, 2>;
    using I3 = std::integral_constant<int, 3>;
    if (type == WARM) {
      step(I3{}, true, false, false);
    } else if (type == RANGE) {
      step(I0{}, false, typeP == RANGE, false);
      step(I1{}, false, true, false);
      step(I2{}, false, true, false);
      step(I3{}, false, true, false);
    } else {  // COOL: plane 0 of the layer above (sweep 1), the run's last plane (sweep 2)
      step(I0{}, false, true, true);
    }
  }
  pdl_trigger();
}

bool quad_supports(unsigned flags) {
  const unsigned fl = flags & (SW_WRITE_R | SW_RESTRICT | SW_INTERP);
  return fl == 0 || fl == SW_WRITE_R || fl == SW_RESTRICT;
}

cudaError_t encode_quad_maps(const double* x, const double* b, int64_t n_alloc, PairMaps* out) {
  const unsigned we[3] = {2, 8, 2}, sn[3] = {8, 2, 2}, cor[3] = {2, 1, 2};
  cudaError_t e;
  if ((e = encode_box_map(x, n_alloc, we, &out->xwe)) != cudaSuccess) return e;
  if ((e = encode_box_map(x, n_alloc, sn, &out->xsn)) != cudaSuccess) return e;
  if ((e = encode_box_map(x, n_alloc, cor, &out->xcor)) != cudaSuccess) return e;
  if ((e = encode_box_map(b, n_alloc, we, &out->bwe)) != cudaSuccess) return e;
  return encode_box_map(b, n_alloc, sn, &out->bsn);
}

namespace {
template <unsigned F>
void quad_launch(unsigned g, cudaStream_t s, const SweepArgs& a, const PairArgs& pa, const PairMaps& pm) {
  launch_plain(sweep2q_kernel<F>, g, 32, QSMEM, s, a, pa, pm);
}
template <unsigned F>
cudaError_t quad_attr() {
  cudaError_t e = cudaFuncSetAttribute(sweep2q_kernel<F>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)QSMEM);
  if (e != cudaSuccess) return e;
  return cudaFuncSetAttribute(sweep2q_kernel<F>, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
}
// every supported flag combination: {plain, +r, +restriction} x {colour} x {x0 == 0}
#define QUAD_FLAG_LIST(X)                                                                                     \
  X(0) X(SW_WRITE_R) X(SW_RESTRICT) X(SW_COLOUR) X(SW_WRITE_R | SW_COLOUR) X(SW_RESTRICT | SW_COLOUR)        \
  X(SW_ZERO_X) X(SW_ZERO_X | SW_WRITE_R) X(SW_ZERO_X | SW_RESTRICT) X(SW_ZERO_X | SW_COLOUR)                  \
  X(SW_ZERO_X | SW_WRITE_R | SW_COLOUR) X(SW_ZERO_X | SW_RESTRICT | SW_COLOUR)
}  // namespace

cudaError_t launch_sweep2q(const SweepArgs& a, const PairArgs& pa, const PairMaps& pm, unsigned flags,
                           cudaStream_t s) {
  if (pa.nctas <= 0) return cudaSuccess;
  const unsigned g = (unsigned)pa.nctas;
  const unsigned col = (a.colour >= 0 || a.colour2 >= 0) ? SW_COLOUR : 0u;
  switch ((flags & (SW_WRITE_R | SW_RESTRICT | SW_INTERP | SW_ZERO_X)) | col) {
#define QUAD_CASE(F)                \
  case (F):                         \
    quad_launch<(F)>(g, s, a, pa, pm); \
    break;
    QUAD_FLAG_LIST(QUAD_CASE)
#undef QUAD_CASE
    default:
      return cudaErrorInvalidValue;
  }
  return cudaGetLastError();
}

cudaError_t quad_kernels_init() {
  cudaError_t e = cudaSuccess;
#define QUAD_ATTR(F) \
  if ((e = quad_attr<(F)>()) != cudaSuccess) return e;
  QUAD_FLAG_LIST(QUAD_ATTR)
#undef QUAD_ATTR
  return e;
}

}  // namespace mgb
