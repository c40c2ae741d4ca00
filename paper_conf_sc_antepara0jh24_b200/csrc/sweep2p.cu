// sweep2p.cu -- two Jacobi sweeps per HBM pass over 2x2-brick pencils (temporal blocking,
// SURVEY §8(f) N1; third design).
//
// The paper deepens the ghost zone to a brick so several smooths run per exchange
// (P:L156); this kernel applies the idea on chip: x0 -> x1 -> x2 in one pass over HBM
// (read x0, b; write x2: 24 B per point for TWO sweeps).  Each sweep is exactly the
// canonical smooth(+residual) of kernels.cu (reading A8), so x2 is bit-identical to two
// separate sweeps.
//
// Data flow (why it is shaped like this: DESIGN.md §7.1).  A CTA of two warps walks a
// stream of half-layer CHUNKS of 2x2-brick pencils (layout.cpp pencil_table):
// [warm-up half, (layer half 0, half 1)..., cool-down half] per run of a tile column.
//   * A chunk = 4 z-planes of the 16x16-cell tile.  Lanes 0-11 of both warps stage it by TMA
//     into a 2-stage shared-memory ring (one mbarrier per stage): the four own x0 bricks'
//     planes (1D bulk, 2 KB each), the 2-cell-deep x0 slabs of the 8 side neighbours
//     (3D tensor boxes {2,8,4} / {8,2,4}), their b faces, the 4 diagonal corner columns.
//   * The k-direction lives in registers: a lane owns a 2x2 cell footprint of the tile
//     (pair column p = lane & 7, row pair jp = lane >> 3, warp = brick row), keeps x0 of
//     planes g-1..g+1 and x1 of planes g-2..g, and per step g
//       - sweep 1 on plane g: x1 of its 4 cells (S/N rows by LDS.128 from the staged bricks,
//         W/E by shuffles, tile edges from the slabs), published to a 2-plane x1 buffer;
//       - x1 of ONE ring cell (the redundant 1-cell ring around the tile the second sweep
//         needs: warp 0 = W/E rows 0-7 + the S row, warp 1 = W/E rows 8-15 + the N row);
//       - sweep 2 on plane g-1 from the x1 registers and the x1 buffer, streamed to HBM with
//         r or the restricted coarse b (the 2x2 footprint is exactly one coarse column, so the
//         2x2x2 restriction sum forms in registers).
//   * b of the own cells by 128-bit loads two planes ahead; one CTA barrier per plane.
// Every cell of a 2x2-brick tile moves 24 B per pass from HBM; through the SM's shared-memory
// crossbar it moves about half of what sweep2.cu's one-brick items move (no k-plane
// re-reads, no x1 round trip for own cells, a 25% instead of 50% redundant ring).
#include <cudaTypedefs.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <type_traits>
#include <vector>

#include "kernels.h"
#include "mg_internal.h"
#include "ptx.cuh"

namespace mgb {

namespace {

constexpr int PN_ST = 2;          // TMA stages (half-layer chunks): chunk c+1 lands while chunk c is swept
constexpr int PN_MINB = 6;        // resident CTAs per SM (37.8 KB of shared memory each, <= 168 registers)
constexpr int PN_THREADS = 64;    // two warps: warp w = brick row w of the tile
// stage layout, offsets in doubles.  Own bricks q = bx + 2 by at 264 q (2112 B apart: the two
// bricks of a tile row sit 64 B apart modulo 128, so a quarter-warp's 128-bit loads of one tile
// row hit all 32 banks); tensor-copy destinations 128-byte aligned.
constexpr int OWN_STRIDE = 264;
constexpr int XW = 1056, XE = 1184, XS = 1312, XN = 1440;  // 2 boxes of 64 each: x0 slabs
constexpr int BW = 1568, BE = 1696;                        // 2 boxes of 64: b of the W / E bricks
constexpr int BS = 1824, BN = 1888;                        // 2 boxes of 32: b of the S / N bricks
constexpr int COR = 1952;                                  // 4 boxes of 8 (16 apart): SW, NW, SE, NE
constexpr int STAGE = 2016;
// x1 buffers (offsets from XP, in doubles): per parity p, tile rows -1..15 at PUB p (row -1: the S ring);
// the N ring rows (tile row 16) at NROW + 16 p, 64 B off the S rows modulo 128, so the S and N ring
// stores of one brick column (one half-warp) fall in complementary banks; the W / E ring columns at
// RWE_OFF (W rows 0-15 at 16 p, E rows at RWE_E + 16 p: the W and E ring stores of a half-warp and
// the edge lanes' 128-bit loads of a quarter-warp are conflict-free)
constexpr int PUB = 17 * 16;
constexpr int NROW = 2 * PUB + 8;
constexpr int RWE_OFF = NROW + 32, RWE_E = 40, RWE_PAR = 16;
constexpr int XP_SIZE = RWE_OFF + RWE_E + 2 * RWE_PAR;  // 656
static_assert(STAGE * 8 % 128 == 0 && XW * 8 % 128 == 0 && BS * 8 % 128 == 0 && COR * 8 % 128 == 0, "align");
static_assert(3 * OWN_STRIDE + 256 <= XW, "own bricks fit");
__device__ __forceinline__ double2 lds_d2(const double* p) { return *reinterpret_cast<const double2*>(p); }
constexpr int MRS = 4;  // chunk record ring slots (record n in slot n % 4)
constexpr size_t SMEM_BYTES = (size_t)(PN_ST * STAGE + XP_SIZE) * 8 + 16 + MRS * kPenRec * 4;
static_assert(SMEM_BYTES + 1024 <= 233472 / PN_MINB, "PN_MINB CTAs per SM must fit in shared memory");

}  // namespace

template <unsigned FLAGS>
__global__ void __launch_bounds__(PN_THREADS, PN_MINB)
    sweep2p_kernel(SweepArgs p, PairArgs pa, const __grid_constant__ PairMaps mp) {
  pdl_wait();
  constexpr bool WRITE_R = (FLAGS & SW_WRITE_R) != 0;
  constexpr bool RESTRICT = (FLAGS & SW_RESTRICT) != 0;
  constexpr bool COLOUR = (FLAGS & SW_COLOUR) != 0;  // red-black half-sweeps (GSRB variant)
  constexpr bool ZX = (FLAGS & SW_ZERO_X) != 0;      // x0 == 0: initZero folded into the first sweep
  constexpr bool PEER = (FLAGS & SW_PEER) != 0;      // x of ghost bricks from their owners' fields
  constexpr unsigned FULL = 0xffffffffu;
  constexpr int RANGE = 0, WARM = 1, COOL = 2;
  // x0 read from the stage, or 0 (ZX: nothing of x0 is staged; every sweep-1 operand is +0, so the
  // first sweep computes the canonical expression on zeros, exactly what initZero + a sweep compute)
  auto x0d = [&](const double* a) { return ZX ? 0.0 : *a; };
  auto x0d2 = [&](const double* a) { return ZX ? make_double2(0.0, 0.0) : lds_d2(a); };
  extern __shared__ __align__(128) unsigned char smem_raw[];
  double* const ST = reinterpret_cast<double*>(smem_raw);  // [PN_ST][STAGE]
  double* const XP = ST + PN_ST * STAGE;                    // x1 of tile rows -1..16 (layout above)
  double* const RWE = XP + RWE_OFF;                         // x1 of the W / E ring columns
  uint64_t* const BAR = reinterpret_cast<uint64_t*>(XP + XP_SIZE);
  int* const MR = reinterpret_cast<int*>(BAR + 2);  // [MRS][kPenRec] chunk records, 16-byte aligned slots
  const int col1 = COLOUR ? p.colour : -1, col2 = COLOUR ? p.colour2 : -1;
  const int t = threadIdx.x, w = t >> 5, l = t & 31;
  if (pa.trace && threadIdx.x == 0) {  // (MG_PEN_TRACE measurement runs only)
    unsigned long long t0;
    unsigned sm;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t0));
    asm volatile("mov.u32 %0, %smid;" : "=r"(sm));
    pa.trace[2 * blockIdx.x] = t0;
    pa.trace[2 * 65536 + blockIdx.x] = sm | ((unsigned long long)pa.ctas[blockIdx.x].y << 32);
  }
  const int2 cr = pa.ctas[blockIdx.x];
  const int32_t* REC = pa.meta + (int64_t)cr.x * kPenRec;  // chunk records: code, 16 brick ids, parent
  const int cnt = cr.y;
  const double alpha = p.c.alpha, beta = p.c.beta, gamma = p.c.gamma, gamma2 = p.gamma2;
  // L2 policies (evict_normal for x0, b or x2 measured no different: DESIGN.md §7.1)
  // (created at each use -- one ALU op -- rather than held: two 64-bit values fewer live in registers)
#define pol_keep l2_evict_last()
#define pol_stream l2_evict_first()

  // ---- own-cell role: cells (2p + a, 8w + 2jp + r) of the tile ----
  const int pc = l & 7, jp = l >> 3, bx = pc >> 2, ib = 2 * (pc & 3), jb = 2 * jp, q = bx + 2 * w;
  const int oO = OWN_STRIDE * q + 8 * jb + ib;  // row jb of brick q at plane 0; row jb+1 at +8
  int oS, sS, oN, sN;                           // S row (jb-1) / N row (jb+2) pair at plane 0, plane stride
  if (jb > 0) oS = oO - 8, sS = 64;
  else if (w == 1) oS = OWN_STRIDE * (q - 2) + 56 + ib, sS = 64;
  else oS = XS + 64 * bx + 8 + ib, sS = 16;  // S slab row j = 7
  if (jb < 6) oN = oO + 16, sN = 64;
  else if (w == 0) oN = OWN_STRIDE * (q + 2) + ib, sN = 64;
  else oN = XN + 64 * bx + ib, sN = 16;  // N slab row j = 0
  const bool edW = pc == 0, edE = pc == 7;
  const int oEd = edE ? XE + 64 * w + 2 * jb : XW + 64 * w + 2 * jb + 1;  // tile-edge W / E x0 (rows jb, jb+1: +2)
  const int R0 = 8 * w + jb;                                              // tile row of my row 0
  const int pO = (R0 + 1) * 16 + 2 * pc;                                  // my row 0 in the x1 buffer
  const bool nrow = R0 + 2 == 16;                                         // row R0 + 2 is the N ring row
  const int pN = nrow ? NROW + 2 * pc : pO + 32, sPN = nrow ? RWE_PAR : PUB;  // its offset, parity stride
  const int oRwe = (edE ? RWE_E : 0) + R0;                                // ring x1 column, rows R0, R0+1

  // ---- ring role: x1 of one cell of the 1-cell ring around the tile ----
  int oc, oo, oown, olo, slo, ohi, shi, ob, sb, oout, rstr, rci, rcj;
  if (l < 16) {  // W (lanes 0-7) / E (8-15) face, tile row 8w + j
    const int side = l >> 3, j = l & 7, cc = side ? 0 : 1;
    const int X = side ? XE : XW;
    oc = X + 64 * w + 2 * j + cc;
    oo = X + 64 * w + 2 * j + (cc ^ 1);
    oown = OWN_STRIDE * (2 * w + side) + 8 * j + (side ? 7 : 0);
    if (j > 0) olo = oc - 2, slo = 16;
    else if (w == 1) olo = X + 14 + cc, slo = 16;
    else olo = COR + (side ? 32 : 0) + cc, slo = 2;  // SW / SE corner
    if (j < 7) ohi = oc + 2, shi = 16;
    else if (w == 0) ohi = X + 64 + cc, shi = 16;
    else ohi = COR + (side ? 48 : 16) + cc, shi = 2;  // NW / NE corner
    ob = (side ? BE : BW) + 64 * w + 2 * j + cc, sb = 16;
    oout = RWE_OFF + RWE_E * side + 8 * w + j, rstr = RWE_PAR;  // RWE[side col + row] + 16 par
    rci = side ? 0 : 7, rcj = j;
  } else {  // S (lanes 16-23) / N (24-31) ring rows over brick column bxr = w (tile columns 8w + i8):
            // the S and N slab rows of one brick column sit in complementary banks
    const int i8 = l & 7, bxr = w, i = 8 * w + i8;
    const bool S = l < 24;
    const int X = S ? XS : XN, rowc = S ? 8 : 0, rowo = S ? 0 : 8;
    oc = X + 64 * bxr + rowc + i8;
    oo = X + 64 * bxr + rowo + i8;
    oown = S ? OWN_STRIDE * bxr + i8 : OWN_STRIDE * (2 + bxr) + 56 + i8;
    if (i > 0) olo = X + 64 * ((i - 1) >> 3) + rowc + ((i - 1) & 7), slo = 16;
    else olo = COR + (S ? 0 : 16) + 1, slo = 2;  // SW / NW corner (i = 7)
    if (i < 15) ohi = X + 64 * ((i + 1) >> 3) + rowc + ((i + 1) & 7), shi = 16;
    else ohi = COR + (S ? 32 : 48), shi = 2;  // SE / NE corner (i = 0)
    ob = (S ? BS : BN) + 32 * bxr + i8, sb = 8;
    oout = S ? i : NROW + i, rstr = S ? PUB : RWE_PAR;  // row -1 / 16, column i
    rci = i8, rcj = S ? 7 : 0;
  }

  if (t == 0) {
    for (int s = 0; s < PN_ST; ++s) mbar_init(&BAR[s], 2);  // one arrive.expect_tx per warp
    mbar_fence_init();
  }
  __syncthreads();

  // ---- chunk records: record n lands in ring slot n % 4 with chunk n-1's TMA (records 0 and 1 by
  // plain loads here), so it is in shared memory once chunk n-1 has been waited for ----
  auto mr = [&](int n, int f) { return MR[(n % MRS) * kPenRec + f]; };
  for (int e = t; e < 2 * kPenRec; e += PN_THREADS)
    if (e < cnt * kPenRec) MR[e] = REC[e];

  // ---- producer: lanes 0-11 of each warp, one TMA copy each per chunk.  Warp 0: the four own
  // bricks' half (1D bulk) and the 8 x0 side slabs; warp 1: the 8 b faces, the 4 corner columns
  // and (lane 12) the record of the chunk after ----
  int issued = 0;
  // PEER: this lane's entry of the chunk's peer ids (warp 0 lanes 0-11: own bricks, side slabs; warp 1
  // lanes 8-11: corner columns), the one of the chunk to issue next held in a register
  const bool xlane = (w == 0 && l < 12) || (w == 1 && l >= 8 && l < 12);
  auto pid_load = [&](int n) -> int {
    return (PEER && xlane && n < cnt) ? __ldg(pa.pid + ((int64_t)(cr.x + n) * 16 + (w == 0 ? l : l + 4))) : -1;
  };
  int pid_cur = pid_load(0);
  auto issue = [&]() {  // both warps (uniform): stage chunk `issued`
    const int n = issued, s = n % PN_ST, code = mr(n, 0), half = code & 1;
    const bool rec = n + 1 >= 2 && n + 1 < cnt;
    const int id = l < 12 ? mr(n, 1 + (w == 0 ? l : l + 4)) : 0;
    double* D = ST + s * STAGE;
    fence_proxy_async();
    if (l == 0)
      mbar_expect_tx(&BAR[s], w == 0 ? (ZX ? 0 : 4 * 2048 + 8 * 512)
                                     : 4 * 512 + 4 * 256 + (ZX ? 0 : 4 * 64) + (rec ? kPenRec * 4 : 0));
    __syncwarp();
    const int kz = id * 8 + 4 * half;
    // x source of this lane's copy: the local field, or (PEER, a ghost brick) its owner's field; the
    // entry's peer id was loaded one chunk ahead (no dependent load in the issue)
    int xid = id;
    const CUtensorMap* xmaps = &mp.xwe;  // xwe, xsn, xcor (consecutive in PairMaps and in rmaps)
    bool remote = false;
    int pid_rank = 0;
    if (PEER) {
      const int pv = pid_cur;
      pid_cur = pid_load(n + 1);
      if (pv >= 0) {
        remote = true;
        pid_rank = pv >> 24;
        xid = pv & 0xffffff;
        xmaps = pa.rmaps + 3 * (pv >> 24);
      }
    }
    const int xkz = xid * 8 + 4 * half;
    if (w == 0) {
      if (ZX) {
        // nothing of x0 is staged
      } else if (PEER && remote && l < 4) {  // the owner's half brick
        tma_load_1d(D + OWN_STRIDE * l, mp.rbase[pid_rank] + (int64_t)xid * 512 + 256 * half, 2048, &BAR[s]);
      } else if (l < 4) {
        // evict_last: the neighbour tiles' slab copies read these bricks' faces shortly after
        tma_load_1d_hint(D + OWN_STRIDE * l, p.x + (int64_t)id * 512 + 256 * half, 2048, &BAR[s], pol_keep);
      } else if (l < 12) {
        const bool xf = l < 8, lowside = ((l - 4) & 2) == 0;  // W / S boxes sit at the high face
        tma_load_3d(D + XW + 64 * (l - 4), xf ? xmaps : xmaps + 1, xf && lowside ? 6 : 0,
                    !xf && lowside ? 6 : 0, xkz, &BAR[s]);
      }
    } else {
      if (l < 4) {
        tma_load_3d(D + BW + 64 * l, &mp.bwe, l < 2 ? 6 : 0, 0, kz, &BAR[s]);
      } else if (l < 8) {
        tma_load_3d(D + BS + 32 * (l - 4), &mp.bsn, 0, l < 6 ? 7 : 0, kz, &BAR[s]);
      } else if (l < 12) {  // SW (6,7), NW (6,0), SE (0,7), NE (0,0)
        const int cc = l - 8;
        if (!ZX) tma_load_3d(D + COR + 16 * cc, xmaps + 2, cc < 2 ? 6 : 0, (cc & 1) ? 0 : 7, xkz, &BAR[s]);
      } else if (l == 12 && rec) {  // slot (n+1) % 4 held record n-3, consumed long ago
        tma_load_1d(MR + ((n + 1) % MRS) * kPenRec, REC + (int64_t)(n + 1) * kPenRec, kPenRec * 4, &BAR[s]);
      }
    }
    ++issued;
  };
  // chunks are waited for in order (uniform counter)
  int nwait = 0;
  auto wait_upto = [&](int n) {
    while (nwait <= n) {
      mbar_wait(&BAR[nwait % PN_ST], (uint32_t)((nwait / PN_ST) & 1));
      ++nwait;
    }
  };

  // ---- registers: x0 planes g-1, g, g+1; x1 planes g-2, g-1, g; b of planes g-1 .. g+2 ----
  // rings indexed by plane mod 4 (= the step's kk, a compile-time constant: no register moves
  // between steps): x0 (planes g-1..g+1), x1 (g-2..g), b (g-1, g), the ring cell's x0 (g-1..g+1)
  // b of the own cells: plane-mod-8 ring of 128-bit loads issued four planes ahead (slot of plane
  // g = g mod 8 = 4 (c mod 2) + kk; a run has an even number of chunks and starts at an even c,
  // so c's parity is known from the chunk's type and half: compile-time slots)
  double2 XR[4][2], YR[4][2], BR[8][2];
  double RR[4] = {0.0, 0.0, 0.0, 0.0}, rpart = 0.0;
#pragma unroll
  for (int r = 0; r < 2; ++r) {
#pragma unroll
    for (int s = 0; s < 4; ++s) XR[s][r] = YR[s][r] = BR[s][r] = BR[s + 4][r] = make_double2(0.0, 0.0);
  }
  // one step: sweep 1 on plane g = 4c + kk, sweep 2 on plane g - 1 (if it is a range plane)
  auto load_b = [&](double2* dst, int id, int code, int kk) {  // rows jb, jb+1 (always a valid brick)
    const double* bp = p.b + (int64_t)id * 512 + 64 * (4 * (code & 1) + kk) + 8 * jb + ib;
    dst[0] = ld_hint2(bp, pol_keep);  // the neighbour tiles' b-face copies reuse these lines from L2
    dst[1] = ld_hint2(bp + 8, pol_keep);
  };
  // this chunk's records, read from the record ring once per chunk (the step reads registers):
  // code / own brick id of chunk c, c + 1 and c - 1 (plane g - 1 of step kk = 0), parent of c and c - 1
  int codeC = 0, idC = 0, codeN = 0, idN = 0, codeP = 0, idP = 0, parC = 0, parP = 0;
  auto step = [&](const int c, auto kkc, auto parc, const bool start, const bool sw2) {
    constexpr int kk = decltype(kkc)::value, par = decltype(parc)::value;  // par = c mod 2
    const double* S0 = ST + (c % PN_ST) * STAGE;
    if (kk == 3) wait_upto(c + 1);
    const double* S1 = kk == 3 ? ST + ((c + 1) % PN_ST) * STAGE : S0;  // stage of plane g+1
    constexpr int kp = (kk + 1) & 3;                                   // its plane in that stage
    constexpr int km1 = (kk + 3) & 3, km2 = (kk + 2) & 3;              // ring slots of planes g-1, g-2
    double2(&Xm)[2] = XR[km1];
    double2(&Xc)[2] = XR[kk];
    double2(&Xp)[2] = XR[kp];
    double2(&Ym)[2] = YR[km2];
    double2(&Yc)[2] = YR[km1];
    double2(&Y)[2] = YR[kk];
    constexpr int bc = 4 * par + kk, bm = kk > 0 ? bc - 1 : 4 * (par ^ 1) + 3, bn = 4 * (par ^ 1) + kk;
    double2(&Bm)[2] = BR[bm];  // b of plane g-1
    double2(&Bc)[2] = BR[bc];  // b of plane g
    double& rcm = RR[km1];
    double& rc = RR[kk];
    double& rcp = RR[kp];
    if (start) {  // first step of a run (warm-up plane 7): prime the register windows
      Xm[0] = x0d2(S0 + oO + 64 * (kk - 1)), Xm[1] = x0d2(S0 + oO + 8 + 64 * (kk - 1));
      Xc[0] = x0d2(S0 + oO + 64 * kk), Xc[1] = x0d2(S0 + oO + 8 + 64 * kk);
      rcm = x0d(S0 + oc + 16 * (kk - 1));
      rc = x0d(S0 + oc + 16 * kk);
      // b of this plane and of the next chunk's planes 0-2 (plane 3 follows below)
      load_b(BR[bc], idC, codeC, kk);
#pragma unroll
      for (int k2 = 0; k2 < 3; ++k2) load_b(BR[4 * (par ^ 1) + k2], idN, codeN, k2);
    }
    // b of plane g+4 (the next chunk's plane kk; harmless where that plane is not swept)
    load_b(BR[bn], idN, codeN, kk);
    const int kz1 = 4 * (codeC & 1) + kk;  // in-brick plane of g (red-black colour)

    // ---------------- sweep 1, own cells, plane g ----------------
    Xp[0] = x0d2(S1 + oO + 64 * kp);
    Xp[1] = x0d2(S1 + oO + 8 + 64 * kp);
    {
      const double2 xs = x0d2(S0 + oS + sS * kk), xn = x0d2(S0 + oN + sN * kk);
      // tile-edge x0 (inner lanes read the W edge lane's words: broadcasts, no extra wavefronts)
      const double e0 = x0d(S0 + oEd + 16 * kk), e1 = x0d(S0 + oEd + 2 + 16 * kk);
      const double wl0 = __shfl_up_sync(FULL, Xc[0].y, 1), er0 = __shfl_down_sync(FULL, Xc[0].x, 1);
      const double wl1 = __shfl_up_sync(FULL, Xc[1].y, 1), er1 = __shfl_down_sync(FULL, Xc[1].x, 1);
      const double W0 = edW ? e0 : wl0, E0 = edE ? e0 : er0, W1 = edW ? e1 : wl1, E1 = edE ? e1 : er1;
      const double2 bb0 = Bc[0], bb1 = Bc[1];
      const double a00 = stencil_a(Xc[0].x, W0, Xc[0].y, xs.x, Xc[1].x, Xm[0].x, Xp[0].x, alpha, beta);
      const double a10 = stencil_a(Xc[0].y, Xc[0].x, E0, xs.y, Xc[1].y, Xm[0].y, Xp[0].y, alpha, beta);
      const double a01 = stencil_a(Xc[1].x, W1, Xc[1].y, Xc[0].x, xn.x, Xm[1].x, Xp[1].x, alpha, beta);
      const double a11 = stencil_a(Xc[1].y, Xc[1].x, E1, Xc[0].y, xn.y, Xm[1].y, Xp[1].y, alpha, beta);
      Y[0].x = keep_cell(col1, ib, jb, kz1) ? Xc[0].x : DADD(Xc[0].x, DMUL(gamma, DSUB(a00, bb0.x)));
      Y[0].y = keep_cell(col1, ib + 1, jb, kz1) ? Xc[0].y : DADD(Xc[0].y, DMUL(gamma, DSUB(a10, bb0.y)));
      Y[1].x = keep_cell(col1, ib, jb + 1, kz1) ? Xc[1].x : DADD(Xc[1].x, DMUL(gamma, DSUB(a01, bb1.x)));
      Y[1].y = keep_cell(col1, ib + 1, jb + 1, kz1) ? Xc[1].y : DADD(Xc[1].y, DMUL(gamma, DSUB(a11, bb1.y)));
      double* P = XP + (kk & 1) * PUB;  // parity of plane g = 4c + kk
      *reinterpret_cast<double2*>(P + pO) = Y[0];
      *reinterpret_cast<double2*>(P + pO + 16) = Y[1];
    }
    // ---------------- sweep 1, ring cell, plane g ----------------
    {
      rcp = x0d(S1 + oc + 16 * kp);
      const double o = x0d(S0 + oo + 16 * kk), own = x0d(S0 + oown + 64 * kk);
      const double lo = x0d(S0 + olo + slo * kk), hi = x0d(S0 + ohi + shi * kk), bv = S0[ob + sb * kk];
      // ((o + own) + (lo + hi)) + (b + t): the canonical ((w+e)+(s+n))+(b+t) up to the order of
      // the operands of single additions (IEEE addition is commutative, so bit for bit equal)
      const double sum = DADD(DADD(DADD(o, own), DADD(lo, hi)), DADD(rcm, rcp));
      const double a = DADD(DMUL(alpha, rc), DMUL(beta, sum));
      const double y = keep_cell(col1, rci, rcj, kz1) ? rc : DADD(rc, DMUL(gamma, DSUB(a, bv)));
      XP[oout + rstr * (kk & 1)] = y;
    }
    // ---------------- sweep 2, own cells, plane g-1 ----------------
    // computed on every step (one basic block with sweep 1 and the ring: the scheduler interleaves
    // the three dependency chains); only the stores depend on sw2
    {
      constexpr int par = (kk + 1) & 1;  // parity of plane g - 1
      const double* P = XP + par * PUB;
      const double2 ys = lds_d2(P + pO - 16), yn = lds_d2(XP + pN + sPN * par);
      const double2 ed = lds_d2(RWE + RWE_PAR * par + oRwe);
      const double wl0 = __shfl_up_sync(FULL, Yc[0].y, 1), er0 = __shfl_down_sync(FULL, Yc[0].x, 1);
      const double wl1 = __shfl_up_sync(FULL, Yc[1].y, 1), er1 = __shfl_down_sync(FULL, Yc[1].x, 1);
      const double W0 = edW ? ed.x : wl0, E0 = edE ? ed.x : er0, W1 = edW ? ed.y : wl1, E1 = edE ? ed.y : er1;
      constexpr int km = (kk + 3) & 3;  // plane g-1 within its chunk
      const double2 bb0 = Bm[0], bb1 = Bm[1];
      const int code2 = kk > 0 ? codeC : codeP, id2 = kk > 0 ? idC : idP;
      const int kz2 = 4 * (code2 & 1) + km;
      const double a00 = stencil_a(Yc[0].x, W0, Yc[0].y, ys.x, Yc[1].x, Ym[0].x, Y[0].x, alpha, beta);
      const double a10 = stencil_a(Yc[0].y, Yc[0].x, E0, ys.y, Yc[1].y, Ym[0].y, Y[0].y, alpha, beta);
      const double a01 = stencil_a(Yc[1].x, W1, Yc[1].y, Yc[0].x, yn.x, Ym[1].x, Y[1].x, alpha, beta);
      const double a11 = stencil_a(Yc[1].y, Yc[1].x, E1, Yc[0].y, yn.y, Ym[1].y, Y[1].y, alpha, beta);
      double2 z0, z1, r0, r1;
      z0.x = keep_cell(col2, ib, jb, kz2) ? Yc[0].x : DADD(Yc[0].x, DMUL(gamma2, DSUB(a00, bb0.x)));
      z0.y = keep_cell(col2, ib + 1, jb, kz2) ? Yc[0].y : DADD(Yc[0].y, DMUL(gamma2, DSUB(a10, bb0.y)));
      z1.x = keep_cell(col2, ib, jb + 1, kz2) ? Yc[1].x : DADD(Yc[1].x, DMUL(gamma2, DSUB(a01, bb1.x)));
      z1.y = keep_cell(col2, ib + 1, jb + 1, kz2) ? Yc[1].y : DADD(Yc[1].y, DMUL(gamma2, DSUB(a11, bb1.y)));
      r0.x = DSUB(bb0.x, a00), r0.y = DSUB(bb0.y, a10), r1.x = DSUB(bb1.x, a01), r1.y = DSUB(bb1.y, a11);
      const int64_t go = (int64_t)id2 * 512 + 64 * kz2 + 8 * jb + ib;
      if (sw2) {
        st_hint2(p.xo + go, z0, pol_stream);  // never re-read by this pass
        st_hint2(p.xo + go + 8, z1, pol_stream);
      }
      if (WRITE_R && sw2) {
        st_hint2(p.r + go, r0, pol_stream);
        st_hint2(p.r + go + 8, r1, pol_stream);
      }
      if (RESTRICT) {
        // this lane's 2x2 footprint x 2 planes is one coarse cell: canonical order
        // ((r000+r100)+(r010+r110)) + ((r001+r101)+(r011+r111))
        const double s = DADD(DADD(r0.x, r0.y), DADD(r1.x, r1.y));
        if ((km & 1) == 0) {
          rpart = s;
        } else if (sw2) {
          const int pr = kk > 0 ? parC : parP;
          const int K = 4 * ((pr >> 2) & 1) + (kz2 >> 1);
          p.bc[(int64_t)(pr >> 3) * 512 + pc + 8 * (4 * w + jp) + 64 * K] = DMUL(0.125, DADD(rpart, s));
        }
      }
    }
    __syncthreads();  // x1 of plane g published; stage c (and c+1) reads of this step done
  };

  __syncthreads();  // records 0, 1
  for (int c = 0; c < cnt; ++c) {
    // chunk c (and with it record c+1) before issuing chunk c+1 into the stage chunk c-1 used
    if (c > 0) wait_upto(c);
    while (issued < cnt && issued <= c + PN_ST - 1) issue();
    codeP = codeC, idP = idC, parP = parC;
    codeC = mr(c, 0), idC = mr(c, 1 + q);
    codeN = mr(c + 1, 0), idN = mr(c + 1, 1 + q);  // record c+1 came with chunk c
    if (RESTRICT) parC = mr(c, 17);
    const int type = (codeC >> 1) & 3, typeP = c > 0 ? (codeP >> 1) & 3 : WARM;
    using I0 = std::integral_constant<int, 0>;
    using I1 = std::integral_constant<int, 1>;
    using I2 = std::integral_constant<int, 2>;
    using I3 = std::integral_constant<int, 3>;
    using P0 = std::integral_constant<int, 0>;  // chunk parity: warm-up and half 1 even,
    using P1 = std::integral_constant<int, 1>;  // half 0 and cool-down odd
    if (type == WARM) {
      step(c, I3{}, P0{}, true, false);
    } else if (type == RANGE && (codeC & 1) == 0) {
      step(c, I0{}, P1{}, false, typeP == RANGE);
      step(c, I1{}, P1{}, false, true);
      step(c, I2{}, P1{}, false, true);
      step(c, I3{}, P1{}, false, true);
    } else if (type == RANGE) {
      step(c, I0{}, P0{}, false, true);
      step(c, I1{}, P0{}, false, true);
      step(c, I2{}, P0{}, false, true);
      step(c, I3{}, P0{}, false, true);
    } else {  // COOL: plane 0 of the layer above (sweep 1), the run's last plane (sweep 2)
      static_assert(COOL == 2, "chunk type codes (layout.cpp pencil_table)");
      step(c, I0{}, P1{}, false, true);
    }
  }
  if (pa.trace) {
    __syncthreads();
    if (threadIdx.x == 0) {
      unsigned long long t1;
      asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t1));
      pa.trace[2 * blockIdx.x + 1] = t1;
    }
  }
  pdl_trigger();
#undef pol_keep
#undef pol_stream
}

bool pencil_supports(unsigned flags) {
  const unsigned fl = flags & (SW_WRITE_R | SW_RESTRICT | SW_INTERP);
  return fl == 0 || fl == SW_WRITE_R || fl == SW_RESTRICT;
}

cudaError_t encode_pencil_maps(const double* x, const double* b, int64_t n_alloc, PairMaps* out) {
  const unsigned we[3] = {2, 8, 4}, sn2[3] = {8, 2, 4}, cor[3] = {2, 1, 4}, sn1[3] = {8, 1, 4};
  cudaError_t e;
  if ((e = encode_box_map(x, n_alloc, we, &out->xwe)) != cudaSuccess) return e;
  if ((e = encode_box_map(x, n_alloc, sn2, &out->xsn)) != cudaSuccess) return e;
  if ((e = encode_box_map(x, n_alloc, cor, &out->xcor)) != cudaSuccess) return e;
  if ((e = encode_box_map(b, n_alloc, we, &out->bwe)) != cudaSuccess) return e;
  return encode_box_map(b, n_alloc, sn1, &out->bsn);
}

// every supported flag combination: {plain, +r, +restriction} x {colour} x {x0 == 0 in the first sweep}
#define PENCIL_FLAG_LIST(X)                                                                              \
  X(0) X(SW_WRITE_R) X(SW_RESTRICT) X(SW_COLOUR) X(SW_WRITE_R | SW_COLOUR) X(SW_RESTRICT | SW_COLOUR)   \
  X(SW_ZERO_X) X(SW_ZERO_X | SW_WRITE_R) X(SW_ZERO_X | SW_RESTRICT) X(SW_ZERO_X | SW_COLOUR)             \
  X(SW_ZERO_X | SW_WRITE_R | SW_COLOUR) X(SW_ZERO_X | SW_RESTRICT | SW_COLOUR)                          \
  X(SW_PEER) X(SW_PEER | SW_WRITE_R) X(SW_PEER | SW_RESTRICT)                                             \
  X(SW_PEER | SW_COLOUR) X(SW_PEER | SW_WRITE_R | SW_COLOUR) X(SW_PEER | SW_RESTRICT | SW_COLOUR)

// MG_PEN_TRACE=1 (measurement runs without graph capture only): every pencil pass records each CTA's
// (start, end) globaltimer and prints the spread of the CTAs' end times -- the pass's tail
static cudaError_t trace_report(const PairArgs& pa, cudaStream_t s) {
  cudaError_t e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) return e;
  std::vector<unsigned long long> h((size_t)pa.nctas * 2);
  e = cudaMemcpy(h.data(), pa.trace, h.size() * 8, cudaMemcpyDeviceToHost);
  if (e != cudaSuccess) return e;
  unsigned long long s0 = ~0ull, s1 = 0, e0 = ~0ull, e1 = 0;
  std::vector<double> ends;
  for (int64_t g = 0; g < pa.nctas; ++g) {
    s0 = std::min(s0, h[2 * g]), s1 = std::max(s1, h[2 * g]);
    e0 = std::min(e0, h[2 * g + 1]), e1 = std::max(e1, h[2 * g + 1]);
  }
  for (int64_t g = 0; g < pa.nctas; ++g) ends.push_back((double)(h[2 * g + 1] - s0) / 1e3);
  std::sort(ends.begin(), ends.end());
  auto pct = [&](double q) { return ends[(size_t)std::min<double>(ends.size() - 1, q * ends.size())]; };
  fprintf(stderr,
          "MG_PEN_TRACE ctas=%lld start spread %.1f us; end: first %.1f, p10 %.1f, p50 %.1f, p90 %.1f, last %.1f us\n",
          (long long)pa.nctas, (s1 - s0) / 1e3, (e0 - s0) / 1e3, pct(0.1), pct(0.5), pct(0.9), (e1 - s0) / 1e3);
  // per CTA: end time vs chunk count and SM (is the tail static imbalance or run-time variation?)
  static const bool dump = getenv("MG_PEN_TRACE_DUMP") != nullptr;
  std::vector<unsigned long long> info((size_t)pa.nctas);
  e = cudaMemcpy(info.data(), pa.trace + 2 * 65536, info.size() * 8, cudaMemcpyDeviceToHost);
  if (e != cudaSuccess) return e;
  std::vector<double> sm_end(256, 0.0);
  std::vector<int> sm_n(256, 0);
  double c_lo = 1e30, c_hi = 0;
  for (int64_t g = 0; g < pa.nctas; ++g) {
    const unsigned sm = (unsigned)(info[g] & 0xffffffffu), cnt = (unsigned)(info[g] >> 32);
    const double end = (double)(h[2 * g + 1] - s0) / 1e3;
    if (sm < 256) sm_end[sm] = std::max(sm_end[sm], end), sm_n[sm]++;
    c_lo = std::min(c_lo, (double)cnt), c_hi = std::max(c_hi, (double)cnt);
    if (dump) fprintf(stderr, "  cta %lld sm %u chunks %u end %.1f\n", (long long)g, sm, cnt, end);
  }
  double mn = 1e30, mx = 0;
  for (int q = 0; q < 256; ++q)
    if (sm_n[q]) mn = std::min(mn, sm_end[q]), mx = std::max(mx, sm_end[q]);
  fprintf(stderr, "MG_PEN_TRACE   chunks per CTA %.0f..%.0f; per-SM last end %.1f..%.1f us\n", c_lo, c_hi, mn, mx);
  return cudaSuccess;
}

cudaError_t launch_sweep2p(const SweepArgs& a, const PairArgs& pa_in, const PairMaps& pm, unsigned flags,
                           cudaStream_t s, bool early) {
  if (pa_in.nctas <= 0) return cudaSuccess;
  static const bool trace = getenv("MG_PEN_TRACE") != nullptr;
  static unsigned long long* tbuf = nullptr;
  PairArgs pa = pa_in;
  if (trace) {
    if (!tbuf && cudaMalloc(&tbuf, 3 * 8 * 65536) != cudaSuccess) return cudaErrorMemoryAllocation;
    pa.trace = tbuf;
  }
  const unsigned g = (unsigned)pa.nctas;
  const size_t sm = SMEM_BYTES;
  const unsigned col = (a.colour >= 0 || a.colour2 >= 0) ? SW_COLOUR : 0u;
  switch ((flags & (SW_WRITE_R | SW_RESTRICT | SW_INTERP | SW_ZERO_X | SW_PEER)) | col) {
#define PENCIL_CASE(F)                                                      \
  case (F):                                                                 \
    launch_ex(early && g_launch_pdl, sweep2p_kernel<(F)>, g, PN_THREADS, sm, s, a, pa, pm); \
    break;
    PENCIL_FLAG_LIST(PENCIL_CASE)
#undef PENCIL_CASE
    default:
      return cudaErrorInvalidValue;
  }
  if (trace) return trace_report(pa, s);
  return cudaGetLastError();
}

cudaError_t pencil_kernels_init() {
  cudaError_t e = cudaSuccess;
#define PENCIL_ATTR(F)                                                                                      \
  if ((e = cudaFuncSetAttribute(sweep2p_kernel<(F)>, cudaFuncAttributeMaxDynamicSharedMemorySize,          \
                                (int)SMEM_BYTES)) != cudaSuccess)                                           \
    return e;                                                                                               \
  if ((e = cudaFuncSetAttribute(sweep2p_kernel<(F)>, cudaFuncAttributePreferredSharedMemoryCarveout, 100)) != \
      cudaSuccess)                                                                                          \
    return e;
  PENCIL_FLAG_LIST(PENCIL_ATTR)
#undef PENCIL_ATTR
  return e;
}

}  // namespace mgb
