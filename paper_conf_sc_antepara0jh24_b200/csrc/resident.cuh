// resident.cuh -- the resident bottom solve's body, shared by the standalone
// bottom kernel (kernels.cu) and the grid-resident coarse solve (coarse_grid.cu): all bricks of
// the coarsest level (no ghosts, <= kResidentMaxBricks) in one CTA, `sweeps` Jacobi sweeps with a
// CTA barrier between them.  One CTA of >= 128 * nbricks threads; sm: 2 * nbricks * 512 doubles.
#pragma once

#include "kernels.h"
#include "ptx.cuh"

namespace mgb {

// msign != 0: a negative adjacency entry marks a domain face (non-periodic bc, reading A22) whose
// ghost is this brick's own reflection: the neighbour of a face cell is the cell itself times msign
// (-1 Dirichlet, +1 Neumann); msign == 0: every entry is a brick (periodic, the paper).
__device__ __forceinline__ void bottom_resident_body(const double* x, double* xo, const double* b, const int32_t* adj, int nbricks,
                                     int sweeps, int zero_x, Coeffs c, double* sm, double msign = 0.0) {
  // A thread owns a k-column of 4 cells (i, j, k0..k0+3) of one brick: its x lives in registers,
  // the in-plane neighbours come from the shared copy of the previous sweep (ping-pong), the two
  // k-halos too; every neighbour offset is resolved through the adjacency table once, up front.
  const int n = nbricks * 512;
  double* xa = sm;
  double* xb = sm + n;
  const int t = threadIdx.x, br = t >> 7, q = t & 127;
  const int i = q & 7, j = (q >> 3) & 7, k0 = 4 * (q >> 6);
  const bool act = br < nbricks;
  const int o = br * 512 + i + 8 * j + 64 * k0;  // my cell k0
  int oW = 0, oE = 0, oS = 0, oN = 0, oB = 0, oT = 0;
  double sW = 1.0, sE = 1.0, sS = 1.0, sN = 1.0, sB = 1.0, sT = 1.0;  // boundary images (msign != 0)
  double xv[4] = {0.0, 0.0, 0.0, 0.0}, bv[4] = {0.0, 0.0, 0.0, 0.0};
  if (act) {
    const int32_t* a = adj + br * 8;
    oW = i > 0 ? o - 1 : a[0] * 512 + 7 + 8 * j + 64 * k0;
    oE = i < 7 ? o + 1 : a[1] * 512 + 0 + 8 * j + 64 * k0;
    oS = j > 0 ? o - 8 : a[2] * 512 + i + 56 + 64 * k0;
    oN = j < 7 ? o + 8 : a[3] * 512 + i + 0 + 64 * k0;
    oB = k0 > 0 ? o - 64 : a[4] * 512 + i + 8 * j + 448;
    oT = k0 < 4 ? o + 256 : a[5] * 512 + i + 8 * j;
    if (msign != 0.0) {  // the face cell's image across a domain face is the cell itself
      if (i == 0 && a[0] < 0) oW = o, sW = msign;
      if (i == 7 && a[1] < 0) oE = o, sE = msign;
      if (j == 0 && a[2] < 0) oS = o, sS = msign;
      if (j == 7 && a[3] < 0) oN = o, sN = msign;
      if (k0 == 0 && a[4] < 0) oB = o, sB = msign;
      if (k0 == 4 && a[5] < 0) oT = o + 192, sT = msign;  // cell k = 7 of this thread's column
    }
#pragma unroll
    for (int kk = 0; kk < 4; ++kk) {
      xv[kk] = zero_x ? 0.0 : __ldcg(x + o + 64 * kk);  // L2: written by other SMs (grid solve)
      bv[kk] = __ldcg(b + o + 64 * kk);
      xa[o + 64 * kk] = xv[kk];
    }
  }
  __syncthreads();
  for (int s = 0; s < sweeps; ++s) {
    if (act) {
      double nx[4];
#pragma unroll
      for (int kk = 0; kk < 4; ++kk) {
        double bt = kk > 0 ? xv[kk - 1] : xa[oB];
        double tp = kk < 3 ? xv[kk + 1] : xa[oT];
        double w = xa[oW + 64 * kk], e = xa[oE + 64 * kk], sv = xa[oS + 64 * kk], nv = xa[oN + 64 * kk];
        if (msign != 0.0) {  // multiplying by +-1 is exact (reading A22's -x_p / +x_p)
          w = DMUL(sW, w), e = DMUL(sE, e), sv = DMUL(sS, sv), nv = DMUL(sN, nv);
          if (kk == 0) bt = DMUL(sB, bt);
          if (kk == 3) tp = DMUL(sT, tp);
        }
        const double av = stencil_a(xv[kk], w, e, sv, nv, bt, tp, c.alpha, c.beta);
        nx[kk] = DADD(xv[kk], DMUL(c.gamma, DSUB(av, bv[kk])));
      }
#pragma unroll
      for (int kk = 0; kk < 4; ++kk) {
        xv[kk] = nx[kk];
        xb[o + 64 * kk] = nx[kk];
      }
    }
    __syncthreads();
    double* tmp = xa;
    xa = xb;
    xb = tmp;
  }
  if (act)
#pragma unroll
    for (int kk = 0; kk < 4; ++kk) xo[o + 64 * kk] = xv[kk];
}

}  // namespace mgb
