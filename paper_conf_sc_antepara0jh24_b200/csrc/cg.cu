// cg.cu -- CG bottom solver (variant, reading A21; SURVEY §8(f) N4 "other bottom
// solvers").  The paper's bottom is `bottom` damped-Jacobi smooths; this variant runs
// at most `iters` iterations of unpreconditioned conjugate gradients on the consistent system
// A x = b - m (m = b's mean: the periodic operator's null space, reading A12) from x = 0 on the
// coarsest level (no ghosts, <= 8 bricks: one CTA of 1024 threads):
//   m = <b, 1> / N;  r = b - m;  p = r;  rr0 = rr = <r, r>
//   repeat:  q = A p;  d = <p, q>;  if not d < 0: stop;  alpha = rr / d
//            x = x + alpha p;  r = r - alpha q;  rr' = <r, r>;  if rr' <= 1e-24 rr0: stop
//            beta = rr' / rr;  p = r + beta p
// with A the canonical applyOp (reading A8) and <.,.> the fixed-order dot product of reading A21:
// products v_i = a_i b_i over the LEXICOGRAPHIC cell index i = gx + nx (gy + ny gz), summed by the
// stride-doubling pairwise tree (v_i += v_{i+s} for i a multiple of 2s, i + s < n; s = 1, 2, 4, ..).
// Every operation separately rounded, so x is bit for bit the same whatever the thread layout.
//
// Layout: a thread owns a k-column of 4 cells of one brick (x, r, q in registers, p also in shared
// memory for the neighbours' stencils).  A dot product writes the products at their lexicographic
// positions; then thread t owns indices 4t..4t+3: tree levels 1, 2 in registers, 4..64 by warp
// shuffles (lane offsets 1..16), 128..2048 over the 32 warp partials in warp 0 -- the same pairs
// in the same order as the tree, 3 CTA barriers per product.
#include "kernels.h"
#include "ptx.cuh"

namespace mgb {

namespace {

constexpr int kCgThreads = 1024;

// <a, b> of the n products already stored at v[lex]: stride-doubling pairwise tree
__device__ __forceinline__ double tree_sum(double* v, double* part, int n) {
  __syncthreads();  // products in place
  const int t = threadIdx.x, lane = t & 31, w = t >> 5;
  const int i0 = 4 * t;
  double s0 = 0.0;
  if (i0 < n) {
    // levels 1 and 2 inside the thread's 4 indices (partner present only if < n)
    double a0 = v[i0];
    if (i0 + 1 < n) a0 = DADD(a0, v[i0 + 1]);
    if (i0 + 2 < n) {
      double a2 = v[i0 + 2];
      if (i0 + 3 < n) a2 = DADD(a2, v[i0 + 3]);
      a0 = DADD(a0, a2);
    }
    s0 = a0;
  }
  // levels 4 .. 64: index 4t pairs with 4t + s, i.e. lane + s/4, when t is a multiple of s/2
#pragma unroll
  for (int o = 1; o <= 16; o *= 2) {
    const double other = __shfl_down_sync(0xffffffffu, s0, o);
    if ((lane & (2 * o - 1)) == 0 && i0 + 4 * o < n) s0 = DADD(s0, other);
  }
  if (lane == 0) part[w] = s0;  // the partial of index 128 w
  __syncthreads();
  if (w == 0) {  // levels 128 .. 2048 over the warp partials
    double p = part[lane];
    const int i = 128 * lane;
#pragma unroll
    for (int o = 1; o <= 16; o *= 2) {
      const double other = __shfl_down_sync(0xffffffffu, p, o);
      if ((lane & (2 * o - 1)) == 0 && i + 128 * o < n) p = DADD(p, other);
    }
    if (lane == 0) part[32] = p;
  }
  __syncthreads();
  return part[32];
}

}  // namespace

__global__ void __launch_bounds__(kCgThreads, 1)
    bottom_cg_kernel(double* __restrict__ xo, const double* __restrict__ b, const int32_t* __restrict__ adj,
                     const int32_t* __restrict__ coord, int nbricks, int nx, int ny, int iters, Coeffs c) {
  pdl_begin();
  extern __shared__ __align__(16) double sm[];
  const int n = nbricks * 512;
  double* ps = sm;          // p (the neighbours' stencils)
  double* v = sm + n;       // products at lexicographic positions
  double* part = v + n;     // 33 warp partials / result
  const int t = threadIdx.x, br = t >> 7, q = t & 127;
  const int i = q & 7, j = (q >> 3) & 7, k0 = 4 * (q >> 6);
  const bool act = br < nbricks;
  const int o = br * 512 + i + 8 * j + 64 * k0;
  int oW = 0, oE = 0, oS = 0, oN = 0, oB = 0, oT = 0, lex0 = 0, lexk = 0;
  double xv[4] = {0.0, 0.0, 0.0, 0.0}, rv[4] = {0.0, 0.0, 0.0, 0.0}, pv[4] = {0.0, 0.0, 0.0, 0.0};
  if (act) {
    const int32_t* a = adj + br * 8;
    oW = i > 0 ? o - 1 : a[0] * 512 + 7 + 8 * j + 64 * k0;
    oE = i < 7 ? o + 1 : a[1] * 512 + 0 + 8 * j + 64 * k0;
    oS = j > 0 ? o - 8 : a[2] * 512 + i + 56 + 64 * k0;
    oN = j < 7 ? o + 8 : a[3] * 512 + i + 0 + 64 * k0;
    oB = k0 > 0 ? o - 64 : a[4] * 512 + i + 8 * j + 448;
    oT = k0 < 4 ? o + 256 : a[5] * 512 + i + 8 * j;
    const int gx = 8 * coord[3 * br] + i, gy = 8 * coord[3 * br + 1] + j, gz = 8 * coord[3 * br + 2] + k0;
    lex0 = gx + nx * (gy + ny * gz);
    lexk = nx * ny;  // one plane up
#pragma unroll
    for (int kk = 0; kk < 4; ++kk) {
      rv[kk] = __ldcg(b + o + 64 * kk);
      v[lex0 + lexk * kk] = DMUL(rv[kk], 1.0);  // <b, 1>
    }
  }
  const double mean = __ddiv_rn(tree_sum(v, part, n), (double)n);
  if (act)
#pragma unroll
    for (int kk = 0; kk < 4; ++kk) {
      rv[kk] = DSUB(rv[kk], mean);  // r = (b - m) - A 0
      pv[kk] = rv[kk];
      ps[o + 64 * kk] = pv[kk];
      v[lex0 + lexk * kk] = DMUL(rv[kk], rv[kk]);
    }
  double rr = tree_sum(v, part, n);  // (its first barrier also publishes p)
  const double rr0 = rr;
  for (int it = 0; it < iters; ++it) {
    double qv[4];
#pragma unroll
    for (int kk = 0; kk < 4; ++kk) {
      if (!act) {
        qv[kk] = 0.0;
        continue;
      }
      const double bt = kk > 0 ? pv[kk - 1] : ps[oB];
      const double tp = kk < 3 ? pv[kk + 1] : ps[oT];
      qv[kk] = stencil_a(pv[kk], ps[oW + 64 * kk], ps[oE + 64 * kk], ps[oS + 64 * kk], ps[oN + 64 * kk], bt, tp,
                         c.alpha, c.beta);
      v[lex0 + lexk * kk] = DMUL(pv[kk], qv[kk]);
    }
    const double d = tree_sum(v, part, n);
    if (!(d < 0.0)) break;  // uniform: every thread read the same value
    const double alpha = __ddiv_rn(rr, d);
    if (act)
#pragma unroll
      for (int kk = 0; kk < 4; ++kk) {
        xv[kk] = DADD(xv[kk], DMUL(alpha, pv[kk]));
        rv[kk] = DSUB(rv[kk], DMUL(alpha, qv[kk]));
        v[lex0 + lexk * kk] = DMUL(rv[kk], rv[kk]);
      }
    const double rr2 = tree_sum(v, part, n);
    if (rr2 <= DMUL(1e-24, rr0)) break;
    const double beta = __ddiv_rn(rr2, rr);
    if (act)
#pragma unroll
      for (int kk = 0; kk < 4; ++kk) {
        pv[kk] = DADD(rv[kk], DMUL(beta, pv[kk]));
        ps[o + 64 * kk] = pv[kk];  // the stencils of the next q read it after tree_sum's barrier
      }
    rr = rr2;
    __syncthreads();  // p published before the next stencils
  }
  if (act)
#pragma unroll
    for (int kk = 0; kk < 4; ++kk) xo[o + 64 * kk] = xv[kk];
}

size_t cg_smem_bytes(int nbricks) { return ((size_t)2 * nbricks * 512 + 40) * sizeof(double); }

cudaError_t launch_bottom_cg(double* xo, const double* b, const int32_t* adj, const int32_t* coord, int nbricks,
                             int nx, int ny, int iters, Coeffs c, cudaStream_t s) {
  if (nbricks <= 0 || nbricks > kResidentMaxBricks) return cudaErrorInvalidValue;
  launch_k(bottom_cg_kernel, 1, kCgThreads, cg_smem_bytes(nbricks), s, xo, b, adj, coord, nbricks, nx, ny, iters, c);
  return cudaGetLastError();
}

cudaError_t cg_kernels_init() {
  return cudaFuncSetAttribute(bottom_cg_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                              (int)cg_smem_bytes(kResidentMaxBricks));
}

}  // namespace mgb
