// coarse.cu -- resident coarse-level solver in one thread-block cluster.
//
// Below ~64 bricks per level every operator of Alg 2 is latency-bound: a launch
// costs more than the work (tools/model_fit.py: alpha ~ 7 us per sweep vs < 1 us of data).
// This kernel runs the whole lower part of the V-cycle -- levels l0 .. L-1: pre-sweeps, the
// restriction fused into the last one, initZero, the 100-sweep bottom, interpolation and the
// post-sweeps -- inside ONE launch of a cluster of kCoarseCtas CTAs that keeps every field of
// those levels in shared memory.  Brick q of a level lives in CTA q % kCoarseCtas, slot
// q / kCoarseCtas; a face neighbour in another CTA is read through distributed shared memory
// (cluster.map_shared_rank); one cluster barrier separates dependent steps.
//
// Arithmetic: the canonical expressions of kernels.cu (reading A8) in the same order --
// sweep x' = x + gamma*(a - b), r = b - a with a = stencil_a(...); restriction pairwise
// i -> j -> k times 0.125; interpolation x_f + x_c; x = 0 for initZero -- so the result is bit
// for bit that of the per-level kernels (tests/test_gpu_parity.py).
#include <cooperative_groups.h>

#include "kernels.h"
#include "ptx.cuh"

namespace cg = cooperative_groups;

namespace mgb {

namespace {

constexpr int C = kCoarseCtas;

struct Carve {
  double* x[kCoarseMaxLevels][2];
  double* b[kCoarseMaxLevels];
  double* r[kCoarseMaxLevels];
  int slots[kCoarseMaxLevels];
};

__device__ __forceinline__ void carve(const CoarseArgs& a, double* sm, Carve& v) {
  size_t off = 0;
  for (int l = 0; l < a.nlev; ++l) {
    const int sl = (a.lv[l].nb + C - 1) / C;
    v.slots[l] = sl;
    const size_t f = (size_t)sl * 512;
    v.x[l][0] = sm + off;
    off += f;
    v.x[l][1] = sm + off;
    off += f;
    v.b[l] = sm + off;
    off += f;
    v.r[l] = sm + off;
    if (l + 1 < a.nlev) off += f;
  }
}

}  // namespace

size_t coarse_smem_bytes(const CoarseArgs& a) {
  size_t d = 0;
  for (int l = 0; l < a.nlev; ++l) {
    const size_t f = (size_t)((a.lv[l].nb + C - 1) / C) * 512;
    d += f * (l + 1 < a.nlev ? 4 : 3);
  }
  return d * sizeof(double);
}

__global__ void __cluster_dims__(kCoarseCtas, 1, 1) __launch_bounds__(kCoarseThreads, 1)
    coarse_cluster_kernel(const __grid_constant__ CoarseArgs a) {
  cg::cluster_group cl = cg::this_cluster();
  const unsigned me = cl.block_rank();
  extern __shared__ __align__(16) double sm[];
  Carve v;
  carve(a, sm, v);
  const int T = blockDim.x;
  // remote (or local) address of cell c of brick q of the field whose local base is p
  auto at = [&](double* base, int q, int c) -> double* {
    double* p = base + (q / C) * 512 + c;
    const unsigned own = (unsigned)(q % C);
    return own == me ? p : cl.map_shared_rank(p, own);
  };

  // initZero of every level (both buffers start from buffer 0), level l0's b from global
  for (int l = 0; l < a.nlev; ++l)
    for (int e = threadIdx.x; e < v.slots[l] * 512; e += T) v.x[l][0][e] = 0.0;
  for (int e = threadIdx.x; e < v.slots[0] * 512; e += T) {
    const int q = (e >> 9) * C + (int)me;
    if (q < a.lv[0].nb) v.b[0][e] = a.b0[(int64_t)q * 512 + (e & 511)];
  }
  int cur[kCoarseMaxLevels];
  for (int l = 0; l < kCoarseMaxLevels; ++l) cur[l] = 0;
  cl.sync();

  // step of a pre / post sweep: the level's Jacobi step or, for the Chebyshev variant,
  // h^2 / (12 nu) with the host's node nu (same IEEE operations as the host's sweep_gamma)
  auto step = [&](int l, const double* nu, int k) {
    return a.cheb ? __ddiv_rn(DMUL(a.lv[l].h, a.lv[l].h), DMUL(12.0, nu[k])) : a.lv[l].c.gamma;
  };
  // one sweep of level l (ping-pong) with step g, optionally with r = b - Ax
  auto sweep = [&](int l, bool write_r, double g) {
    const CoarseLevel& L = a.lv[l];
    double* xs = v.x[l][cur[l]];
    double* xd = v.x[l][cur[l] ^ 1];
    const double* bl = v.b[l];
    double* rl = v.r[l];
    for (int e = threadIdx.x; e < v.slots[l] * 512; e += T) {
      const int q = (e >> 9) * C + (int)me;
      if (q >= L.nb) continue;
      const int c = e & 511, i = c & 7, j = (c >> 3) & 7, k = c >> 6;
      const int32_t* ad = L.adj + (int64_t)q * 8;
      const double xc = xs[e];
      const double w = i > 0 ? xs[e - 1] : *at(xs, __ldg(ad + 0), c + 7);
      const double ee = i < 7 ? xs[e + 1] : *at(xs, __ldg(ad + 1), c - 7);
      const double s = j > 0 ? xs[e - 8] : *at(xs, __ldg(ad + 2), c + 56);
      const double n = j < 7 ? xs[e + 8] : *at(xs, __ldg(ad + 3), c - 56);
      const double bt = k > 0 ? xs[e - 64] : *at(xs, __ldg(ad + 4), c + 448);
      const double tp = k < 7 ? xs[e + 64] : *at(xs, __ldg(ad + 5), c - 448);
      const double av = stencil_a(xc, w, ee, s, n, bt, tp, L.c.alpha, L.c.beta);
      const double bb = bl[e];
      xd[e] = DADD(xc, DMUL(g, DSUB(av, bb)));
      if (write_r) rl[e] = DSUB(bb, av);
    }
    cur[l] ^= 1;
    cl.sync();
  };
  // b of level l+1 = R r of level l (the parent brick may live in another CTA)
  auto restrict_to = [&](int l) {
    const CoarseLevel& L = a.lv[l];
    for (int e = threadIdx.x; e < v.slots[l] * 64; e += T) {
      const int q = (e >> 6) * C + (int)me;
      if (q >= L.nb) continue;
      const int cc = e & 63, I = cc & 3, J = (cc >> 2) & 3, K = cc >> 4;
      const double* r = v.r[l] + (e >> 6) * 512 + 2 * I + 16 * J + 128 * K;
      const double val = DMUL(0.125, DADD(DADD(DADD(r[0], r[1]), DADD(r[8], r[9])),
                                          DADD(DADD(r[64], r[65]), DADD(r[72], r[73]))));
      const int pr = __ldg(L.parent + q), oct = pr & 7;
      const int ox = oct & 1, oy = (oct >> 1) & 1, oz = oct >> 2;
      *at(v.b[l + 1], pr >> 3, (4 * ox + I) + 8 * (4 * oy + J) + 64 * (4 * oz + K)) = val;
    }
    cl.sync();
  };
  // x of level l += x of level l+1 at the parent cell
  auto interp_from = [&](int l) {
    const CoarseLevel& L = a.lv[l];
    double* xf = v.x[l][cur[l]];
    double* xcb = v.x[l + 1][cur[l + 1]];
    for (int e = threadIdx.x; e < v.slots[l] * 512; e += T) {
      const int q = (e >> 9) * C + (int)me;
      if (q >= L.nb) continue;
      const int c = e & 511, i = c & 7, j = (c >> 3) & 7, k = c >> 6;
      const int pr = __ldg(L.parent + q), oct = pr & 7;
      const int ox = oct & 1, oy = (oct >> 1) & 1, oz = oct >> 2;
      xf[e] = DADD(xf[e], *at(xcb, pr >> 3, (4 * ox + (i >> 1)) + 8 * (4 * oy + (j >> 1)) + 64 * (4 * oz + (k >> 1))));
    }
    cl.sync();
  };

  const int last = a.nlev - 1;
  for (int l = 0; l < last; ++l) {  // Alg 2 steps 1-8 on levels l0 .. L-2
    for (int s = 0; s < a.pre; ++s) sweep(l, s == a.pre - 1, step(l, a.nu_pre, s));
    restrict_to(l);
  }
  for (int s = 0; s < a.bottom; ++s) sweep(last, false, a.lv[last].c.gamma);  // steps 10-15 (Jacobi)
  for (int l = last - 1; l >= 0; --l) {                                       // steps 16-23
    interp_from(l);
    for (int s = 0; s < a.post; ++s) sweep(l, false, step(l, a.nu_post, s));
  }
  for (int e = threadIdx.x; e < v.slots[0] * 512; e += T) {  // x of level l0 for the level above
    const int q = (e >> 9) * C + (int)me;
    if (q < a.lv[0].nb) a.x0[(int64_t)q * 512 + (e & 511)] = v.x[0][cur[0]][e];
  }
}

cudaError_t launch_coarse(const CoarseArgs& a, cudaStream_t s) {
  const size_t sm = coarse_smem_bytes(a);
  if (sm > kCoarseMaxSmem || a.nlev < 1 || a.nlev > kCoarseMaxLevels) return cudaErrorInvalidValue;
  coarse_cluster_kernel<<<kCoarseCtas, kCoarseThreads, sm, s>>>(a);
  return cudaGetLastError();
}

cudaError_t coarse_kernels_init() {
  return cudaFuncSetAttribute(coarse_cluster_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kCoarseMaxSmem);
}

}  // namespace mgb
