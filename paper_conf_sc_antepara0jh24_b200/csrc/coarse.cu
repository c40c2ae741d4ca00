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
  int32_t* adj[kCoarseMaxLevels];     // copies of the level tables: global loads would go through
  int32_t* parent[kCoarseMaxLevels];  // L1, which every cluster barrier invalidates
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
  int32_t* ip = reinterpret_cast<int32_t*>(sm + off);
  for (int l = 0; l < a.nlev; ++l) {
    v.adj[l] = ip;
    ip += a.lv[l].nb * 8;
    v.parent[l] = ip;
    ip += (a.lv[l].nb + 3) & ~3;
  }
}

}  // namespace

size_t coarse_smem_bytes(const CoarseArgs& a) {
  size_t d = 0;
  for (int l = 0; l < a.nlev; ++l) {
    const size_t f = (size_t)((a.lv[l].nb + C - 1) / C) * 512;
    d += f * (l + 1 < a.nlev ? 4 : 3);
  }
  size_t t = 0;  // adjacency + parent tables (int32)
  for (int l = 0; l < a.nlev; ++l) t += (size_t)a.lv[l].nb * 8 + ((a.lv[l].nb + 3) & ~3);
  return d * sizeof(double) + t * sizeof(int32_t);
}

__global__ void __cluster_dims__(kCoarseCtas, 1, 1) __launch_bounds__(kCoarseThreads, 1)
    coarse_cluster_kernel(const __grid_constant__ CoarseArgs a) {
  pdl_begin();
  cg::cluster_group cl = cg::this_cluster();
  const unsigned me = cl.block_rank();
  extern __shared__ __align__(16) double sm[];
  __shared__ Carve v;  // field bases per level (in shared memory: indexed by a run-time level)
  if (threadIdx.x == 0) carve(a, sm, v);
  __syncthreads();
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
  for (int l = 0; l < a.nlev; ++l) {
    for (int e = threadIdx.x; e < a.lv[l].nb * 8; e += T) v.adj[l][e] = a.lv[l].adj[e];
    if (l + 1 < a.nlev)
      for (int e = threadIdx.x; e < a.lv[l].nb; e += T) v.parent[l][e] = a.lv[l].parent[e];
  }
  unsigned curm = 0;  // bit l: which x buffer of level l holds x
  auto cur = [&](int l) { return (int)((curm >> l) & 1u); };
  cl.sync();

  // step of a pre / post sweep: the level's Jacobi step or, for the Chebyshev variant,
  // h^2 / (12 nu) with the host's node nu (same IEEE operations as the host's sweep_gamma)
  auto step = [&](int l, const double* nu, int k) {
    return a.cheb ? __ddiv_rn(DMUL(a.lv[l].h, a.lv[l].h), DMUL(12.0, nu[k])) : a.lv[l].c.gamma;
  };
  // one sweep of level l (ping-pong) with step g, optionally with r = b - Ax.  A thread takes up
  // to kPer cells per batch and issues all their neighbour loads (local LDS or DSMEM) before any
  // arithmetic, so the remote-load latencies overlap instead of adding up per cell.
  constexpr int kPer = 4;
  auto sweep = [&](int l, bool write_r, double g) {
    const CoarseLevel& L = a.lv[l];
    double* xs = v.x[l][cur(l)];
    double* __restrict__ xd = v.x[l][cur(l) ^ 1];
    const double* __restrict__ bl = v.b[l];
    double* __restrict__ rl = v.r[l];
    const int ncell = v.slots[l] * 512;
    for (int e0 = threadIdx.x; e0 < ncell; e0 += T * kPer) {
      double nv[kPer][7];
      bool ok[kPer];
#pragma unroll
      for (int u = 0; u < kPer; ++u) {
        const int e = e0 + u * T;
        const int q = (e >> 9) * C + (int)me;
        ok[u] = e < ncell && q < L.nb;
        if (ok[u]) {
          const int c = e & 511, i = c & 7, j = (c >> 3) & 7, k = c >> 6;
          const int32_t* ad = v.adj[l] + q * 8;
          nv[u][0] = xs[e];
          nv[u][1] = i > 0 ? xs[e - 1] : *at(xs, ad[0], c + 7);
          nv[u][2] = i < 7 ? xs[e + 1] : *at(xs, ad[1], c - 7);
          nv[u][3] = j > 0 ? xs[e - 8] : *at(xs, ad[2], c + 56);
          nv[u][4] = j < 7 ? xs[e + 8] : *at(xs, ad[3], c - 56);
          nv[u][5] = k > 0 ? xs[e - 64] : *at(xs, ad[4], c + 448);
          nv[u][6] = k < 7 ? xs[e + 64] : *at(xs, ad[5], c - 448);
        }
      }
#pragma unroll
      for (int u = 0; u < kPer; ++u) {
        if (!ok[u]) continue;
        const int e = e0 + u * T;
        const double av = stencil_a(nv[u][0], nv[u][1], nv[u][2], nv[u][3], nv[u][4], nv[u][5], nv[u][6],
                                    L.c.alpha, L.c.beta);
        const double bb = bl[e];
        xd[e] = DADD(nv[u][0], DMUL(g, DSUB(av, bb)));
        if (write_r) rl[e] = DSUB(bb, av);
      }
    }
    curm ^= 1u << l;
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
      const int pr = v.parent[l][q], oct = pr & 7;
      const int ox = oct & 1, oy = (oct >> 1) & 1, oz = oct >> 2;
      *at(v.b[l + 1], pr >> 3, (4 * ox + I) + 8 * (4 * oy + J) + 64 * (4 * oz + K)) = val;
    }
    cl.sync();
  };
  // x of level l += x of level l+1 at the parent cell
  auto interp_from = [&](int l) {
    const CoarseLevel& L = a.lv[l];
    double* xf = v.x[l][cur(l)];
    double* xcb = v.x[l + 1][cur(l + 1)];
    for (int e = threadIdx.x; e < v.slots[l] * 512; e += T) {
      const int q = (e >> 9) * C + (int)me;
      if (q >= L.nb) continue;
      const int c = e & 511, i = c & 7, j = (c >> 3) & 7, k = c >> 6;
      const int pr = v.parent[l][q], oct = pr & 7;
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
    if (q < a.lv[0].nb) a.x0[(int64_t)q * 512 + (e & 511)] = v.x[0][cur(0)][e];
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
