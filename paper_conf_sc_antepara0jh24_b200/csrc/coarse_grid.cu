// coarse_grid.cu -- grid-resident coarse-level solver (second design).
//
// Below a few thousand bricks per level every operator of Alg 2 is latency-bound: a
// launch plus its ramp costs more than the work (tools/model_fit.py: ~6-7 us per op for levels
// <= 64^3 at 512^3 per GPU, ~60 ops).  This kernel runs the lower part of the V-cycle -- levels
// l0 .. L-1 (ghost-free): pre-sweeps with the restriction fused into the last one, initZero
// (folded into the first sweep), the bottom, interpolation and the post-sweeps -- as ONE launch of
// one 1024-thread CTA per SM.  Fields stay where the per-level kernels keep them (the level
// buffers in HBM, L2-resident at these sizes); dependent steps are separated by a grid barrier
// (an arrive counter and a generation word, ~1-2 us) instead of a kernel boundary.  Unlike the
// 8-CTA cluster design (coarse.cu), every SM works on every level.  The bottom (<= 8 bricks) runs
// inside CTA 0 with x in registers and the ping-pong in shared memory (the resident bottom of
// kernels.cu) while the other CTAs wait at the barrier.
//
// Arithmetic: the canonical expressions of kernels.cu (reading A8) in the same order, so the
// result is bit for bit that of the per-level kernels (tests/test_gpu_parity.py).
// Field loads bypass L1 (ld.global.cg): another SM wrote them before the last barrier.
#include "kernels.h"
#include "ptx.cuh"
#include "resident.cuh"

namespace mgb {

namespace {

__device__ __forceinline__ double ldcg(const double* p) { return __ldcg(p); }

__device__ __forceinline__ unsigned ld_acquire_u32(const unsigned* p) {
  unsigned v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}

// Grid barrier: bar[0] = arrive count (0 between barriers), bar[1] = generation.  Thread 0 of
// each CTA arrives after a CTA barrier and a gpu-scope fence (so the CTA's writes are visible);
// the last arriver resets the count and bumps the generation.  Bounded spin: a barrier that never
// completes (CTAs not co-resident) traps instead of hanging the device.  Measured ~4 us per
// barrier with one CTA per SM -- about what a graph-replayed launch costs; a
// flag-per-CTA variant polled by one warp (no atomics) measured slower.
__device__ __forceinline__ void grid_sync(unsigned* bar, unsigned& gen) {
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    const unsigned arrived = atomicAdd(&bar[0], 1u);
    if (arrived == gridDim.x - 1) {
      atomicExch(&bar[0], 0u);
      __threadfence();
      atomicExch(&bar[1], gen + 1);
    } else {
      long long spins = 0;
      while (ld_acquire_u32(&bar[1]) == gen) {
        if (++spins > (1ll << 28)) __trap();
      }
    }
    __threadfence();
  }
  ++gen;
  __syncthreads();
}

}  // namespace

__global__ void __launch_bounds__(kGridCoarseThreads, 1) coarse_grid_kernel(const __grid_constant__ GridCoarseArgs a) {
  pdl_wait();
  extern __shared__ __align__(16) double sm[];  // CTA 0: the bottom's ping-pong
  const int64_t G = (int64_t)gridDim.x * blockDim.x;
  const int64_t gt = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  unsigned gen = ld_acquire_u32(&a.bar[1]);  // every CTA reads it before its first arrival
  unsigned curm = 0;                          // bit l: which x buffer of level l holds x (all start at 0)
  auto cur = [&](int l) { return (int)((curm >> l) & 1u); };

  // the canonical stencil of cell c of brick q (neighbours across brick faces via the adjacency)
  auto cell_a = [&](const GridLevel& L, const double* xs, int64_t q, int c, bool zero, double& xc) {
    if (zero) {
      xc = 0.0;
      return stencil_a(0.0, 0.0, 0.0, 0.0, 0.0, 0.0, 0.0, L.c.alpha, L.c.beta);
    }
    const int i = c & 7, j = (c >> 3) & 7, k = c >> 6;
    const int32_t* ad = L.adj + q * 8;
    const double* xb = xs + q * 512;
    xc = ldcg(xb + c);
    const double w = i > 0 ? ldcg(xb + c - 1) : ldcg(xs + (int64_t)__ldg(ad + 0) * 512 + c + 7);
    const double e = i < 7 ? ldcg(xb + c + 1) : ldcg(xs + (int64_t)__ldg(ad + 1) * 512 + c - 7);
    const double s = j > 0 ? ldcg(xb + c - 8) : ldcg(xs + (int64_t)__ldg(ad + 2) * 512 + c + 56);
    const double n = j < 7 ? ldcg(xb + c + 8) : ldcg(xs + (int64_t)__ldg(ad + 3) * 512 + c - 56);
    const double bt = k > 0 ? ldcg(xb + c - 64) : ldcg(xs + (int64_t)__ldg(ad + 4) * 512 + c + 448);
    const double tp = k < 7 ? ldcg(xb + c + 64) : ldcg(xs + (int64_t)__ldg(ad + 5) * 512 + c - 448);
    return stencil_a(xc, w, e, s, n, bt, tp, L.c.alpha, L.c.beta);
  };
  // one Jacobi sweep of level l (ping-pong) with step g; x == 0 when `zero` (folded initZero).
  // A thread takes two cells per round and issues both cells' loads before any arithmetic (the
  // L2 latencies overlap instead of adding up).
  auto sweep = [&](int l, double g, bool zero) {
    const GridLevel& L = a.lv[l];
    const double* xs = L.x[cur(l)];
    double* xd = L.x[cur(l) ^ 1];
    const int64_t n = L.nb * 512;
    for (int64_t e0 = gt; e0 < n; e0 += 2 * G) {
      const int64_t e1 = e0 + G;
      const bool has1 = e1 < n;
      double xc0, xc1 = 0.0, bb1 = 0.0, av1 = 0.0;
      const double bb0 = ldcg(L.b + e0);
      if (has1) bb1 = ldcg(L.b + e1);
      const double av0 = cell_a(L, xs, e0 >> 9, (int)(e0 & 511), zero, xc0);
      if (has1) av1 = cell_a(L, xs, e1 >> 9, (int)(e1 & 511), zero, xc1);
      xd[e0] = DADD(xc0, DMUL(g, DSUB(av0, bb0)));
      if (has1) xd[e1] = DADD(xc1, DMUL(g, DSUB(av1, bb1)));
    }
    curm ^= 1u << l;
    grid_sync(a.bar, gen);
  };
  // the last pre-sweep of level l with the restriction of its residual r = b - Ax into b of
  // level l+1: a thread takes the 2x2x2 fine cells of one coarse cell and adds their r in the
  // canonical order ((r000+r100)+(r010+r110)) + ((r001+r101)+(r011+r111)), times 0.125
  auto sweep_restrict = [&](int l, double g, bool zero) {
    const GridLevel& L = a.lv[l];
    const double* xs = L.x[cur(l)];
    double* xd = L.x[cur(l) ^ 1];
    double* bc = a.lv[l + 1].b;
    for (int64_t e = gt; e < L.nb * 64; e += G) {
      const int64_t q = e >> 6;
      const int o = (int)(e & 63), I = o & 3, J = (o >> 2) & 3, K = o >> 4;
      double rr[8];
#pragma unroll
      for (int d = 0; d < 8; ++d) {
        const int c = (2 * I + (d & 1)) + 8 * (2 * J + ((d >> 1) & 1)) + 64 * (2 * K + (d >> 2));
        double xc;
        const double av = cell_a(L, xs, q, c, zero, xc);
        const double bb = ldcg(L.b + q * 512 + c);
        xd[q * 512 + c] = DADD(xc, DMUL(g, DSUB(av, bb)));
        rr[d] = DSUB(bb, av);
      }
      const double v = DMUL(0.125, DADD(DADD(DADD(rr[0], rr[1]), DADD(rr[2], rr[3])),
                                        DADD(DADD(rr[4], rr[5]), DADD(rr[6], rr[7]))));
      const int pr = __ldg(L.parent + q), oct = pr & 7;
      const int ox = oct & 1, oy = (oct >> 1) & 1, oz = oct >> 2;
      bc[(int64_t)(pr >> 3) * 512 + (4 * ox + I) + 8 * (4 * oy + J) + 64 * (4 * oz + K)] = v;
    }
    curm ^= 1u << l;
    grid_sync(a.bar, gen);
  };
  // x of level l += x of level l+1 at the parent cell (in place)
  auto interp_from = [&](int l) {
    const GridLevel& L = a.lv[l];
    double* xf = L.x[cur(l)];
    const double* xcb = a.lv[l + 1].x[cur(l + 1)];
    for (int64_t e = gt; e < L.nb * 512; e += G) {
      const int64_t q = e >> 9;
      const int c = (int)(e & 511), i = c & 7, j = (c >> 3) & 7, k = c >> 6;
      const int pr = __ldg(L.parent + q), oct = pr & 7;
      const int ox = oct & 1, oy = (oct >> 1) & 1, oz = oct >> 2;
      xf[e] = DADD(ldcg(xf + e),
                   ldcg(xcb + (int64_t)(pr >> 3) * 512 + (4 * ox + (i >> 1)) + 8 * (4 * oy + (j >> 1)) +
                        64 * (4 * oz + (k >> 1))));
    }
    grid_sync(a.bar, gen);
  };
  auto step = [&](int l, const double* nu, int k) {  // pre / post step (Chebyshev: h^2 / (12 nu_k))
    return a.cheb ? __ddiv_rn(DMUL(a.lv[l].h, a.lv[l].h), DMUL(12.0, nu[k])) : a.lv[l].c.gamma;
  };

  const int last = a.nlev - 1;
  for (int l = 0; l < last; ++l) {  // Alg 2 steps 1-8 (every level starts from x = 0)
    for (int s = 0; s + 1 < a.pre; ++s) sweep(l, step(l, a.nu_pre, s), s == 0);
    sweep_restrict(l, step(l, a.nu_pre, a.pre - 1), a.pre == 1);
  }
  if (a.bottom > 0) {  // steps 10-15: damped Jacobi from x = 0
    const GridLevel& L = a.lv[last];
    if (L.nb <= kResidentMaxBricks) {
      if (blockIdx.x == 0)
        bottom_resident_body(L.x[0], L.x[1], L.b, L.adj, (int)L.nb, a.bottom, 1, L.c, sm);
      curm ^= 1u << last;  // the result is in x[1]
      grid_sync(a.bar, gen);
    } else {
      for (int s = 0; s < a.bottom; ++s) sweep(last, L.c.gamma, s == 0);
    }
  } else {  // no bottom sweeps: x = 0 at the bottom level
    const GridLevel& L = a.lv[last];
    for (int64_t e = gt; e < L.nb * 512; e += G) L.x[0][e] = 0.0;
    grid_sync(a.bar, gen);
  }
  for (int l = last - 1; l >= 0; --l) {  // steps 16-23
    interp_from(l);
    for (int s = 0; s < a.post; ++s) sweep(l, step(l, a.nu_post, s), false);
  }
  if (cur(0) != 0) {  // x of level l0 for the level above lives in buffer 0
    const GridLevel& L = a.lv[0];
    for (int64_t e = gt; e < L.nb * 512; e += G) L.x[0][e] = ldcg(L.x[1] + e);
  }
  pdl_trigger();
}

static int g_grid_ctas = 0;

cudaError_t coarse_grid_init() {
  int dev = 0, sms = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  if ((e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev)) != cudaSuccess) return e;
  g_grid_ctas = sms;
  return cudaFuncSetAttribute(coarse_grid_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                              (int)(2 * kResidentMaxBricks * 512 * sizeof(double)));
}

cudaError_t launch_coarse_grid(const GridCoarseArgs& a, cudaStream_t s) {
  if (a.nlev < 1 || a.nlev > kCoarseMaxLevels || !a.bar || g_grid_ctas <= 0 )
    return cudaErrorInvalidValue;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)g_grid_ctas);
  cfg.blockDim = dim3(kGridCoarseThreads);
  cfg.dynamicSmemBytes = 2 * kResidentMaxBricks * 512 * sizeof(double);
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeCooperative;  // all CTAs co-resident (the grid barrier needs it)
  at[0].val.cooperative = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, coarse_grid_kernel, a);
}

}  // namespace mgb
