// bottom_cluster.cu -- the bottom solve (Alg 2 steps 10-15: 100 damped-Jacobi sweeps on the
// coarsest level) resident in ONE thread-block cluster, for 9..64 bricks: the
// replicated global coarsest level of a 2x1x1 .. 2x2x2 decomposition (16-64 bricks)
// and a one-rank coarsest level of up to 64 bricks.
//
// The one-CTA resident bottom (resident.cuh) holds <= 8 bricks; this is the same thread mapping
// spread over a cluster of ceil(nbricks / BPC) CTAs of 128 BPC threads, BPC bricks per CTA -- the
// fewest that keep the cluster within 16 CTAs (a sweep is bound by each SM's shared-memory traffic,
// so more SMs per level pay: 64 bricks 0.10 ms on 16 CTAs vs 0.14 ms on 8): brick q
// lives in CTA q / BPC, slot q % BPC (contiguous ids: the x rows of a brick layer stay together).  A thread owns a
// k-column of 4 cells of one brick (x in registers, b in registers), and every neighbour cell --
// in its own brick, in another brick of its CTA or in another CTA's shared memory -- is addressed
// by a generic address -- plain shared memory in the own CTA, the cluster window (mapa) for another
// CTA's -- resolved ONCE before the sweeps.  Per sweep: the 18 neighbour loads of a thread issued
// back to back (local ~30 cycles, remote ~215, overlapped), the
// canonical sweep expression, the new x to the local ping-pong buffer, one cluster barrier
// (arrive.release / wait.acquire) -- instead of a grid-wide step per sweep.
//
// Arithmetic: exactly bottom_resident_body's (stencil_a, x + gamma (a - b), the msign images of a
// non-periodic level), so the result is bit for bit the resident kernel's (tests/test_gpu_parity.py).
#include <cstdlib>

#include "kernels.h"
#include "ptx.cuh"

namespace mgb {

namespace {

constexpr int kBcMaxPerCta = 8;  // bricks per CTA (template BPC: 1, 2, 4 or 8; 128 threads per brick)
constexpr int kBcMaxCtas = 16;   // cluster size (> 8: the non-portable cluster sizes B200 allows)
constexpr size_t bc_smem(int bpc) { return 2 * (size_t)bpc * 512 * sizeof(double); }

__device__ __forceinline__ uint32_t cl_rank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
// the generic address of the same shared-memory location in CTA `rank` of the cluster
__device__ __forceinline__ const double* cl_map_generic(const double* p, uint32_t rank) {
  uint64_t r;
  asm volatile("mapa.u64 %0, %1, %2;" : "=l"(r) : "l"(p), "r"(rank));
  return reinterpret_cast<const double*>(r);
}
// every CTA's writes of this sweep visible to every CTA's reads of the next (and no CTA leaves
// while another may still read its buffers)
__device__ __forceinline__ void cl_barrier() {
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}

}  // namespace

// MS: a non-periodic level (msign != 0).  64 registers per thread (1024 threads): the images'
// signs are a 6-bit mask (x * msign where a bit is set; the resident kernel's x * 1.0 elsewhere is
// the identity), so nothing spills -- every cluster barrier invalidates L1, where spills would live.
template <bool MS, int BPC>
__global__ void __launch_bounds__(128 * BPC, 1)
    bottom_cluster_kernel(const double* __restrict__ x, double* __restrict__ xo, const double* __restrict__ b,
                          const int32_t* __restrict__ adj, int nbricks, int sweeps, int zero_x, Coeffs c,
                          double msign) {
  pdl_begin();
  constexpr int kBcPerCta = BPC, kBcField = BPC * 512;
  extern __shared__ __align__(16) double sm[];  // [2][kBcField]: ping-pong x of this CTA's bricks
  const uint32_t me = cl_rank();
  const int t = threadIdx.x, bl = t >> 7, q = t & 127;
  const int i = q & 7, j = (q >> 3) & 7, k0 = 4 * (q >> 6);
  const int br = (int)me * kBcPerCta + bl;  // global brick id
  const bool act = br < nbricks;
  const int o = bl * 512 + i + 8 * j + 64 * k0;  // my cell k0 in this CTA's buffer
  // generic address (buffer 0) of cell `cell` of brick nq: this CTA's shared memory directly (plain
  // shared loads), another CTA's through its window in the cluster (mapa: distributed shared memory)
  auto at = [&](int nq, int cell) -> const double* {
    const double* p = sm + (nq % kBcPerCta) * 512 + cell;
    const uint32_t r = (uint32_t)(nq / kBcPerCta);
    return r == me ? p : cl_map_generic(p, r);
  };
  const double *aW = sm, *aE = sm, *aS = sm, *aN = sm, *aB = sm, *aT = sm;
  unsigned img = 0;  // bit d: neighbour d is this cell's image across a domain face (MS)
  double xv[4] = {0.0, 0.0, 0.0, 0.0}, bv[4] = {0.0, 0.0, 0.0, 0.0};
  if (act) {
    const int32_t* a = adj + br * 8;
    const int cl = i + 8 * j + 64 * k0;  // my cell k0 in its brick
    const double* own = sm + o;
    aW = i > 0 ? own - 1 : (a[0] < 0 ? own : at(a[0], 7 + 8 * j + 64 * k0));
    aE = i < 7 ? own + 1 : (a[1] < 0 ? own : at(a[1], 0 + 8 * j + 64 * k0));
    aS = j > 0 ? own - 8 : (a[2] < 0 ? own : at(a[2], i + 56 + 64 * k0));
    aN = j < 7 ? own + 8 : (a[3] < 0 ? own : at(a[3], i + 0 + 64 * k0));
    aB = k0 > 0 ? own - 64 : (a[4] < 0 ? own : at(a[4], i + 8 * j + 448));
    aT = k0 < 4 ? own + 256 : (a[5] < 0 ? own + 192 : at(a[5], i + 8 * j));  // (image: cell k = 7)
    if (MS)
      img = (i == 0 && a[0] < 0 ? 1u : 0u) | (i == 7 && a[1] < 0 ? 2u : 0u) | (j == 0 && a[2] < 0 ? 4u : 0u) |
            (j == 7 && a[3] < 0 ? 8u : 0u) | (k0 == 0 && a[4] < 0 ? 16u : 0u) | (k0 == 4 && a[5] < 0 ? 32u : 0u);
    const int64_t g = (int64_t)br * 512 + cl;
#pragma unroll
    for (int kk = 0; kk < 4; ++kk) {
      xv[kk] = zero_x ? 0.0 : __ldcg(x + g + 64 * kk);
      bv[kk] = __ldcg(b + g + 64 * kk);
      sm[o + 64 * kk] = xv[kk];
    }
  }
  auto im = [&](unsigned bit, double v) { return (MS && (img & bit)) ? DMUL(msign, v) : v; };
  cl_barrier();
  for (int s = 0; s < sweeps; ++s) {
    const int rd = (s & 1) ? kBcField : 0;  // buffer holding x of this sweep
    double* wr = sm + ((s & 1) ? 0 : kBcField);          // buffer of the next
    if (act) {
      double w[4], e[4], sv[4], nv[4];
#pragma unroll
      for (int kk = 0; kk < 4; ++kk) {
        w[kk] = aW[rd + 64 * kk];
        e[kk] = aE[rd + 64 * kk];
        sv[kk] = aS[rd + 64 * kk];
        nv[kk] = aN[rd + 64 * kk];
      }
      const double bo = aB[rd], to = aT[rd];
#pragma unroll
      for (int kk = 0; kk < 4; ++kk) {
        // (multiplying by +-1 is exact: reading A22's -x_p / +x_p)
        const double bt = kk > 0 ? xv[kk - 1] : im(16u, bo);
        const double tp = kk < 3 ? xv[kk + 1] : im(32u, to);
        const double av = stencil_a(xv[kk], im(1u, w[kk]), im(2u, e[kk]), im(4u, sv[kk]), im(8u, nv[kk]), bt, tp,
                                    c.alpha, c.beta);
        w[kk] = DADD(xv[kk], DMUL(c.gamma, DSUB(av, bv[kk])));  // (w[kk] dead: holds the new x)
      }
#pragma unroll
      for (int kk = 0; kk < 4; ++kk) {
        xv[kk] = w[kk];
        wr[o + 64 * kk] = w[kk];
      }
    }
    cl_barrier();
  }
  if (act)
#pragma unroll
    for (int kk = 0; kk < 4; ++kk) xo[(int64_t)br * 512 + i + 8 * j + 64 * (k0 + kk)] = xv[kk];
}

// bricks per CTA for a level of nbricks: the fewest that keep the cluster within 16 CTAs, at least
// `min_bpc` (MG_BC_BPC, measurements) -- fewer bricks per CTA spread the shared-memory traffic of a
// sweep (its limiter) over more SMs
static int bc_bpc(int nbricks) {
  static const int forced = getenv("MG_BC_BPC") ? atoi(getenv("MG_BC_BPC")) : 0;
  int bpc = 1;
  while (bpc < kBcMaxPerCta && (nbricks + bpc - 1) / bpc > kBcMaxCtas) bpc *= 2;
  if (forced > bpc && forced <= kBcMaxPerCta) bpc = forced;
  return bpc;
}

template <bool MS, int BPC>
static cudaError_t launch_bc(const double* x, double* xo, const double* b, const int32_t* adj, int nbricks, int sweeps,
                             bool zero_x, Coeffs c, cudaStream_t s, double msign) {
  const unsigned ctas = (unsigned)((nbricks + BPC - 1) / BPC);
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(ctas);
  cfg.blockDim = dim3(128 * BPC);
  cfg.dynamicSmemBytes = bc_smem(BPC);
  cfg.stream = s;
  cudaLaunchAttribute at[2];
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = ctas;
  at[0].val.clusterDim.y = 1;
  at[0].val.clusterDim.z = 1;
  at[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[1].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = g_launch_pdl ? 2 : 1;
  const cudaError_t e = cudaLaunchKernelEx(&cfg, bottom_cluster_kernel<MS, BPC>, x, xo, b, adj, nbricks, sweeps,
                                           zero_x ? 1 : 0, c, msign);
  return e != cudaSuccess ? e : cudaGetLastError();
}

cudaError_t launch_bottom_cluster(const double* x, double* xo, const double* b, const int32_t* adj, int nbricks,
                                  int sweeps, bool zero_x, Coeffs c, cudaStream_t s, double msign) {
  if (nbricks <= 0 || nbricks > kClusterBottomMaxBricks) return cudaErrorInvalidValue;
  const bool ms = msign != 0.0;
  switch (bc_bpc(nbricks)) {
#define BC_CASE(B)                                                                               \
  case B:                                                                                        \
    return ms ? launch_bc<true, B>(x, xo, b, adj, nbricks, sweeps, zero_x, c, s, msign)          \
              : launch_bc<false, B>(x, xo, b, adj, nbricks, sweeps, zero_x, c, s, msign);
    BC_CASE(1)
    BC_CASE(2)
    BC_CASE(4)
    BC_CASE(8)
#undef BC_CASE
  }
  return cudaErrorInvalidValue;
}

bool cluster_bottom_enabled() {
  static const bool off = getenv("MG_NO_CLUSTER_BOTTOM") != nullptr;  // (A/B measurements)
  return !off;
}

bool cluster_bottom_small() {
  static const bool on = getenv("MG_BC_SMALL") != nullptr;  // (A/B: the cluster for <= 8 bricks too)
  return on && cluster_bottom_enabled();
}

cudaError_t bottom_cluster_init() {
  cudaError_t e = cudaSuccess;
#define BC_ATTR(MS, B)                                                                                              \
  if ((e = cudaFuncSetAttribute(bottom_cluster_kernel<MS, B>, cudaFuncAttributeMaxDynamicSharedMemorySize,          \
                                (int)bc_smem(B))) != cudaSuccess)                                                   \
    return e;                                                                                                       \
  if ((e = cudaFuncSetAttribute(bottom_cluster_kernel<MS, B>, cudaFuncAttributeNonPortableClusterSizeAllowed, 1)) != \
      cudaSuccess)                                                                                                  \
    return e;
  BC_ATTR(false, 1) BC_ATTR(false, 2) BC_ATTR(false, 4) BC_ATTR(false, 8)
  BC_ATTR(true, 1) BC_ATTR(true, 2) BC_ATTR(true, 4) BC_ATTR(true, 8)
#undef BC_ATTR
  return e;
}

}  // namespace mgb
