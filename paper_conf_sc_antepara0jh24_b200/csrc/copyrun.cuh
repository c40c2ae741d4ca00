// copyrun.cuh -- the body of the ghost-exchange copy kernels (local: kernels.cu copy_runs_kernel;
// between processes: peer.cu peer_copy_kernel).  A CopyRun (kernels.h) is either a contiguous run of
// n doubles (box == 0: whole bricks, the paper's packing-free exchange) or the same run of
// bricks of which only a sub-box of cells per brick is copied (box != 0: the ghost cells within the
// exchange depth of the owned region, DESIGN.md §9 "depth-limited exchange").
#pragma once
#include <cstdint>

#include "kernels.h"

namespace mgb {

// box = lo_x | hi_x << 4 | lo_y << 8 | hi_y << 12 | lo_z << 16 | hi_z << 20 | E << 24 (cells of a brick
// [lo, hi) per axis, cell index i + E (j + E k))
__host__ __device__ inline int32_t copy_box(int lx, int hx, int ly, int hy, int lz, int hz, int E) {
  return lx | hx << 4 | ly << 8 | hy << 12 | lz << 16 | hz << 20 | E << 24;
}

template <bool REMOTE>
__device__ __forceinline__ void copy_run_body(const CopyRun& r, int64_t i0, int64_t step) {
  if (r.box == 0) {
    const double2* src = reinterpret_cast<const double2*>(r.src);
    double2* dst = reinterpret_cast<double2*>(r.dst);
    const int64_t n2 = r.n / 2;
    for (int64_t i = i0; i < n2; i += step) dst[i] = REMOTE ? src[i] : __ldg(src + i);
    return;
  }
  const int lx = r.box & 15, nx = ((r.box >> 4) & 15) - lx;
  const int ly = (r.box >> 8) & 15, ny = ((r.box >> 12) & 15) - ly;
  const int lz = (r.box >> 16) & 15, nz = ((r.box >> 20) & 15) - lz;
  const int E = (r.box >> 24) & 15, BV = E * E * E;
  // 32-bit index arithmetic (a run holds at most a few thousand bricks of <= 512 cells: < 2^31 items);
  // 64-bit division costs an order of magnitude more instructions than the copy itself
  const unsigned nb = (unsigned)(r.n / BV), st = (unsigned)step;
  if (((lx | nx) & 1) == 0) {  // 16-byte words
    const unsigned w = (unsigned)nx >> 1, per = w * (unsigned)(ny * nz), total = nb * per;
    for (unsigned i = (unsigned)i0; i < total; i += st) {
      const unsigned b = i / per, q = i - b * per;
      const unsigned ix = q % w, t = q / w, iy = t % (unsigned)ny, iz = t / (unsigned)ny;
      const int64_t off = (int64_t)b * BV + (int)(((lz + iz) * E + (ly + iy)) * E + lx + 2 * ix);
      const double2* s = reinterpret_cast<const double2*>(r.src + off);
      *reinterpret_cast<double2*>(r.dst + off) = REMOTE ? *s : __ldg(s);
    }
  } else {
    const unsigned per = (unsigned)(nx * ny * nz), total = nb * per;
    for (unsigned i = (unsigned)i0; i < total; i += st) {
      const unsigned b = i / per, q = i - b * per;
      const unsigned ix = q % (unsigned)nx, t = q / (unsigned)nx, iy = t % (unsigned)ny, iz = t / (unsigned)ny;
      const int64_t off = (int64_t)b * BV + (int)(((lz + iz) * E + (ly + iy)) * E + lx + ix);
      r.dst[off] = REMOTE ? r.src[off] : __ldg(r.src + off);
    }
  }
}

}  // namespace mgb
