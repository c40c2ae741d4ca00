// peer.cu -- ghost exchange between processes over peer memory (CUDA IPC over NVLink / NVSwitch),
// device-initiated and flag-synchronised (SURVEY §8(e) "CUDA-IPC P2P", §8(f) N2 "device-initiated
// halo puts with flags").
//
// Every rank maps every other rank's workspace (cudaIpcOpenMemHandle); an exchange is ONE kernel
// that copies the receiver's ghost brick runs straight out of the senders' fields (remote 128-bit
// loads through the peer mapping: the paper's packing-free exchange), with the ordering done
// on the device by flags in each rank's workspace instead of host-side MPI / NCCL calls:
//   1. CTA 0 publishes "ready(e)" to every participant (a system-scope release store into the
//      participant's flag slot for this rank), after a system-scope fence: everything this rank's
//      stream wrote before the exchange (the sweep that produced the surface bricks) is visible.
//   2. Every CTA waits until every participant's "ready(e)" has arrived in its own (local) slots,
//      then copies its share of the runs.
//   3. The last CTA to finish publishes "done(e)" and waits for every participant's "done(e)": no
//      rank can overwrite a field another rank is still reading (with a CA period k > 1 a rank runs k
//      sweeps between exchanges, the second of which rewrites the buffer the neighbours read).
// e is a per-rank epoch counter in device memory, bumped by the last CTA: every rank issues the same
// sequence of exchanges (they are collective), so the epochs advance in lockstep and the kernel can
// be captured once in the V-cycle's CUDA graph and replayed.  A bounded wait (globaltimer) traps
// instead of hanging the device.  The global max of the residual norm (Alg 1) and the
// replicated bottom's gather use the same protocol with every rank as participant.
#include <cuda_runtime.h>

#include <algorithm>

#include "kernels.h"
#include "copyrun.cuh"
#include "ptx.cuh"

namespace mgb {

namespace {

constexpr unsigned long long kPeerTimeoutNs = 20ull * 1000 * 1000 * 1000;  // 20 s, then trap

__device__ __forceinline__ unsigned long long ld_acquire_sys(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_sys(unsigned long long* p, unsigned long long v) {
  asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ unsigned long long globaltimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}

// wait until slot kind (0 ready, 1 done) of every participant holds >= e
__device__ void peer_wait(const PeerSync& s, int kind, unsigned long long e) {
  const unsigned long long t0 = globaltimer();
  for (int i = 0; i < s.npart; ++i) {
    const unsigned long long* f = s.flags + ((size_t)s.part[i] * 2 + kind) * kPeerSlotU64;
    while (ld_acquire_sys(f) < e)
      if (globaltimer() - t0 > kPeerTimeoutNs) __trap();
  }
}

__device__ void peer_signal(const PeerSync& s, int kind, unsigned long long e) {
  __threadfence_system();
  for (int i = 0; i < s.npart; ++i) st_release_sys(s.remote[(size_t)s.part[i] * 2 + kind], e);
}

// the end of a peer kernel: the last CTA publishes done(e), waits for everyone's done(e), bumps the epoch
__device__ void peer_finish(const PeerSync& s, unsigned long long e) {
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    const unsigned nblk = gridDim.x * gridDim.y;
    if (atomicAdd(s.done, 1u) == nblk - 1) {
      peer_signal(s, 1, e);
      peer_wait(s, 1, e);
      *s.epoch = e;
      *s.done = 0;
      __threadfence();
    }
  }
}

// blockIdx.y = run; the x-blocks stride over its 16-byte words (the local copy kernel's grid)
__global__ void __launch_bounds__(256) peer_copy_kernel(const CopyRun* __restrict__ runs, PeerSync s) {
  pdl_wait();  // the sweep that produced this rank's surface bricks has completed
  const unsigned long long e = *(volatile unsigned long long*)s.epoch + 1;
  if (threadIdx.x == 0) {
    if (blockIdx.x == 0 && blockIdx.y == 0) peer_signal(s, 0, e);
    peer_wait(s, 0, e);
  }
  __syncthreads();
  const CopyRun r = runs[blockIdx.y];
  // remote (peer-mapped) loads: no read-only cache, the data changes between epochs
  copy_run_body<true>(r, (int64_t)blockIdx.x * blockDim.x + threadIdx.x, (int64_t)gridDim.x * blockDim.x);
  peer_finish(s, e);
  pdl_trigger();
}

// global MAX of one non-negative double (its uint64 bits, exact and order-free): every rank writes its
// value into slot `me` of every participant's value array, then takes the max of its own array
__global__ void peer_allmax_kernel(unsigned long long* acc, PeerSync s, unsigned long long* const* remote_vals,
                                   unsigned long long* vals, int me, int world) {
  pdl_wait();
  const unsigned long long e = *(volatile unsigned long long*)s.epoch + 1;
  if (threadIdx.x == 0) {
    const unsigned long long v = *acc;
    *(volatile unsigned long long*)(vals + me) = v;
    for (int i = 0; i < s.npart; ++i) *(volatile unsigned long long*)(remote_vals[s.part[i]] + me) = v;
    peer_signal(s, 0, e);
    peer_wait(s, 0, e);
    unsigned long long m = 0;
    for (int r = 0; r < world; ++r) m = max(m, *(volatile unsigned long long*)(vals + r));
    *acc = m;
  }
  peer_finish(s, e);
  pdl_trigger();
}

// Before a pencil pass that reads its ghost bricks straight from the neighbours' fields (SW_PEER, the
// exchange fused into the pass): publish ready(e) -- this rank's x of the pass is complete, and its
// previous pass has finished reading the neighbours' fields -- and wait for every neighbour's ready(e).
// Then no rank reads a field its owner has not finished (RAW) and no rank overwrites, in its next
// pass, a buffer a neighbour is still reading (WAR: the neighbour's ready(e+1) comes after its pass e).
__global__ void peer_handshake_kernel(PeerSync s) {
  pdl_wait();     // the kernel that wrote this pass's x is complete ...
  pdl_trigger();  // ... so the pass (launched early) may place its CTAs now; they wait for this kernel
  if (threadIdx.x == 0) {
    const unsigned long long e = *(volatile unsigned long long*)s.epoch + 1;
    peer_signal(s, 0, e);
    peer_wait(s, 0, e);
    *s.epoch = e;
    __threadfence();
  }
}

}  // namespace

cudaError_t launch_peer_handshake(const PeerSync& s, cudaStream_t st) {
  launch_k(peer_handshake_kernel, 1, 32, 0, st, s);
  return cudaGetLastError();
}

cudaError_t launch_peer_copy(const CopyRun* runs, int nruns, int64_t max_n, const PeerSync& s, cudaStream_t st) {
  // every rank launches the kernel even without runs of its own (the flags keep the epochs in step)
  const int64_t words = std::max<int64_t>(max_n / 2, 1);
  const int ny = std::max(nruns, 1);
  const int64_t want = (int64_t)148 * 8 * 4 / ny;
  const unsigned gx = (unsigned)std::max<int64_t>(1, std::min<int64_t>((words + 255) / 256, std::max<int64_t>(1, want)));
  if (nruns <= 0) {
    // a dummy run of length 0
    launch_k(peer_copy_kernel, dim3(1, 1), 256, 0, st, s.dummy_run, s);
  } else {
    launch_k(peer_copy_kernel, dim3(gx, (unsigned)nruns), 256, 0, st, runs, s);
  }
  return cudaGetLastError();
}

cudaError_t launch_peer_allmax(unsigned long long* acc, const PeerSync& s, unsigned long long* const* remote_vals,
                               unsigned long long* vals, int me, int world, cudaStream_t st) {
  launch_k(peer_allmax_kernel, 1, 32, 0, st, acc, s, remote_vals, vals, me, world);
  return cudaGetLastError();
}

}  // namespace mgb
