// nvls.cu — SURVEY 8(f) f3 / 8(e) step 3: the per-rank partial maps summed INSIDE the NVSwitch
// (NVLink SHARP multimem), one process per GPU.  PAPER.md:198 counts this communication in the
// runtime; PAPER.md:147 has NCCL carry multi-device traffic — this is the hand-written
// alternative to NCCL's all_reduce for the one exchange of the path.
//
// The buffer (the dense map or the packed union of hit submaps) is mapped by every rank AND by a
// multicast object covering all ranks' copies (the mapping is plumbing: torch symmetric memory
// creates it).  Rank r reduces the r-th 1/world slice: `multimem.ld_reduce.add.f64` returns the
// sum of the element over all ranks (the switch adds), `multimem.st` writes that sum back to every
// rank's copy.  Two signal-pad barriers bracket it: after every rank's accumulation (before any
// reduce reads) and after every slice is written (before any rank reads its map).
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>

#include "internal.h"

namespace toastb200 {

namespace {

// Signal-pad barrier over `world` ranks (thread p of CTA 0 handles peer p): mark this rank's
// arrival in every peer's pad (waiting until the peer consumed the previous mark), then wait for
// and consume every peer's mark in this rank's pad.  System-scope atomics: the pads live in the
// peers' memory (NVLink P2P).
__global__ void nvls_barrier_kernel(unsigned* const* __restrict__ pads, int rank, int world) {
    const int p = (int)threadIdx.x;
    __threadfence_system();  // release: this rank's earlier writes before its arrival mark
    if (p < world) {
        unsigned* remote = pads[p] + rank;
        while (atomicCAS_system(remote, 0u, 1u) != 0u) {
        }
        unsigned* local = pads[rank] + p;
        while (atomicCAS_system(local, 1u, 0u) != 1u) {
        }
    }
    __syncthreads();
    __threadfence_system();  // acquire: the peers' writes before anything after the barrier
}

// Rank `rank`'s slice [lo, hi) of the multicast buffer: sum over ranks, stored to every rank.
__global__ void __launch_bounds__(256) nvls_allreduce_kernel(double* __restrict__ mc, int64_t lo, int64_t hi) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t i = lo + (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < hi; i += stride) {
        double v;
        asm volatile("multimem.ld_reduce.relaxed.sys.global.add.f64 %0, [%1];" : "=d"(v) : "l"(mc + i) : "memory");
        asm volatile("multimem.st.relaxed.sys.global.f64 [%0], %1;" ::"l"(mc + i), "d"(v) : "memory");
    }
}

}  // namespace

cudaError_t launch_map_allreduce_nvls(double* mc, int64_t n, unsigned* const* pads, int rank, int world,
                                      cudaStream_t st) {
    const int64_t per = (n + world - 1) / world;
    const int64_t lo = std::min<int64_t>(n, (int64_t)rank * per), hi = std::min<int64_t>(n, lo + per);
    if (world > 1) nvls_barrier_kernel<<<1, 32 * ((world + 31) / 32), 0, st>>>(pads, rank, world);
    if (hi > lo) {
        const int64_t want = (hi - lo + 255) / 256;
        const int grid = (int)std::min<int64_t>(want, (int64_t)num_sms() * 8);
        nvls_allreduce_kernel<<<grid, 256, 0, st>>>(mc, lo, hi);
    }
    if (world > 1) nvls_barrier_kernel<<<1, 32 * ((world + 31) / 32), 0, st>>>(pads, rank, world);
    return cudaGetLastError();
}

}  // namespace toastb200
