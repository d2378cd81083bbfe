// reduce.cuh — deterministic block/grid reductions shared by the CUDA
// translation units of the library (kernels.cu, aniso.cu).  No fp64 atomics:
// every block publishes its partial sums, a ticket picks the last block,
// which sums the partials in block order (scheduling-independent bits).
#pragma once

#include <cuda_runtime.h>

#include "mas_internal.h"

namespace mas {

constexpr int kThreads = 256;  // 8 warps (stream kernels)

// --------------------------------------------------------------------------
// deterministic reductions
// --------------------------------------------------------------------------
__device__ __forceinline__ double warp_sum(double v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_down_sync(0xffffffffu, v, o);
    return v;  // valid in lane 0
}

// Block-reduce NS sums, publish the block partial, take a ticket.  Returns
// true in the last block to finish, where `v` then holds the grid totals
// (valid in thread 0), summed in a fixed order independent of scheduling.
// sysfence: the block's global writes are also read by peer GPUs (P2P
// transport), so order them at system scope before the ticket.
template <int NS, int NTHR = kThreads>
__device__ bool grid_reduce(double (&v)[NS], const Scratch& scr, int tkt, bool sysfence = false) {
    __shared__ double wsum[NS][NTHR / 32];
    __shared__ bool last;
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
#pragma unroll
    for (int s = 0; s < NS; s++) {
        double t = warp_sum(v[s]);
        if (lane == 0) wsum[s][w] = t;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
#pragma unroll
        for (int s = 0; s < NS; s++) {
            double t = 0.0;
            for (int q = 0; q < NTHR / 32; q++) t += wsum[s][q];
            scr.partials[(size_t)blockIdx.x * NS + s] = t;
        }
        if (sysfence)
            __threadfence_system();
        else
            __threadfence();
        unsigned old = atomicAdd(&scr.ticket[tkt], 1u);
        last = (old == gridDim.x - 1);
    }
    __syncthreads();
    if (!last) return false;
    __threadfence();
#pragma unroll
    for (int s = 0; s < NS; s++) {
        double t = 0.0;
        for (unsigned b = threadIdx.x; b < gridDim.x; b += NTHR)
            t += __ldcg(&scr.partials[(size_t)b * NS + s]);
        t = warp_sum(t);
        __syncthreads();
        if (lane == 0) wsum[s][w] = t;
        __syncthreads();
        if (threadIdx.x == 0) {
            double u = 0.0;
            for (int q = 0; q < NTHR / 32; q++) u += wsum[s][q];
            v[s] = u;
        }
    }
    if (threadIdx.x == 0) scr.ticket[tkt] = 0u;
    return true;
}

}  // namespace mas
