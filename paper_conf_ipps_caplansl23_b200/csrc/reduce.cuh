// reduce.cuh — deterministic block/grid reductions shared by the CUDA
// translation units of the library (kernels.cu, aniso.cu).  No fp64 atomics:
// every block publishes its partial sums, a ticket picks the last block,
// which sums the partials in block order (scheduling-independent bits).
#pragma once

#include <cuda_runtime.h>

#include <cstdio>

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


// --------------------------------------------------------------------------
// P2P transport: one-shot allreduce through peer mailboxes (NVLink stores)
// --------------------------------------------------------------------------
// The reducing kernel's last block writes its rank-local partials into slot
// [rank] of EVERY rank's mailbox, then (after a system-scope fence) the
// sequence number.  A consumer kernel waits in thread 0 of each block until
// all nranks entries of its own mailbox carry the expected sequence and sums
// them in rank order: every rank obtains the same bits, so every rank takes
// the same stop / breakdown decision and the loop needs no host handshake.
// A publication of iteration k needs every rank past its consumer of
// iteration k-1 (each kernel waits for all ranks' previous partials), so one
// mailbox slot per kernel kind suffices.
__device__ __forceinline__ unsigned long long p2p_seq(unsigned long long epoch, int k) {
    return (epoch << 32) | (unsigned long long)(unsigned)(k + 1);
}
__device__ __forceinline__ unsigned long long gtimer_ns() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}
constexpr unsigned long long kP2PTimeoutNs = 60ull * 1000000000ull;
// slow path: spin (with a 60 s limit: fail loudly rather than hang)
static __device__ __noinline__ void p2p_wait(const volatile unsigned long long* sp, unsigned long long seq,
                                      int rank, int slot, int from) {
    const unsigned long long t0 = gtimer_ns();
    while (*sp != seq) {
        __nanosleep(100);
        if (gtimer_ns() - t0 > kP2PTimeoutNs) {
            printf("maspcg: P2P mailbox wait timed out (rank %d, slot %d, from rank %d)\n", rank,
                   slot, from);
            __trap();
        }
    }
}

// the calling thread waits for and sums the nranks entries (rank order)
template <int N>
__device__ __forceinline__ void p2p_gather_one(const P2P& t, int slot, unsigned long long seq,
                                               double (&out)[N]) {
    const Mail* mb = t.own + slot * t.nranks;
#pragma unroll
    for (int n = 0; n < N; n++) out[n] = 0.0;
    for (int q = 0; q < t.nranks; q++) {
        const volatile unsigned long long* sp = &mb[q].seq;
        if (*sp != seq) p2p_wait(sp, seq, t.rank, slot, q);
        __threadfence_system();  // the values were written before the sequence
        const volatile double* v = mb[q].v;
#pragma unroll
        for (int n = 0; n < N; n++) out[n] += v[n];
    }
}

// thread 0 of the last block: publish n rank-local partials to every rank
static __device__ void p2p_publish(const P2P& t, int slot, unsigned long long seq, const double* v, int n) {
    for (int q = 0; q < t.nranks; q++) {
        volatile Mail* m = t.peers[q] + slot * t.nranks + t.rank;
        for (int i = 0; i < n; i++) m->v[i] = v[i];
    }
    __threadfence_system();
    for (int q = 0; q < t.nranks; q++) {
        volatile Mail* m = t.peers[q] + slot * t.nranks + t.rank;
        m->seq = seq;
    }
}

}  // namespace mas
