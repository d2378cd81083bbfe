// comm.cpp — multi-GPU plumbing over NCCL (NVLink 5 / NVSwitch).
//
// The paper's halo ("seam") exchanges are CUDA-aware MPI with GPU
// peer-to-peer transfers (§V-C; Fig. 4),
// and distributed PCG needs a global sum per dot product.  Here: one process
// per GPU (as the paper's launch script, Listing 6), NCCL
// send/recv of the contiguous r-seam planes (layout R15 makes them
// contiguous, no packing) and an in-place fp64 allreduce of 1-3 scalars.
#include <nccl.h>

#include <cstring>
#include <string>

#include "grid.h"

namespace mas {

struct Comm {
    ncclComm_t nccl = nullptr;
    int nranks = 1, rank = 0;
};

static mas_status_t nccl_fail(ncclResult_t r, const char* what) {
    set_last_error(std::string(what) + ": " + ncclGetErrorString(r));
    return MAS_ERR_NCCL;
}

mas_status_t comm_unique_id(unsigned char out[128]) {
    static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId size");
    ncclUniqueId id;
    ncclResult_t r = ncclGetUniqueId(&id);
    if (r != ncclSuccess) return nccl_fail(r, "ncclGetUniqueId");
    memcpy(out, id.internal, 128);
    return MAS_OK;
}

mas_status_t comm_create(const mas_dist_t* d, Comm** out) {
    Comm* c = new Comm();
    c->nranks = d->nranks;
    c->rank = d->rank;
    ncclUniqueId id;
    memcpy(id.internal, d->nccl_id, 128);
    ncclResult_t r = ncclCommInitRank(&c->nccl, d->nranks, id, d->rank);
    if (r != ncclSuccess) {
        delete c;
        return nccl_fail(r, "ncclCommInitRank");
    }
    *out = c;
    return MAS_OK;
}

void comm_destroy(Comm* c) {
    if (!c) return;
    if (c->nccl) ncclCommDestroy(c->nccl);
    delete c;
}

mas_status_t comm_allreduce(Comm* c, double* buf, int n, cudaStream_t s) {
    if (!c || c->nranks == 1) return MAS_OK;
    ncclResult_t r = ncclAllReduce(buf, buf, n, ncclFloat64, ncclSum, c->nccl, s);
    return r == ncclSuccess ? MAS_OK : nccl_fail(r, "ncclAllReduce");
}

mas_status_t comm_seams(Comm* c, const double* in, int ncomp, int nl, long long plane, double* glo,
                        double* ghi, cudaStream_t s) {
    if (!c || c->nranks == 1) return MAS_OK;
    const long long Nl = (long long)nl * plane;
    ncclResult_t r = ncclGroupStart();
    if (r != ncclSuccess) return nccl_fail(r, "ncclGroupStart");
    for (int m = 0; m < ncomp; m++) {
        const double* first = in + m * Nl;
        const double* last = in + m * Nl + (long long)(nl - 1) * plane;
        if (c->rank > 0) {
            ncclSend(first, plane, ncclFloat64, c->rank - 1, c->nccl, s);
            ncclRecv(glo + m * plane, plane, ncclFloat64, c->rank - 1, c->nccl, s);
        }
        if (c->rank < c->nranks - 1) {
            ncclSend(last, plane, ncclFloat64, c->rank + 1, c->nccl, s);
            ncclRecv(ghi + m * plane, plane, ncclFloat64, c->rank + 1, c->nccl, s);
        }
    }
    r = ncclGroupEnd();
    return r == ncclSuccess ? MAS_OK : nccl_fail(r, "seam send/recv");
}

mas_status_t comm_barrier(Comm* c, cudaStream_t s) {
    if (!c || c->nranks == 1) return MAS_OK;
    double* d = nullptr;
    if (cudaMallocAsync(&d, sizeof(double), s) != cudaSuccess) return MAS_ERR_CUDA;
    cudaMemsetAsync(d, 0, sizeof(double), s);
    mas_status_t st = comm_allreduce(c, d, 1, s);
    cudaFreeAsync(d, s);
    if (cudaStreamSynchronize(s) != cudaSuccess) return MAS_ERR_CUDA;
    return st;
}

}  // namespace mas
