// comm.cpp — multi-GPU plumbing over NCCL (NVLink 5 / NVSwitch).
//
// The paper's halo ("seam") exchanges are CUDA-aware MPI with GPU
// peer-to-peer transfers (§V-C; Fig. 4),
// and distributed PCG needs a global sum per dot product.  Here: one process
// per GPU (as the paper's launch script, Listing 6), NCCL
// send/recv of the contiguous r-seam planes (layout R15 makes them
// contiguous, no packing) and an in-place fp64 allreduce of 1-3 scalars.
//
// A second transport, "virtual ranks", runs P ranks as P host threads of one
// process on ONE GPU (each with its own stream).  It implements the same two
// collectives with device copies, CUDA events and host barriers, so the
// multi-rank driver, ghost-plane kernels and stop handshake can be validated
// on a single B200 (this run has no multi-GPU box).  It is selected by a
// mas_dist_t.nccl_id beginning with "MASVIRT\0" followed by an 8-byte group
// key.  It is a test transport, not a performance path, and is honoured only
// with MAS_TEST_TRANSPORTS=1 in the environment.
#include <nccl.h>

#include <chrono>
#include <cstdlib>
#include <condition_variable>
#include <cstdio>
#include <thread>
#include <cstring>
#include <map>
#include <mutex>
#include <string>
#include <vector>

#include "grid.h"

namespace mas {

// ---------------------------------------------------------------------------
// virtual-rank group
// ---------------------------------------------------------------------------
struct VGroup {
    int n = 0;
    int refs = 0;
    std::mutex m;
    std::condition_variable cv;
    int arrived = 0;
    long gen = 0;
    double* stage = nullptr;                   // [n][8] allreduce staging (device)
    std::vector<cudaEvent_t> ev_in, ev_out;    // per rank: staged / summed
    std::vector<cudaEvent_t> ev_seam, ev_pull; // per rank: seam data ready / pulls done
    std::vector<const double*> seam_src;       // per rank: interior field of this seam call
    std::vector<int> seam_nl;
    std::vector<std::vector<unsigned char>> gather;  // allgather staging (host)
    std::vector<cudaEvent_t> ev_sync;          // per rank: comm_vsync
    std::vector<const double*> xsend;          // per rank: comm_exchange send buffers [lo, hi]

    void barrier() {
        std::unique_lock<std::mutex> lk(m);
        const long g = gen;
        if (++arrived == n) {
            arrived = 0;
            gen++;
            cv.notify_all();
        } else {
            cv.wait(lk, [&] { return gen != g; });
        }
    }
};

static std::mutex g_vmap_mutex;
static std::map<unsigned long long, VGroup*> g_vmap;

struct Comm {
    ncclComm_t nccl = nullptr;
    ncclComm_t nccl_seam = nullptr;  // split communicator: seams run on their own stream
    int nranks = 1, rank = 0;
    VGroup* vg = nullptr;
    unsigned long long vkey = 0;
    std::string hdir;                // host-exchange transport: shared directory
    long hseq = 0;                   // host-exchange call counter
};

static const char kVirtMagic[8] = {'M', 'A', 'S', 'V', 'I', 'R', 'T', 0};
static const char kHostMagic[8] = {'M', 'A', 'S', 'H', 'O', 'S', 'T', 0};

static mas_status_t nccl_fail(ncclResult_t r, const char* what) {
    set_last_error(std::string(what) + ": " + ncclGetErrorString(r));
    return MAS_ERR_NCCL;
}

static mas_status_t cuda_fail(cudaError_t e, const char* what) {
    set_last_error(std::string(what) + ": " + cudaGetErrorString(e));
    return MAS_ERR_CUDA;
}

// ---------------------------------------------------------------------------
// host-exchange transport (tests): P processes sharing ONE GPU exchange the
// setup-time collectives through files in a shared directory; everything
// else (CUDA IPC mappings, the P2P kernels) is the multi-GPU code.  NCCL
// cannot run two ranks on one device, so this is how the cross-process P2P
// path is exercised on a single B200.  Selected by a mas_dist_t.nccl_id of
// "MASHOST\0" + a NUL-terminated directory path.  Not a performance path.
// ---------------------------------------------------------------------------
static mas_status_t h_exchange(Comm* c, const void* mine, size_t n, std::vector<unsigned char>& all) {
    const long seq = ++c->hseq;
    auto name = [&](int r) { return c->hdir + "/x" + std::to_string(seq) + "." + std::to_string(r); };
    {
        const std::string tmp = name(c->rank) + ".tmp";
        FILE* f = fopen(tmp.c_str(), "wb");
        if (!f || fwrite(mine, 1, n, f) != n) {
            if (f) fclose(f);
            set_last_error("host exchange: cannot write " + tmp);
            return MAS_ERR_NCCL;
        }
        fclose(f);
        if (rename(tmp.c_str(), name(c->rank).c_str()) != 0) {
            set_last_error("host exchange: rename failed");
            return MAS_ERR_NCCL;
        }
    }
    all.assign(n * c->nranks, 0);
    for (int r = 0; r < c->nranks; r++) {
        const auto t0 = std::chrono::steady_clock::now();
        for (;;) {
            FILE* f = fopen(name(r).c_str(), "rb");
            if (f) {
                const size_t got = fread(all.data() + r * n, 1, n, f);
                fclose(f);
                if (got == n) break;
            }
            if (std::chrono::steady_clock::now() - t0 > std::chrono::seconds(120)) {
                set_last_error("host exchange: timed out waiting for rank " + std::to_string(r));
                return MAS_ERR_NCCL;
            }
            std::this_thread::sleep_for(std::chrono::microseconds(200));
        }
    }
    return MAS_OK;
}

static mas_status_t h_allreduce(Comm* c, double* buf, int n, cudaStream_t s) {
    double mine[8] = {0};
    cudaError_t e;
    if ((e = cudaMemcpyAsync(mine, buf, n * sizeof(double), cudaMemcpyDeviceToHost, s)) != cudaSuccess ||
        (e = cudaStreamSynchronize(s)) != cudaSuccess)
        return cuda_fail(e, "host allreduce");
    std::vector<unsigned char> all;
    mas_status_t st = h_exchange(c, mine, sizeof(mine), all);
    if (st != MAS_OK) return st;
    double sum[8] = {0};
    for (int r = 0; r < c->nranks; r++)
        for (int t = 0; t < n; t++) sum[t] += reinterpret_cast<const double*>(all.data() + r * sizeof(mine))[t];
    if ((e = cudaMemcpyAsync(buf, sum, n * sizeof(double), cudaMemcpyHostToDevice, s)) != cudaSuccess ||
        (e = cudaStreamSynchronize(s)) != cudaSuccess)
        return cuda_fail(e, "host allreduce");
    return MAS_OK;
}

static mas_status_t h_seams(Comm* c, const double* in, int ncomp, int nl, long long plane, double* glo,
                            double* ghi, cudaStream_t s, int stride) {
    const int lo = c->rank - stride, hi = c->rank + stride;
    // payload: [first plane, last plane] of every component
    const size_t pb = sizeof(double) * plane;
    std::vector<unsigned char> mine(2 * ncomp * pb);
    cudaError_t e;
    for (int m = 0; m < ncomp; m++) {
        const double* base = in + (long long)m * nl * plane;
        if ((e = cudaMemcpyAsync(mine.data() + (2 * m) * pb, base, pb, cudaMemcpyDeviceToHost, s)) !=
                cudaSuccess ||
            (e = cudaMemcpyAsync(mine.data() + (2 * m + 1) * pb, base + (long long)(nl - 1) * plane, pb,
                                 cudaMemcpyDeviceToHost, s)) != cudaSuccess)
            return cuda_fail(e, "host seams");
    }
    if ((e = cudaStreamSynchronize(s)) != cudaSuccess) return cuda_fail(e, "host seams");
    std::vector<unsigned char> all;
    mas_status_t st = h_exchange(c, mine.data(), mine.size(), all);
    if (st != MAS_OK) return st;
    for (int m = 0; m < ncomp; m++) {
        if (lo >= 0) {  // the lower neighbour's last plane
            const unsigned char* src = all.data() + lo * mine.size() + (2 * m + 1) * pb;
            if ((e = cudaMemcpyAsync(glo + m * plane, src, pb, cudaMemcpyHostToDevice, s)) != cudaSuccess)
                return cuda_fail(e, "host seams");
        }
        if (hi < c->nranks) {  // the upper neighbour's first plane
            const unsigned char* src = all.data() + hi * mine.size() + (2 * m) * pb;
            if ((e = cudaMemcpyAsync(ghi + m * plane, src, pb, cudaMemcpyHostToDevice, s)) != cudaSuccess)
                return cuda_fail(e, "host seams");
        }
    }
    if ((e = cudaStreamSynchronize(s)) != cudaSuccess) return cuda_fail(e, "host seams");
    return MAS_OK;
}

static mas_status_t h_xchg(Comm* c, int lo, int hi, const double* send_lo, const double* send_hi,
                           double* recv_lo, double* recv_hi, size_t count, cudaStream_t s) {
    const size_t b = count * sizeof(double);
    std::vector<unsigned char> mine(2 * b, 0);
    cudaError_t e;
    if (lo >= 0 && (e = cudaMemcpyAsync(mine.data(), send_lo, b, cudaMemcpyDeviceToHost, s)) != cudaSuccess)
        return cuda_fail(e, "host exchange");
    if (hi >= 0 && (e = cudaMemcpyAsync(mine.data() + b, send_hi, b, cudaMemcpyDeviceToHost, s)) != cudaSuccess)
        return cuda_fail(e, "host exchange");
    if ((e = cudaStreamSynchronize(s)) != cudaSuccess) return cuda_fail(e, "host exchange");
    std::vector<unsigned char> all;
    mas_status_t st = h_exchange(c, mine.data(), mine.size(), all);
    if (st != MAS_OK) return st;
    if (lo >= 0 && (e = cudaMemcpyAsync(recv_lo, all.data() + lo * 2 * b + b, b, cudaMemcpyHostToDevice, s)) !=
                       cudaSuccess)
        return cuda_fail(e, "host exchange");
    if (hi >= 0 && (e = cudaMemcpyAsync(recv_hi, all.data() + hi * 2 * b, b, cudaMemcpyHostToDevice, s)) !=
                       cudaSuccess)
        return cuda_fail(e, "host exchange");
    if ((e = cudaStreamSynchronize(s)) != cudaSuccess) return cuda_fail(e, "host exchange");
    return MAS_OK;
}

mas_status_t comm_unique_id(unsigned char out[128]) {
    static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId size");
    ncclUniqueId id;
    ncclResult_t r = ncclGetUniqueId(&id);
    if (r != ncclSuccess) return nccl_fail(r, "ncclGetUniqueId");
    memcpy(out, id.internal, 128);
    return MAS_OK;
}

static mas_status_t vgroup_join(const mas_dist_t* d, Comm* c) {
    unsigned long long key;
    memcpy(&key, d->nccl_id + 8, 8);
    VGroup* g;
    {
        std::lock_guard<std::mutex> lk(g_vmap_mutex);
        auto it = g_vmap.find(key);
        if (it == g_vmap.end()) {
            g = new VGroup();
            g->n = d->nranks;
            g->ev_in.resize(g->n);
            g->ev_out.resize(g->n);
            g->ev_seam.resize(g->n);
            g->ev_pull.resize(g->n);
            g->seam_src.assign(g->n, nullptr);
            g->seam_nl.assign(g->n, 0);
            g->gather.resize(g->n);
            g->ev_sync.resize(g->n);
            g->xsend.assign(2 * g->n, nullptr);
            cudaError_t e = cudaMalloc(&g->stage, sizeof(double) * 8 * g->n);
            for (int r = 0; r < g->n && e == cudaSuccess; r++) {
                e = cudaEventCreateWithFlags(&g->ev_in[r], cudaEventDisableTiming);
                if (e == cudaSuccess) e = cudaEventCreateWithFlags(&g->ev_out[r], cudaEventDisableTiming);
                if (e == cudaSuccess) e = cudaEventCreateWithFlags(&g->ev_seam[r], cudaEventDisableTiming);
                if (e == cudaSuccess) e = cudaEventCreateWithFlags(&g->ev_pull[r], cudaEventDisableTiming);
                if (e == cudaSuccess) e = cudaEventCreateWithFlags(&g->ev_sync[r], cudaEventDisableTiming);
            }
            if (e != cudaSuccess) return cuda_fail(e, "virtual group setup");
            g_vmap[key] = g;
        } else {
            g = it->second;
            if (g->n != d->nranks) {
                set_last_error("virtual group: nranks mismatch");
                return MAS_ERR_ARG;
            }
        }
        g->refs++;
    }
    c->vg = g;
    c->vkey = key;
    g->barrier();  // collective create
    return MAS_OK;
}

// The virtual-rank and host-exchange transports exist to validate the
// multi-rank code on one GPU; a production run never selects them by
// accident: their ids are honoured only with MAS_TEST_TRANSPORTS=1 set.
static bool test_transports_enabled() {
    const char* e = getenv("MAS_TEST_TRANSPORTS");
    return e && atoi(e) == 1;
}

mas_status_t comm_create(const mas_dist_t* d, Comm** out) {
    const bool host_magic = memcmp(d->nccl_id, kHostMagic, 8) == 0;
    const bool virt_magic = memcmp(d->nccl_id, kVirtMagic, 8) == 0;
    if ((host_magic || virt_magic) && !test_transports_enabled()) {
        set_last_error("test transport id (virtual ranks / host exchange) without MAS_TEST_TRANSPORTS=1");
        return MAS_ERR_ARG;
    }
    Comm* c = new Comm();
    c->nranks = d->nranks;
    c->rank = d->rank;
    if (host_magic) {
        char path[121];
        memcpy(path, d->nccl_id + 8, 120);
        path[120] = 0;
        c->hdir = path;
        std::vector<unsigned char> all;
        const unsigned char one = 1;
        mas_status_t s = h_exchange(c, &one, 1, all);  // collective create
        if (s != MAS_OK) {
            delete c;
            return s;
        }
        *out = c;
        return MAS_OK;
    }
    if (virt_magic) {
        mas_status_t s = vgroup_join(d, c);
        if (s != MAS_OK) {
            delete c;
            return s;
        }
        *out = c;
        return MAS_OK;
    }
    ncclUniqueId id;
    memcpy(id.internal, d->nccl_id, 128);
    ncclResult_t r = ncclCommInitRank(&c->nccl, d->nranks, id, d->rank);
    if (r != ncclSuccess) {
        delete c;
        return nccl_fail(r, "ncclCommInitRank");
    }
    // NCCL operations of one communicator must not run concurrently on two
    // streams: the seams (comm stream) get their own communicator
    r = ncclCommSplit(c->nccl, 0, d->rank, &c->nccl_seam, nullptr);
    if (r != ncclSuccess) {
        ncclCommDestroy(c->nccl);
        delete c;
        return nccl_fail(r, "ncclCommSplit");
    }
    *out = c;
    return MAS_OK;
}

void comm_destroy(Comm* c) {
    if (!c) return;
    if (c->nccl_seam) ncclCommDestroy(c->nccl_seam);
    if (c->nccl) ncclCommDestroy(c->nccl);
    if (c->vg) {
        VGroup* g = c->vg;
        g->barrier();
        std::lock_guard<std::mutex> lk(g_vmap_mutex);
        if (--g->refs == 0) {
            for (int r = 0; r < g->n; r++) {
                cudaEventDestroy(g->ev_in[r]);
                cudaEventDestroy(g->ev_out[r]);
                cudaEventDestroy(g->ev_seam[r]);
                cudaEventDestroy(g->ev_pull[r]);
                cudaEventDestroy(g->ev_sync[r]);
            }
            cudaFree(g->stage);
            g_vmap.erase(c->vkey);
            delete g;
        }
    }
    delete c;
}

// ---------------------------------------------------------------------------
// allreduce (sum, fp64, n <= 8)
// ---------------------------------------------------------------------------
static mas_status_t v_allreduce(Comm* c, double* buf, int n, cudaStream_t s) {
    VGroup* g = c->vg;
    const int r = c->rank;
    cudaError_t e;
    // stage[r] may still be read by the previous call's sums of other ranks
    for (int j = 0; j < g->n; j++)
        if (j != r && (e = cudaStreamWaitEvent(s, g->ev_out[j], 0)) != cudaSuccess)
            return cuda_fail(e, "virtual allreduce wait");
    if ((e = cudaMemcpyAsync(g->stage + 8 * r, buf, sizeof(double) * n, cudaMemcpyDeviceToDevice, s)) !=
            cudaSuccess ||
        (e = cudaEventRecord(g->ev_in[r], s)) != cudaSuccess)
        return cuda_fail(e, "virtual allreduce stage");
    g->barrier();
    for (int j = 0; j < g->n; j++)
        if ((e = cudaStreamWaitEvent(s, g->ev_in[j], 0)) != cudaSuccess)
            return cuda_fail(e, "virtual allreduce wait");
    if ((e = launch_rank_sum(buf, g->stage, g->n, n, s)) != cudaSuccess ||
        (e = cudaEventRecord(g->ev_out[r], s)) != cudaSuccess)
        return cuda_fail(e, "virtual allreduce sum");
    g->barrier();
    return MAS_OK;
}

mas_status_t comm_allreduce(Comm* c, double* buf, int n, cudaStream_t s) {
    // a 1-rank NCCL communicator still runs ncclAllReduce (the NCCL code path
    // on one GPU, mas_grid_create with a 1-rank mas_dist_t)
    if (!c || (c->nranks == 1 && !c->nccl)) return MAS_OK;
    if (c->vg) return v_allreduce(c, buf, n, s);
    if (!c->hdir.empty()) return h_allreduce(c, buf, n, s);
    ncclResult_t r = ncclAllReduce(buf, buf, n, ncclFloat64, ncclSum, c->nccl, s);
    return r == ncclSuccess ? MAS_OK : nccl_fail(r, "ncclAllReduce");
}

// ---------------------------------------------------------------------------
// seams: edge r-planes to the r-neighbours' ghost planes
// ---------------------------------------------------------------------------
static mas_status_t v_seams(Comm* c, const double* in, int ncomp, int nl, long long plane,
                            double* glo, double* ghi, cudaStream_t s, int stride) {
    VGroup* g = c->vg;
    const int r = c->rank;
    cudaError_t e;
    g->seam_src[r] = in;
    g->seam_nl[r] = nl;
    if ((e = cudaEventRecord(g->ev_seam[r], s)) != cudaSuccess) return cuda_fail(e, "virtual seam record");
    g->barrier();
    const size_t bytes = sizeof(double) * plane;
    for (int side = 0; side < 2; side++) {
        const int nb = side == 0 ? r - stride : r + stride;
        if (nb < 0 || nb >= g->n) continue;
        if ((e = cudaStreamWaitEvent(s, g->ev_seam[nb], 0)) != cudaSuccess)
            return cuda_fail(e, "virtual seam wait");
        const double* src = g->seam_src[nb];
        const int nbl = g->seam_nl[nb];
        for (int m = 0; m < ncomp; m++) {
            // lower neighbour's last plane -> my glo; upper neighbour's first plane -> my ghi
            const double* from = src + ((long long)m * nbl + (side == 0 ? nbl - 1 : 0)) * plane;
            double* to = (side == 0 ? glo : ghi) + (long long)m * plane;
            if ((e = cudaMemcpyAsync(to, from, bytes, cudaMemcpyDeviceToDevice, s)) != cudaSuccess)
                return cuda_fail(e, "virtual seam copy");
        }
    }
    if ((e = cudaEventRecord(g->ev_pull[r], s)) != cudaSuccess) return cuda_fail(e, "virtual seam record");
    g->barrier();
    // my edge planes must not be overwritten before the neighbours pulled them
    for (int nb : {r - stride, r + stride})
        if (nb >= 0 && nb < g->n && (e = cudaStreamWaitEvent(s, g->ev_pull[nb], 0)) != cudaSuccess)
            return cuda_fail(e, "virtual seam wait");
    return MAS_OK;
}

// r-seams: the r-neighbours are rank -/+ nb_stride (nb_stride = ptheta under
// an (r, theta) decomposition with theta fastest in the rank numbering)
mas_status_t comm_seams(Comm* c, const double* in, int ncomp, int nl, long long plane, double* glo,
                        double* ghi, cudaStream_t s, int nb_stride) {
    if (!c || c->nranks == 1) return MAS_OK;
    if (c->vg) return v_seams(c, in, ncomp, nl, plane, glo, ghi, s, nb_stride);
    if (!c->hdir.empty()) return h_seams(c, in, ncomp, nl, plane, glo, ghi, s, nb_stride);
    const int lo = c->rank - nb_stride, hi = c->rank + nb_stride;
    const long long Nl = (long long)nl * plane;
    ncclResult_t r = ncclGroupStart();
    if (r != ncclSuccess) return nccl_fail(r, "ncclGroupStart");
    for (int m = 0; m < ncomp; m++) {
        const double* first = in + m * Nl;
        const double* last = in + m * Nl + (long long)(nl - 1) * plane;
        if (lo >= 0) {
            ncclSend(first, plane, ncclFloat64, lo, c->nccl_seam, s);
            ncclRecv(glo + m * plane, plane, ncclFloat64, lo, c->nccl_seam, s);
        }
        if (hi < c->nranks) {
            ncclSend(last, plane, ncclFloat64, hi, c->nccl_seam, s);
            ncclRecv(ghi + m * plane, plane, ncclFloat64, hi, c->nccl_seam, s);
        }
    }
    r = ncclGroupEnd();
    return r == ncclSuccess ? MAS_OK : nccl_fail(r, "seam send/recv");
}

// ---------------------------------------------------------------------------
// exchange of packed buffers (theta-ghost rows of the 2-D decomposition)
// ---------------------------------------------------------------------------
static mas_status_t v_xchg(Comm* c, int lo, int hi, const double* send_lo, const double* send_hi,
                           double* recv_lo, double* recv_hi, size_t count, cudaStream_t s) {
    VGroup* g = c->vg;
    const int r = c->rank;
    cudaError_t e;
    g->xsend[2 * r] = send_lo;
    g->xsend[2 * r + 1] = send_hi;
    if ((e = cudaEventRecord(g->ev_seam[r], s)) != cudaSuccess) return cuda_fail(e, "virtual exchange");
    g->barrier();
    const size_t b = count * sizeof(double);
    if (lo >= 0) {  // lower neighbour's send_hi -> my recv_lo
        if ((e = cudaStreamWaitEvent(s, g->ev_seam[lo], 0)) != cudaSuccess ||
            (e = cudaMemcpyAsync(recv_lo, g->xsend[2 * lo + 1], b, cudaMemcpyDeviceToDevice, s)) != cudaSuccess)
            return cuda_fail(e, "virtual exchange");
    }
    if (hi >= 0) {  // upper neighbour's send_lo -> my recv_hi
        if ((e = cudaStreamWaitEvent(s, g->ev_seam[hi], 0)) != cudaSuccess ||
            (e = cudaMemcpyAsync(recv_hi, g->xsend[2 * hi], b, cudaMemcpyDeviceToDevice, s)) != cudaSuccess)
            return cuda_fail(e, "virtual exchange");
    }
    if ((e = cudaEventRecord(g->ev_pull[r], s)) != cudaSuccess) return cuda_fail(e, "virtual exchange");
    g->barrier();
    for (int nb : {lo, hi})
        if (nb >= 0 && (e = cudaStreamWaitEvent(s, g->ev_pull[nb], 0)) != cudaSuccess)
            return cuda_fail(e, "virtual exchange");
    return MAS_OK;
}

mas_status_t comm_exchange(Comm* c, int lo, int hi, const double* send_lo, const double* send_hi,
                           double* recv_lo, double* recv_hi, size_t count, cudaStream_t s) {
    if (!c || c->nranks == 1) return MAS_OK;  // collective: every rank calls (host/virtual barriers)
    if (c->vg) return v_xchg(c, lo, hi, send_lo, send_hi, recv_lo, recv_hi, count, s);
    if (!c->hdir.empty()) return h_xchg(c, lo, hi, send_lo, send_hi, recv_lo, recv_hi, count, s);
    ncclResult_t r = ncclGroupStart();
    if (r != ncclSuccess) return nccl_fail(r, "ncclGroupStart");
    if (lo >= 0) {
        ncclSend(send_lo, count, ncclFloat64, lo, c->nccl_seam, s);
        ncclRecv(recv_lo, count, ncclFloat64, lo, c->nccl_seam, s);
    }
    if (hi >= 0) {
        ncclSend(send_hi, count, ncclFloat64, hi, c->nccl_seam, s);
        ncclRecv(recv_hi, count, ncclFloat64, hi, c->nccl_seam, s);
    }
    r = ncclGroupEnd();
    return r == ncclSuccess ? MAS_OK : nccl_fail(r, "theta-row send/recv");
}

// ---------------------------------------------------------------------------
// setup-time helpers of the P2P transport
// ---------------------------------------------------------------------------
bool comm_is_virtual(const Comm* c) { return c && c->vg; }
bool comm_is_nccl(const Comm* c) { return c && c->nccl; }

// ---------------------------------------------------------------------------
// waiting on the NCCL loop without hanging: poll the event, and between polls
// the communicators' asynchronous error state (a peer that died or a network
// error); on an error or after the timeout (MAS_COMM_TIMEOUT_S, default 600 s)
// both communicators are aborted and MAS_ERR_NCCL is returned.
// ---------------------------------------------------------------------------
static double comm_timeout_s() {
    static const double t = [] {
        const char* e = getenv("MAS_COMM_TIMEOUT_S");
        const double v = e ? atof(e) : 600.0;
        return v > 0 ? v : 600.0;
    }();
    return t;
}

static mas_status_t comm_abort(Comm* c, const std::string& why) {
    if (c->nccl_seam) ncclCommAbort(c->nccl_seam);
    if (c->nccl) ncclCommAbort(c->nccl);
    c->nccl_seam = c->nccl = nullptr;
    set_last_error(why);
    return MAS_ERR_NCCL;
}

mas_status_t comm_check_async(Comm* c) {
    if (!c || !c->nccl) return MAS_OK;
    for (ncclComm_t cm : {c->nccl, c->nccl_seam}) {
        ncclResult_t ar = ncclSuccess;
        if (cm && ncclCommGetAsyncError(cm, &ar) == ncclSuccess && ar != ncclSuccess && ar != ncclInProgress)
            return comm_abort(c, std::string("NCCL asynchronous error: ") + ncclGetErrorString(ar));
    }
    return MAS_OK;
}

mas_status_t comm_wait_event(Comm* c, cudaEvent_t ev) {
    if (!c || !c->nccl) {
        cudaError_t e = cudaEventSynchronize(ev);
        return e == cudaSuccess ? MAS_OK : cuda_fail(e, "cudaEventSynchronize");
    }
    const auto t0 = std::chrono::steady_clock::now();
    for (unsigned n = 0;; n++) {
        cudaError_t e = cudaEventQuery(ev);
        if (e == cudaSuccess) return MAS_OK;
        if (e != cudaErrorNotReady) return cuda_fail(e, "cudaEventQuery");
        if ((n & 63) == 63) {
            mas_status_t st = comm_check_async(c);
            if (st != MAS_OK) return st;
            const double dt = std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
            if (dt > comm_timeout_s())
                return comm_abort(c, "NCCL loop: no progress for " + std::to_string((int)dt) +
                                         " s (MAS_COMM_TIMEOUT_S); communicators aborted");
        }
        std::this_thread::yield();
    }
}

mas_status_t comm_sync_stream(Comm* c, cudaStream_t s) {
    if (!c || !c->nccl) {
        cudaError_t e = cudaStreamSynchronize(s);
        return e == cudaSuccess ? MAS_OK : cuda_fail(e, "cudaStreamSynchronize");
    }
    cudaEvent_t ev;
    cudaError_t e = cudaEventCreateWithFlags(&ev, cudaEventDisableTiming);
    if (e == cudaSuccess) e = cudaEventRecord(ev, s);
    if (e != cudaSuccess) return cuda_fail(e, "comm_sync_stream");
    mas_status_t st = comm_wait_event(c, ev);
    cudaEventDestroy(ev);
    return st;
}
int comm_rank(const Comm* c) { return c ? c->rank : 0; }
int comm_nranks(const Comm* c) { return c ? c->nranks : 1; }

// all[r * n .. r * n + n) = rank r's `mine` (host buffers), for every rank r
mas_status_t comm_allgather_bytes(Comm* c, const void* mine, void* all, size_t n, cudaStream_t s) {
    if (!c || c->nranks == 1) {
        memcpy(all, mine, n);
        return MAS_OK;
    }
    if (!c->hdir.empty()) {
        std::vector<unsigned char> v;
        mas_status_t st = h_exchange(c, mine, n, v);
        if (st == MAS_OK) memcpy(all, v.data(), n * c->nranks);
        return st;
    }
    if (c->vg) {
        VGroup* g = c->vg;
        g->gather[c->rank].assign((const unsigned char*)mine, (const unsigned char*)mine + n);
        g->barrier();
        for (int r = 0; r < g->n; r++) memcpy((unsigned char*)all + r * n, g->gather[r].data(), n);
        g->barrier();
        return MAS_OK;
    }
    unsigned char* d = nullptr;
    cudaError_t e = cudaMalloc(&d, n * (c->nranks + 1));
    if (e != cudaSuccess) return cuda_fail(e, "allgather buffer");
    mas_status_t st = MAS_OK;
    if ((e = cudaMemcpyAsync(d, mine, n, cudaMemcpyHostToDevice, s)) != cudaSuccess) {
        st = cuda_fail(e, "allgather copy");
    } else {
        ncclResult_t r = ncclAllGather(d, d + n, n, ncclChar, c->nccl, s);
        if (r != ncclSuccess)
            st = nccl_fail(r, "ncclAllGather");
        else if ((e = cudaMemcpyAsync(all, d + n, n * c->nranks, cudaMemcpyDeviceToHost, s)) !=
                     cudaSuccess ||
                 (e = cudaStreamSynchronize(s)) != cudaSuccess)
            st = cuda_fail(e, "allgather copy back");
    }
    cudaFree(d);
    return st;
}

// Virtual ranks only: order stream s after the work every rank has enqueued
// so far.  The P2P kernels' mailbox waits are then already satisfied when a
// kernel starts: on one GPU a spinning consumer could otherwise occupy the
// SMs its producer (another virtual rank's kernel) needs.
mas_status_t comm_vsync(Comm* c, cudaStream_t s) {
    if (!c || !c->vg) return MAS_OK;
    VGroup* g = c->vg;
    cudaError_t e;
    if ((e = cudaEventRecord(g->ev_sync[c->rank], s)) != cudaSuccess) return cuda_fail(e, "vsync record");
    g->barrier();
    for (int r = 0; r < g->n; r++)
        if (r != c->rank && (e = cudaStreamWaitEvent(s, g->ev_sync[r], 0)) != cudaSuccess)
            return cuda_fail(e, "vsync wait");
    g->barrier();  // every rank captured the events before they are recorded again
    return MAS_OK;
}

mas_status_t comm_barrier(Comm* c, cudaStream_t s) {
    if (!c || c->nranks == 1) return MAS_OK;
    if (c->vg) {
        if (cudaStreamSynchronize(s) != cudaSuccess) return MAS_ERR_CUDA;
        c->vg->barrier();
        return MAS_OK;
    }
    if (!c->hdir.empty()) {
        if (cudaStreamSynchronize(s) != cudaSuccess) return MAS_ERR_CUDA;
        std::vector<unsigned char> all;
        const unsigned char one = 1;
        return h_exchange(c, &one, 1, all);
    }
    double* d = nullptr;
    if (cudaMallocAsync(&d, sizeof(double), s) != cudaSuccess) return MAS_ERR_CUDA;
    cudaMemsetAsync(d, 0, sizeof(double), s);
    mas_status_t st = comm_allreduce(c, d, 1, s);
    cudaFreeAsync(d, s);
    if (cudaStreamSynchronize(s) != cudaSuccess) return MAS_ERR_CUDA;
    return st;
}

}  // namespace mas
