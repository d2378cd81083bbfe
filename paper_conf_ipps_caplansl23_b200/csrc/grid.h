// grid.h — host-side objects behind the opaque ABI handles.
#pragma once

#include <string>
#include <vector>

#include "mas_internal.h"

namespace mas {

struct Tables {  // local 1-D tables, layout of Geo (mas_internal.h)
    std::vector<double> wRm, wRp, irc2, vr, wTm, wTp, isc2, vt, wPm, wPp, vp;
};

struct Comm;  // comm.cpp (NCCL)

}  // namespace mas

struct mas_grid {
    int nr = 0, nt = 0, np = 0;
    int i0 = 0, nl = 0;
    // (r, theta) decomposition: nranks = pr * ptheta, rank = rrank * ptheta + trank
    int ptheta = 1, pr = 1, rrank = 0, trank = 0;
    int j0 = 0, ntl = 0;      // this rank's theta rows [j0, j0 + ntl)
    int pole_flags = 0;
    int nranks = 1, rank = 0;
    int device = 0;
    std::vector<double> rF, rC, tF, tC, pF, pC;
    mas::Tables tab;
    double* d_tab = nullptr;  // device copy of the theta/phi tables + irc2/vr
    double* d_tab_tn = nullptr;  // theta-node placement: [wTm wTp isc2 vt](nt+1) (both poles, ptheta 1)
    double* d_tab_pn = nullptr;  // phi-node placement: [wPm wPp vp](np)
    double* d_tab_rn = nullptr;  // r-node placement (one rank): [wRm wRp irc2 vr](nr-1)
    std::vector<double> rn_host; // the same, host copy (the op folds the boundary conditions into wR)
    mas::Comm* comm = nullptr;
};

namespace mas {

int validate_mesh(int nr, int nt, int np, const double* rF, const double* rC, const double* tF,
                  const double* tC, const double* pF, const double* pC, int pole_flags,
                  int periodic_phi, int pr, int ptheta, std::string* why);
void partition(int nr, int nranks, int rank, int* i0, int* nl);
void build_tables(mas_grid* g);
std::vector<double> tnode_tables(const mas_grid* g);
std::vector<double> pnode_tables(const mas_grid* g);
std::vector<double> rnode_tables(const mas_grid* g);

// ---- comm.cpp -------------------------------------------------------------
mas_status_t comm_unique_id(unsigned char out[128]);
mas_status_t comm_create(const mas_dist_t* d, Comm** out);
void comm_destroy(Comm* c);
// sum n doubles in place over all ranks
mas_status_t comm_allreduce(Comm* c, double* buf, int n, cudaStream_t s);
// exchange r-seams of an ncomp-component field with interior `in`
// ([ncomp][nl][plane]): send first/last plane to rank-1/rank+1, receive the
// neighbours' edge planes into glo / ghi ([ncomp][plane]).
mas_status_t comm_seams(Comm* c, const double* in, int ncomp, int nl, long long plane, double* glo,
                        double* ghi, cudaStream_t s, int nb_stride = 1);
// exchange contiguous buffers of `count` doubles with ranks lo / hi (-1: none):
// send_lo -> lo, recv_lo <- lo's send_hi; send_hi -> hi, recv_hi <- hi's send_lo
mas_status_t comm_exchange(Comm* c, int lo, int hi, const double* send_lo, const double* send_hi,
                           double* recv_lo, double* recv_hi, size_t count, cudaStream_t s);
mas_status_t comm_barrier(Comm* c, cudaStream_t s);
// P2P transport setup helpers
bool comm_is_virtual(const Comm* c);
bool comm_is_nccl(const Comm* c);
// NCCL loop waits: poll the event / stream and ncclCommGetAsyncError, abort
// the communicators on an error or after MAS_COMM_TIMEOUT_S (default 600 s)
mas_status_t comm_check_async(Comm* c);
mas_status_t comm_wait_event(Comm* c, cudaEvent_t ev);
mas_status_t comm_sync_stream(Comm* c, cudaStream_t s);
int comm_rank(const Comm* c);
int comm_nranks(const Comm* c);
mas_status_t comm_allgather_bytes(Comm* c, const void* mine, void* all, size_t n, cudaStream_t s);
mas_status_t comm_vsync(Comm* c, cudaStream_t s);

}  // namespace mas
