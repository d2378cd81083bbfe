// capi.cpp — the extern "C" boundary (include/mas_pcg.h) and the PCG driver.
//
// Host logic only: argument checking, device buffers, the iteration loop
// that enqueues kernel A / kernel B (kernels.cu) with NCCL allreduces and
// seam exchanges between them (multi-GPU), and the convergence handshake.
// The host never sees alpha/beta/residuals during the solve: they live in
// PcgState on the device (PAPER.md lesson: avoid host involvement and launch
// gaps; asynchronous launches).
#include <cuda_runtime.h>

#include <cmath>
#include <cstddef>
#include <cstdlib>
#include <cstring>
#include <functional>
#include <new>
#include <string>
#include <vector>

#include <nvtx3/nvToolsExt.h>

#include "grid.h"

namespace mas {

// NVTX ranges (header-only NVTX3): solve / setup / per-iteration phases show
// up in Nsight Systems timelines like the paper's Fig. 4.
struct NvtxRange {
    explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
    ~NvtxRange() { nvtxRangePop(); }
};

static thread_local std::string g_last_error;
void set_last_error(const std::string& msg) { g_last_error = msg; }

#define CU(call)                                                                        \
    do {                                                                                \
        cudaError_t e_ = (call);                                                        \
        if (e_ != cudaSuccess) {                                                        \
            set_last_error(std::string(#call) + ": " + cudaGetErrorString(e_));         \
            return MAS_ERR_CUDA;                                                        \
        }                                                                               \
    } while (0)

#define ST(call)                                   \
    do {                                           \
        mas_status_t s_ = (call);                  \
        if (s_ != MAS_OK) return s_;               \
    } while (0)

static mas_status_t arg_error(const std::string& why) {
    set_last_error(why);
    return MAS_ERR_ARG;
}

static bool is_device_ptr(const void* p) {
    cudaPointerAttributes at;
    if (cudaPointerGetAttributes(&at, p) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    return at.type == cudaMemoryTypeDevice || at.type == cudaMemoryTypeManaged;
}

template <class T>
static mas_status_t dmalloc(T** p, size_t n) {
    if (n == 0) { *p = nullptr; return MAS_OK; }
    cudaError_t e = cudaMalloc(reinterpret_cast<void**>(p), n * sizeof(T));
    if (e != cudaSuccess) {
        cudaGetLastError();
        set_last_error(std::string("cudaMalloc: ") + cudaGetErrorString(e));
        return e == cudaErrorMemoryAllocation ? MAS_ERR_NOMEM : MAS_ERR_CUDA;
    }
    return MAS_OK;
}

}  // namespace mas

using namespace mas;

struct mas_op {
    mas_grid* g = nullptr;
    int ncomp = 1;
    mas_bc_t bci = MAS_BC_DIRICHLET, bco = MAS_BC_NEUMANN;
    long long Nl = 0;           // local cells per component
    double *kappa = nullptr, *c = nullptr, *dinv = nullptr;
    double *kg = nullptr;       // kappa ghosts [2][plane] (lo, hi)
    double *dg = nullptr;       // dinv ghosts
    double *wR = nullptr;       // [2*nl] bc-folded radial tables (wRm, wRp)
    Geo geo{};
    // PCG work vectors [ncomp][nl][plane]
    double *r = nullptr, *p[2] = {nullptr, nullptr}, *q = nullptr;
    double *rg = nullptr;       // r ghosts [2][ncomp][plane]
    double *pg[2] = {nullptr, nullptr};
    double *xg = nullptr;       // x ghosts (init residual)
    double *stage_a = nullptr, *stage_b = nullptr;  // host-pointer staging
    PcgState* st = nullptr;
    double* hist = nullptr;     // [3][cap]: rho, sigma, rr
    int hist_cap = 0;
    Scratch scr{};
    double* dot_out = nullptr;
    int* bad = nullptr;
    int* host_flag = nullptr;   // mapped pinned
    int* host_flag_dev = nullptr;
    int chunk = 16;
    int b_blocks = 0;
    int max_blocks = 0;
    cudaEvent_t ev[2] = {nullptr, nullptr};
    // multi-GPU: seams run on their own stream while kernel A works on the
    // interior chunks (which need no ghost plane)
    cudaStream_t cs = nullptr;
    cudaEvent_t ev_ready = nullptr, ev_seam = nullptr;
    long long launches = 0;
    // optional per-kernel timing of the solve (CUDA events on its stream)
    int prof = 0;
    std::vector<cudaEvent_t> pev;  // 6 per iteration: A, B, L_par start/end
    double prof_a_ms = 0.0, prof_b_ms = 0.0, prof_c_ms = 0.0, prof_init_ms = 0.0;
    int prof_n = 0;
    // single-GPU solve loop as one CUDA graph: a device-side while node whose
    // body is two PCG iterations (A, B, A, B); rebuilt when x or the history
    // buffers move.
    cudaGraphExec_t gexec = nullptr;
    cudaStream_t cap_stream = nullptr;
    const double* g_x = nullptr;
    const double* g_hist = nullptr;
    int g_aniso = -1;
    int g_pre = -1;
    int use_graph = 1;
    int graph_pre = 0;                 // MAS_GRAPH_PRE: iteration 1 outside the graph
    // P2P transport (mas_op_enable_p2p): mailbox allreduce + in-place reads of
    // the r-neighbours' edge planes over NVLink instead of NCCL in the loop
    int p2p = 0;
    Mail* mbox = nullptr;              // own mailbox [2 slots][nranks]
    Mail** d_peers = nullptr;          // device array [nranks] of every rank's mailbox
    std::vector<void*> ipc_opened;     // cudaIpcOpenMemHandle mappings (closed at destroy)
    const double* nb_r[2] = {nullptr, nullptr};  // rank-1 / rank+1 r arrays
    // the single-reduction loop's other ping-pong buffers of the r-neighbours
    // (r2, w = q, w2), mapped when the loop was on before mas_op_enable_p2p
    const double* nb_cg[3][2] = {{nullptr, nullptr}, {nullptr, nullptr}, {nullptr, nullptr}};
    int p2p_cg1 = 0;
    const double* nb_p[2][2] = {{nullptr, nullptr}, {nullptr, nullptr}};  // [parity][lo/hi]
    int nb_nl[2] = {0, 0};             // their slab sizes
    unsigned long long epoch = 0;      // solves so far (mailbox sequence numbers)
    // (r, theta) decomposition (NEXT-3): theta-ghost rows, packed [2][ncomp][nl][np]
    int tlo = -1, thi = -1;            // theta-neighbour ranks (-1: pole / wall side)
    double *kgt = nullptr, *dgt = nullptr;       // kappa, 1/D rows (static, per op_load)
    double *xgt = nullptr, *rgt = nullptr;       // x (apply / init), r (NCCL loop)
    double *pgt[2] = {nullptr, nullptr};         // p_{k-1} (NCCL loop)
    double* tpack = nullptr;                     // pack buffer of the own first/last rows
    const double* nbt_r[2] = {nullptr, nullptr};                         // P2P: theta nbrs' r
    const double* nbt_p[2][2] = {{nullptr, nullptr}, {nullptr, nullptr}};  // [parity][lo/hi]
    int nbt_ntl[2] = {0, 0};                     // their theta rows
    // field-aligned conduction term L_par (NEXT-4, mas_op_set_aniso)
    int aniso = 0;
    double* ca = nullptr;                        // corner coefficients [3][nl][nt][np]
    double* cag = nullptr;                       // r-slabs: their ghost planes [2][3][plane]
    double* pkg = nullptr;                       // r-slabs: p_k ghost planes [2][plane]
    // per-radius sums (mas_op_radial_sums): weights and results, device
    double* rs_w = nullptr;
    double* rs_out = nullptr;
    double* astage = nullptr;                    // host kpar / b staging [4][nl][nt][np]
    // single-reduction PCG (NEXT-1, mas_op_set_single_reduction): ping-pong r,
    // w = L D^-1 r and s = L p (r: r / r2, w: q / w2, s: p[0] / p[1]), p in place
    int cg1 = 0;
    double *r2 = nullptr, *w2 = nullptr, *pcg = nullptr;
    // placement (NEXT-2): 0 cell centres; 1 theta nodes with pole rows (local
    // rows 0 and nt hold one value per radius: k_pole_avg after every stencil);
    // 2 r nodes, 3 phi nodes (face-centred: other 1-D tables only)
    int tnode = 0;
    int placement = MAS_PLACE_CELL;
    // vector-Laplacian curvature terms of the 3-component operator (NEXT-2, R31)
    int curv = 0;
    // the field-aligned term's iteration part fused into kernel A
    // (MAS_LPAR_FUSED=1 at setup; default: the separate k_aniso<PCGA>)
    int lpar_fused = 0;
    cudaGraphExec_t gexec1 = nullptr;
    const double* g1_x = nullptr;
    double* atab = nullptr;                      // AnisoTab arrays (device)
    AnisoTab at{};
};

extern "C" {

const char* mas_version(void) { return "maspcg 0.1 sm_100a"; }

const char* mas_status_string(mas_status_t s) {
    switch (s) {
        case MAS_OK: return "ok";
        case MAS_NOT_CONVERGED: return "not converged (x holds the last iterate)";
        case MAS_ERR_ARG: return "invalid argument";
        case MAS_ERR_CUDA: return "CUDA error";
        case MAS_ERR_NCCL: return "NCCL error";
        case MAS_ERR_NOMEM: return "out of device memory";
        case MAS_ERR_BREAKDOWN: return "PCG breakdown (<p,Lp> <= 0 or non-finite)";
    }
    return "unknown status";
}

const char* mas_last_error(void) { return g_last_error.c_str(); }

mas_status_t mas_comm_unique_id(unsigned char out[128]) {
    if (!out) return arg_error("null out");
    return comm_unique_id(out);
}

mas_status_t mas_grid_create(int nr, int nt, int np, const double* r_node, const double* r_half,
                             const double* t_node, const double* t_half, const double* p_node,
                             const double* p_half, int pole_flags, int periodic_phi,
                             const mas_dist_t* dist, mas_grid_t** out) {
    return mas_grid_create_2d(nr, nt, np, r_node, r_half, t_node, t_half, p_node, p_half,
                              pole_flags, periodic_phi, dist, 1, out);
}

mas_status_t mas_grid_create_2d(int nr, int nt, int np, const double* r_node, const double* r_half,
                                const double* t_node, const double* t_half, const double* p_node,
                                const double* p_half, int pole_flags, int periodic_phi,
                                const mas_dist_t* dist, int ptheta, mas_grid_t** out) {
    if (!out) return arg_error("null out");
    *out = nullptr;
    const int nranks = dist ? dist->nranks : 1;
    const int rank = dist ? dist->rank : 0;
    if (dist && (rank < 0 || rank >= nranks)) return arg_error("bad rank");
    if (ptheta < 1 || nranks % ptheta) return arg_error("ptheta must divide nranks");
    const int pr = nranks / ptheta;
    std::string why;
    if (!validate_mesh(nr, nt, np, r_node, r_half, t_node, t_half, p_node, p_half, pole_flags,
                       periodic_phi, pr, ptheta, &why))
        return arg_error(why);
    mas_grid* g = new (std::nothrow) mas_grid();
    if (!g) return MAS_ERR_NOMEM;
    g->nr = nr; g->nt = nt; g->np = np;
    g->pole_flags = pole_flags;
    g->nranks = nranks; g->rank = rank;
    g->rF.assign(r_node, r_node + nr + 1); g->rC.assign(r_half, r_half + nr);
    g->tF.assign(t_node, t_node + nt + 1); g->tC.assign(t_half, t_half + nt);
    g->pF.assign(p_node, p_node + np + 1); g->pC.assign(p_half, p_half + np);
    g->ptheta = ptheta;
    g->pr = pr;
    g->rrank = rank / ptheta;  // theta fastest in the rank numbering
    g->trank = rank % ptheta;
    partition(nr, pr, g->rrank, &g->i0, &g->nl);
    partition(nt, ptheta, g->trank, &g->j0, &g->ntl);
    build_tables(g);
    if (cudaGetDevice(&g->device) != cudaSuccess) {
        cudaGetLastError();
        delete g;
        set_last_error("no CUDA device");
        return MAS_ERR_CUDA;
    }
    // device tables: [irc2 vr](nl) [wTm wTp isc2 vt](nt) [wPm wPp vp](np)
    const Tables& T = g->tab;
    std::vector<double> h;
    for (auto* v : {&T.irc2, &T.vr, &T.wTm, &T.wTp, &T.isc2, &T.vt, &T.wPm, &T.wPp, &T.vp})
        h.insert(h.end(), v->begin(), v->end());
    mas_status_t s = dmalloc(&g->d_tab, h.size());
    if (s != MAS_OK) { delete g; return s; }
    if (cudaMemcpy(g->d_tab, h.data(), h.size() * sizeof(double), cudaMemcpyHostToDevice) !=
        cudaSuccess) {
        cudaFree(g->d_tab);
        delete g;
        set_last_error("cudaMemcpy tables");
        return MAS_ERR_CUDA;
    }
    if (pole_flags == (MAS_POLE_NORTH | MAS_POLE_SOUTH) && ptheta == 1 && nt >= 2) {
        // the theta-node placement's tables (NEXT-2): both poles on the mesh
        const std::vector<double> tn = tnode_tables(g);
        s = dmalloc(&g->d_tab_tn, tn.size());
        if (s == MAS_OK && cudaMemcpy(g->d_tab_tn, tn.data(), tn.size() * sizeof(double),
                                      cudaMemcpyHostToDevice) != cudaSuccess)
            s = MAS_ERR_CUDA;
        if (s != MAS_OK) {
            cudaFree(g->d_tab);
            if (g->d_tab_tn) cudaFree(g->d_tab_tn);
            delete g;
            set_last_error("theta-node tables");
            return s;
        }
    }
    {  // the face-centred placements' tables (NEXT-2): phi nodes always, r nodes on one rank
        const std::vector<double> pn = pnode_tables(g);
        s = dmalloc(&g->d_tab_pn, pn.size());
        if (s == MAS_OK && cudaMemcpy(g->d_tab_pn, pn.data(), pn.size() * sizeof(double),
                                      cudaMemcpyHostToDevice) != cudaSuccess)
            s = MAS_ERR_CUDA;
        if (s == MAS_OK && nranks == 1 && nr >= 2) {
            g->rn_host = rnode_tables(g);
            s = dmalloc(&g->d_tab_rn, g->rn_host.size());
            if (s == MAS_OK && cudaMemcpy(g->d_tab_rn, g->rn_host.data(), g->rn_host.size() * sizeof(double),
                                          cudaMemcpyHostToDevice) != cudaSuccess)
                s = MAS_ERR_CUDA;
        }
        if (s != MAS_OK) {
            for (double* p : {g->d_tab, g->d_tab_tn, g->d_tab_pn, g->d_tab_rn})
                if (p) cudaFree(p);
            delete g;
            set_last_error("face-placement tables");
            return s;
        }
    }
    if (dist) {  // nranks == 1 with a real NCCL id: a 1-rank communicator (the NCCL loop on one GPU)
        s = comm_create(dist, &g->comm);
        if (s != MAS_OK) {
            for (double* p : {g->d_tab, g->d_tab_tn, g->d_tab_pn, g->d_tab_rn})
                if (p) cudaFree(p);
            delete g;
            return s;
        }
    }
    *out = g;
    return MAS_OK;
}

mas_status_t mas_partition(int nr, int nranks, int rank, int* i0, int* nr_local) {
    if (!i0 || !nr_local) return arg_error("null argument");
    if (nranks < 1 || nr < nranks || rank < 0 || rank >= nranks)
        return arg_error("need 1 <= nranks <= nr and 0 <= rank < nranks");
    partition(nr, nranks, rank, i0, nr_local);
    return MAS_OK;
}

mas_status_t mas_grid_local_extent(const mas_grid_t* g, int* i0, int* nr_local) {
    if (!g || !i0 || !nr_local) return arg_error("null argument");
    *i0 = g->i0;
    *nr_local = g->nl;
    return MAS_OK;
}

mas_status_t mas_grid_local_extent_2d(const mas_grid_t* g, int* i0, int* nr_local, int* j0,
                                      int* nt_local) {
    if (!g || !i0 || !nr_local || !j0 || !nt_local) return arg_error("null argument");
    *i0 = g->i0;
    *nr_local = g->nl;
    *j0 = g->j0;
    *nt_local = g->ntl;
    return MAS_OK;
}

mas_status_t mas_grid_destroy(mas_grid_t* g) {
    if (!g) return MAS_OK;
    for (double* p : {g->d_tab, g->d_tab_tn, g->d_tab_pn, g->d_tab_rn})
        if (p) cudaFree(p);
    comm_destroy(g->comm);
    delete g;
    return MAS_OK;
}

}  // extern "C"

// ---------------------------------------------------------------------------
// op internals
// ---------------------------------------------------------------------------
static Halo halo_of(const mas_op* op, const double* in, const double* ghosts, int ncomp) {
    Halo h;
    h.in = in;
    const long long plane = op->geo.plane;
    h.glo = (ghosts && !op->geo.glob_lo) ? ghosts : nullptr;
    h.ghi = (ghosts && !op->geo.glob_hi) ? ghosts + (long long)ncomp * plane : nullptr;
    h.slo = h.shi = (int)plane;
    return h;
}

// P2P transport: the ghost planes are the r-neighbours' own edge planes,
// read in place (lo: last plane of rank-1's array, hi: first plane of rank+1's)
static Halo peer_halo(const mas_op* op, const double* in, const double* lo, const double* hi) {
    Halo h;
    h.in = in;
    const long long plane = op->geo.plane;
    h.glo = (lo && !op->geo.glob_lo) ? lo + (long long)(op->nb_nl[0] - 1) * plane : nullptr;
    h.ghi = (hi && !op->geo.glob_hi) ? hi : nullptr;
    h.slo = (int)(op->nb_nl[0] * plane);
    h.shi = (int)(op->nb_nl[1] * plane);
    return h;
}

// the fields kernel A reads with an r-halo in iteration k: r_{k-1}, p_{k-1}
static Halo r_halo(const mas_op* op) {
    return op->p2p ? peer_halo(op, op->r, op->nb_r[0], op->nb_r[1])
                   : halo_of(op, op->r, op->rg, op->ncomp);
}
static Halo pold_halo(const mas_op* op, int k) {
    const int par = (k + 1) & 1;
    return op->p2p ? peer_halo(op, op->p[par], op->nb_p[par][0], op->nb_p[par][1])
                   : halo_of(op, op->p[par], op->g->comm ? op->pg[par] : nullptr, op->ncomp);
}
// theta-ghost rows (2-D decomposition): a packed copy, or the theta
// neighbours' own arrays in place (P2P)
static TRows packed_rows(const mas_op* op, const double* buf, int ncomp) {
    TRows t{};
    if (!buf) return t;
    const int nl = op->geo.nl, np = op->geo.np;
    t.lo = op->tlo >= 0 ? buf : nullptr;
    t.hi = op->thi >= 0 ? buf + (long long)ncomp * nl * np : nullptr;
    t.cs_lo = t.cs_hi = nl * np;
    t.ps_lo = t.ps_hi = np;
    return t;
}
static TRows peer_rows(const mas_op* op, const double* lo, const double* hi) {
    TRows t{};
    const int nl = op->geo.nl, np = op->geo.np;
    if (lo) {
        t.lo = lo + (long long)(op->nbt_ntl[0] - 1) * np;  // its last row
        t.ps_lo = op->nbt_ntl[0] * np;
        t.cs_lo = nl * t.ps_lo;
    }
    if (hi) {
        t.hi = hi;  // its first row
        t.ps_hi = op->nbt_ntl[1] * np;
        t.cs_hi = nl * t.ps_hi;
    }
    return t;
}
static TRows r_trows(const mas_op* op) {
    return op->p2p ? peer_rows(op, op->nbt_r[0], op->nbt_r[1]) : packed_rows(op, op->rgt, op->ncomp);
}
static TRows pold_trows(const mas_op* op, int k) {
    const int par = (k + 1) & 1;
    return op->p2p ? peer_rows(op, op->nbt_p[par][0], op->nbt_p[par][1])
                   : packed_rows(op, op->pgt[par], op->ncomp);
}
static bool split_theta(const mas_op* op) { return op->g->ptheta > 1; }

// exchange the first / last theta rows of `field` ([ncomp][nl][nt][np]) with
// the theta neighbours into recv ([2][ncomp][nl][np]); collective
static mas_status_t tseams(mas_op* op, const double* field, int ncomp, double* recv, cudaStream_t s) {
    if (!split_theta(op)) return MAS_OK;
    const size_t n = (size_t)ncomp * op->geo.nl * op->geo.np;
    CU(launch_pack_rows(op->geo, ncomp, field, op->tpack, s));
    return comm_exchange(op->g->comm, op->tlo, op->thi, op->tpack, op->tpack + n, recv, recv + n, n, s);
}
static int rstride(const mas_op* op) { return op->g->ptheta; }

static P2P p2p_args(const mas_op* op) {
    P2P t{};
    if (op->p2p) {
        t.own = op->mbox;
        t.peers = op->d_peers;
        t.nranks = comm_nranks(op->g->comm);
        t.rank = comm_rank(op->g->comm);
    }
    return t;
}

// p_k (= p[k & 1]) with its r-neighbour planes as the L_par kernel reads them:
// in place from the neighbours' arrays (P2P), from the p_k seam buffers (NCCL
// loop, exchanged after kernel A), or none (one GPU)
static Halo aniso_p_halo(const mas_op* op, int k) {
    const int par = k & 1;
    if (op->p2p) return peer_halo(op, op->p[par], op->nb_p[par][0], op->nb_p[par][1]);
    if (op->g->comm) return halo_of(op, op->p[par], op->pkg, 1);
    return Halo{op->p[par], nullptr, nullptr, 0, 0};
}

// r-slabs: the corner plane above the slab is rank+1's plane 0 (ghost copy)
static const double* aniso_ca_hi(const mas_op* op) {
    return (op->cag && !op->geo.glob_hi) ? op->cag + 3 * op->geo.plane : nullptr;
}

// the iteration's L_par runs inside kernel A (k_stencil<PCGA, 1, *, LPAR>)
static bool lpar_in_a(const mas_op* op) { return op->aniso && op->lpar_fused; }
// kernel A's arguments for the fused term (nullptr ca: off)
static void set_lpar_args(const mas_op* op, StencilArgs& a) {
    a.ca = lpar_in_a(op) ? op->ca : nullptr;
    a.ca_hi = lpar_in_a(op) ? aniso_ca_hi(op) : nullptr;
    a.ivr = op->at.ivr;
}

// D (optional) and 1/D: the 7-point diagonal (k_diag), plus the field-aligned
// term's diagonal (R26) when L_par is on (D then goes through a device buffer:
// the caller's, or q, which is free outside a solve).
static mas_status_t op_diag(mas_op* op, double* D_out, cudaStream_t s) {
    double* D = (op->aniso || op->tnode) && !D_out ? op->q : D_out;
    CU(launch_diag(op->geo, halo_of(op, op->kappa, op->kg, 1), packed_rows(op, op->kgt, 1), op->c, D,
                   op->dinv, op->bad, s));
    if (op->aniso) CU(launch_aniso_diag(op->geo, op->ca, aniso_ca_hi(op), D, op->dinv, op->bad, s));
    // theta nodes: a pole row's diagonal is the cap's (the phi average of its
    // slices' diagonals), 1/D from that
    if (op->tnode) CU(launch_pole_avg(op->geo, 1, D, op->dinv, 0, op->geo.nl, s));
    return MAS_OK;
}

// theta nodes: the pole rows of an ncomp-field (all local planes)
static mas_status_t pole_pass(const mas_op* op, double* y, int ncomp, cudaStream_t s) {
    if (op->tnode) CU(launch_pole_avg(op->geo, ncomp, y, nullptr, 0, op->geo.nl, s));
    return MAS_OK;
}

static AnisoArgs aniso_args(const mas_op* op, int mode, Halo u, double* out) {
    AnisoArgs a{};
    a.g = op->geo;
    a.chunk = op->chunk;
    a.max_blocks = op->max_blocks;
    a.ca = op->ca;
    a.ca_hi = aniso_ca_hi(op);
    a.p2p = p2p_args(op);
    a.ivr = op->at.ivr;
    a.u = u;
    a.out = out;
    a.st = op->st;
    a.scr = op->scr;
    (void)mode;
    return a;
}

// copy coefficients in (host or device pointers), compute D and 1/D, exchange
// the static kappa / dinv seams, check the coefficients on the device.
static mas_status_t op_load(mas_op* op, const double* kappa, const double* mass, cudaStream_t s,
                            double* D_out) {
    const size_t bytes = op->Nl * sizeof(double);
    CU(cudaMemcpyAsync(op->kappa, kappa, bytes, cudaMemcpyDefault, s));
    if (mass)
        CU(cudaMemcpyAsync(op->c, mass, bytes, cudaMemcpyDefault, s));
    else
        CU(cudaMemsetAsync(op->c, 0, bytes, s));
    const long long plane = op->geo.plane;
    if (op->g->comm)
        ST(comm_seams(op->g->comm, op->kappa, 1, op->g->nl, plane, op->kg, op->kg + plane, s,
                      rstride(op)));
    ST(tseams(op, op->kappa, 1, op->kgt, s));
    CU(cudaMemsetAsync(op->bad, 0, sizeof(int), s));
    ST(op_diag(op, D_out, s));
    if (op->g->comm)
        ST(comm_seams(op->g->comm, op->dinv, 1, op->g->nl, plane, op->dg, op->dg + plane, s,
                      rstride(op)));
    ST(tseams(op, op->dinv, 1, op->dgt, s));
    int bad = 0;
    CU(cudaMemcpyAsync(&bad, op->bad, sizeof(int), cudaMemcpyDeviceToHost, s));
    CU(cudaStreamSynchronize(s));
    if (op->g->comm) {  // agree on the verdict across ranks
        double* d = op->dot_out;
        double hb = bad;
        CU(cudaMemcpyAsync(d, &hb, sizeof(double), cudaMemcpyHostToDevice, s));
        ST(comm_allreduce(op->g->comm, d, 1, s));
        CU(cudaMemcpyAsync(&hb, d, sizeof(double), cudaMemcpyDeviceToHost, s));
        CU(cudaStreamSynchronize(s));
        bad = hb != 0.0;
    }
    if (bad) return arg_error("kappa/c negative or non-finite, or Jacobi diagonal D <= 0");
    return MAS_OK;
}

static void op_free(mas_op* op) {
    if (!op) return;
    for (double* p : {op->kgt, op->dgt, op->xgt, op->rgt, op->pgt[0], op->pgt[1], op->tpack, op->ca,
                      op->atab, op->cag, op->pkg, op->rs_w, op->rs_out, op->astage, op->r2, op->w2,
                      op->pcg})
        if (p) cudaFree(p);
    if (op->gexec1) cudaGraphExecDestroy(op->gexec1);
    for (double* p : {op->kappa, op->c, op->dinv, op->kg, op->dg, op->wR, op->r, op->p[0], op->p[1],
                      op->q, op->rg, op->pg[0], op->pg[1], op->xg, op->stage_a, op->stage_b,
                      op->hist, op->dot_out, op->scr.partials})
        if (p) cudaFree(p);
    if (op->st) cudaFree(op->st);
    if (op->scr.ticket) cudaFree(op->scr.ticket);
    if (op->bad) cudaFree(op->bad);
    if (op->host_flag) cudaFreeHost(op->host_flag);
    for (auto& e : op->ev)
        if (e) cudaEventDestroy(e);
    for (auto& e : op->pev) cudaEventDestroy(e);
    if (op->gexec) cudaGraphExecDestroy(op->gexec);
    if (op->cs) cudaStreamDestroy(op->cs);
    if (op->ev_ready) cudaEventDestroy(op->ev_ready);
    if (op->ev_seam) cudaEventDestroy(op->ev_seam);
    if (op->cap_stream) cudaStreamDestroy(op->cap_stream);
    for (void* p : op->ipc_opened) cudaIpcCloseMemHandle(p);
    if (op->mbox) cudaFree(op->mbox);
    if (op->d_peers) cudaFree(op->d_peers);
    delete op;
}

static mas_status_t ensure_hist(mas_op* op, int maxit) {
    if (op->hist_cap >= maxit + 2) return MAS_OK;
    if (op->hist) cudaFree(op->hist);
    op->hist = nullptr;
    op->hist_cap = 0;
    ST(dmalloc(&op->hist, 3 * (size_t)(maxit + 2)));
    op->hist_cap = maxit + 2;
    return MAS_OK;
}

static mas_status_t ensure_prof_events(mas_op* op, int k) {
    while (op->pev.size() < 6 * (size_t)k) {
        cudaEvent_t e;
        CU(cudaEventCreate(&e));
        op->pev.push_back(e);
    }
    return MAS_OK;
}

// Build (or reuse) the graph of the whole iteration loop:
//   A(1) [L_par(1)] B(1) -> while (!stopped) { A B A B }   (iterations 2, 3, ...)
// Kernel A of iteration 1 is its own instantiation (FIRSTK), so it sits
// ahead of the while node, in the same graph: one graph launch per solve.
// Kernels read k, alpha, beta and the stop decision from PcgState; the
// deciding kernel's last block sets the while-condition to 0.
// (MAS_GRAPH_PRE=1, an experiment hook, launches iteration 1 as plain
// kernels ahead of a graph holding only the while node, the round-1 form.)
static mas_status_t loop_graph(mas_op* op, StencilArgs a, StreamArgs b, AnisoArgs an, bool pre_plain) {
    const int aniso_key = op->aniso ? (lpar_in_a(op) ? 2 : 1) : 0;
    if (op->gexec && op->g_x == a.x && op->g_hist == a.rho_hist && op->g_aniso == aniso_key &&
        op->g_pre == (int)pre_plain)
        return MAS_OK;
    if (op->gexec) {
        cudaGraphExecDestroy(op->gexec);
        op->gexec = nullptr;
    }
    if (!op->cap_stream) CU(cudaStreamCreateWithFlags(&op->cap_stream, cudaStreamNonBlocking));
    const int nc = op->ncomp;
    cudaGraph_t g;
    CU(cudaGraphCreate(&g, 0));
    cudaError_t e = cudaSuccess;
    std::vector<cudaGraphNode_t> deps;
    if (!pre_plain) {  // iteration 1 into the top-level graph, as a chain of kernel nodes
        e = cudaStreamBeginCaptureToGraph(op->cap_stream, g, nullptr, nullptr, 0,
                                          cudaStreamCaptureModeThreadLocal);
        if (e == cudaSuccess) {
            StencilArgs a1 = a;
            a1.pold = pold_halo(op, 1);  // not read in iteration 1
            a1.tpold = pold_trows(op, 1);
            a1.pnew = op->p[1];
            e = launch_stencil(MODE_PCGA, nc, a1, op->cap_stream, true);
            if (e == cudaSuccess && op->aniso && !lpar_in_a(op)) {
                AnisoArgs an1 = an;
                an1.u = aniso_p_halo(op, 1);
                e = launch_aniso(MODE_PCGA, an1, op->cap_stream);
            }
            // (theta nodes: kernel B does the pole pass on q itself)
            if (e == cudaSuccess) e = launch_pcg_b(b, op->b_blocks, op->cap_stream);
            cudaGraph_t out = g;
            cudaError_t e2 = cudaStreamEndCapture(op->cap_stream, &out);
            if (e == cudaSuccess) e = e2;
        }
        // the chain's leaf (the node no other node depends on) precedes the loop
        size_t n = 0;
        if (e == cudaSuccess) e = cudaGraphGetNodes(g, nullptr, &n);
        std::vector<cudaGraphNode_t> nodes(n);
        if (e == cudaSuccess && n) e = cudaGraphGetNodes(g, nodes.data(), &n);
        for (size_t i = 0; i < n && e == cudaSuccess; i++) {
            size_t nd = 0;
            e = cudaGraphNodeGetDependentNodes(nodes[i], nullptr, &nd);
            if (e == cudaSuccess && nd == 0) deps.push_back(nodes[i]);
        }
        if (e == cudaSuccess && deps.size() != 1) e = cudaErrorInvalidValue;
    }
    cudaGraphConditionalHandle h;
    if (e == cudaSuccess) e = cudaGraphConditionalHandleCreate(&h, g, 1, cudaGraphCondAssignDefault);
    cudaGraphNodeParams p = {};
    p.type = cudaGraphNodeTypeConditional;
    p.conditional.handle = h;
    p.conditional.type = cudaGraphCondTypeWhile;
    p.conditional.size = 1;
    cudaGraphNode_t node;
    if (e == cudaSuccess) e = cudaGraphAddNode(&node, g, deps.data(), deps.size(), &p);
    if (e == cudaSuccess) {
        cudaGraph_t body = p.conditional.phGraph_out[0];
        e = cudaStreamBeginCaptureToGraph(op->cap_stream, body, nullptr, nullptr, 0,
                                          cudaStreamCaptureModeThreadLocal);
        if (e == cudaSuccess) {
            a.cond = (unsigned long long)h;
            b.cond = (unsigned long long)h;
            an.cond = (unsigned long long)h;
            // the body covers an even and an odd iteration: k = 2, 3, 4, ...
            for (int kk = 2; kk <= 3 && e == cudaSuccess; kk++) {
                a.pold = pold_halo(op, kk);
                a.tpold = pold_trows(op, kk);
                a.pnew = op->p[kk & 1];
                e = launch_stencil(MODE_PCGA, nc, a, op->cap_stream);
                an.u = aniso_p_halo(op, kk);
                if (e == cudaSuccess && op->aniso && !lpar_in_a(op)) e = launch_aniso(MODE_PCGA, an, op->cap_stream);
                if (e == cudaSuccess) e = launch_pcg_b(b, op->b_blocks, op->cap_stream);
            }
            cudaGraph_t out = body;
            cudaError_t e2 = cudaStreamEndCapture(op->cap_stream, &out);
            if (e == cudaSuccess) e = e2;
        }
    }
    if (e == cudaSuccess) e = cudaGraphInstantiate(&op->gexec, g, 0);
    cudaGraphDestroy(g);
    if (e != cudaSuccess) {
        cudaGetLastError();
        op->gexec = nullptr;
        set_last_error(std::string("loop graph: ") + cudaGetErrorString(e));
        return MAS_ERR_CUDA;
    }
    op->g_x = a.x;
    op->g_hist = a.rho_hist;
    op->g_aniso = aniso_key;
    op->g_pre = (int)pre_plain;
    return MAS_OK;
}

// ---------------------------------------------------------------------------
// single-reduction PCG (reading R28)
// ---------------------------------------------------------------------------
// kernel k >= 1 of the Chronopoulos-Gear loop: r_{k-1}, w_{k-1}, s_{k-2} in,
// s_{k-1}, r_k, w_k out (ping-pong by parity), p and x in place
// (r-slabs: the three halo fields come with the ghost planes exchanged just
// before the kernel: r -> rg, w -> pg[0], s -> pg[1])
static void cg1_args(const mas_op* op, int k, StencilArgs& a) {
    const int nc = op->ncomp;
    double* R[2] = {op->r, op->r2};
    double* Wb[2] = {op->q, op->w2};
    double* S[2] = {op->p[0], op->p[1]};
    if (op->p2p) {  // the r-neighbours' buffers of the same parity, read in place
        const double* const* nR[2] = {op->nb_r, op->nb_cg[0]};
        const double* const* nW[2] = {op->nb_cg[1], op->nb_cg[2]};
        const int ru = (k - 1) & 1, rs = k & 1;
        a.u = peer_halo(op, R[ru], nR[ru][0], nR[ru][1]);
        a.w = peer_halo(op, Wb[ru], nW[ru][0], nW[ru][1]);
        a.pold = peer_halo(op, S[rs], op->nb_p[rs][0], op->nb_p[rs][1]);
    } else {
        a.u = halo_of(op, R[(k - 1) & 1], op->rg, nc);
        a.w = halo_of(op, Wb[(k - 1) & 1], op->pg[0], nc);
        a.pold = halo_of(op, S[k & 1], op->pg[1], nc);
    }
    a.sout = S[(k - 1) & 1];
    a.rout = R[k & 1];
    a.out = Wb[k & 1];
    a.pnew = op->pcg;
}

// graph: init (w0 = L D^-1 r0) -> while (!stopped) { CG1(k odd), CG1(k even) }
static mas_status_t cg1_graph(mas_op* op, StencilArgs a) {
    if (op->gexec1 && op->g1_x == a.x) return MAS_OK;
    if (op->gexec1) {
        cudaGraphExecDestroy(op->gexec1);
        op->gexec1 = nullptr;
    }
    if (!op->cap_stream) CU(cudaStreamCreateWithFlags(&op->cap_stream, cudaStreamNonBlocking));
    const int nc = op->ncomp;
    cudaGraph_t g;
    CU(cudaGraphCreate(&g, 0));
    cudaError_t e = cudaStreamBeginCaptureToGraph(op->cap_stream, g, nullptr, nullptr, 0,
                                                  cudaStreamCaptureModeThreadLocal);
    if (e == cudaSuccess) {
        StencilArgs a0 = a;
        a0.u = op->p2p ? peer_halo(op, op->r, op->nb_r[0], op->nb_r[1]) : halo_of(op, op->r, nullptr, nc);
        a0.out = op->q;
        e = launch_stencil(MODE_CG1, nc, a0, op->cap_stream, true);
        cudaGraph_t out = g;
        cudaError_t e2 = cudaStreamEndCapture(op->cap_stream, &out);
        if (e == cudaSuccess) e = e2;
    }
    size_t n = 0;
    if (e == cudaSuccess) e = cudaGraphGetNodes(g, nullptr, &n);
    cudaGraphNode_t leaf = nullptr;
    if (e == cudaSuccess && n == 1) e = cudaGraphGetNodes(g, &leaf, &n);
    if (e == cudaSuccess && !leaf) e = cudaErrorInvalidValue;
    cudaGraphConditionalHandle h;
    if (e == cudaSuccess) e = cudaGraphConditionalHandleCreate(&h, g, 1, cudaGraphCondAssignDefault);
    cudaGraphNodeParams p = {};
    p.type = cudaGraphNodeTypeConditional;
    p.conditional.handle = h;
    p.conditional.type = cudaGraphCondTypeWhile;
    p.conditional.size = 1;
    cudaGraphNode_t node;
    if (e == cudaSuccess) e = cudaGraphAddNode(&node, g, &leaf, 1, &p);
    if (e == cudaSuccess) {
        e = cudaStreamBeginCaptureToGraph(op->cap_stream, p.conditional.phGraph_out[0], nullptr, nullptr, 0,
                                          cudaStreamCaptureModeThreadLocal);
        if (e == cudaSuccess) {
            a.cond = (unsigned long long)h;
            for (int k = 1; k <= 2 && e == cudaSuccess; k++) {
                cg1_args(op, k, a);
                e = launch_stencil(MODE_CG1, nc, a, op->cap_stream);
            }
            cudaGraph_t out = p.conditional.phGraph_out[0];
            cudaError_t e2 = cudaStreamEndCapture(op->cap_stream, &out);
            if (e == cudaSuccess) e = e2;
        }
    }
    if (e == cudaSuccess) e = cudaGraphInstantiate(&op->gexec1, g, 0);
    cudaGraphDestroy(g);
    if (e != cudaSuccess) {
        cudaGetLastError();
        op->gexec1 = nullptr;
        set_last_error(std::string("single-reduction loop graph: ") + cudaGetErrorString(e));
        return MAS_ERR_CUDA;
    }
    op->g1_x = a.x;
    return MAS_OK;
}

// the seams kernel k >= 1 reads: r_{k-1}, w_{k-1}, s_{k-2} (NCCL loop on r-slabs)
static mas_status_t cg1_seams(mas_op* op, int k, cudaStream_t s) {
    Comm* comm = op->g->comm;
    if (!comm) return MAS_OK;
    const int nc = op->ncomp;
    const long long plane = op->geo.plane;
    double* R[2] = {op->r, op->r2};
    double* Wb[2] = {op->q, op->w2};
    double* S[2] = {op->p[0], op->p[1]};
    ST(comm_seams(comm, R[(k - 1) & 1], nc, op->g->nl, plane, op->rg, op->rg + nc * plane, s));
    ST(comm_seams(comm, Wb[(k - 1) & 1], nc, op->g->nl, plane, op->pg[0], op->pg[0] + nc * plane, s));
    ST(comm_seams(comm, S[k & 1], nc, op->g->nl, plane, op->pg[1], op->pg[1] + nc * plane, s));
    return MAS_OK;
}

static mas_status_t cg1_solve(mas_op* op, const double* fd, double* xd, double tol, int maxit, int* iters,
                              double* relres, double* res_hist, cudaStream_t s) {
    const int nc = op->ncomp;
    const size_t bytes = nc * op->Nl * sizeof(double);
    Comm* comm = op->g->comm;
    const long long plane = op->geo.plane;
    op->launches = 0;
    const bool p2p = op->p2p != 0;
    PcgState init{};
    if (p2p) init.epoch = ++op->epoch;
    init.tol = tol;
    init.maxit = maxit;
    init.k = 0;
    init.stopped = 0;
    init.status = MAS_NOT_CONVERGED;
    CU(cudaMemcpyAsync(op->st, &init, sizeof(init), cudaMemcpyHostToDevice, s));
    *op->host_flag = 0;
    // kernel 1 reads s_{-1} = p[1] and p_{-1} = pcg with beta_0 = 0: finite zeros
    CU(cudaMemsetAsync(op->p[1], 0, bytes, s));
    CU(cudaMemsetAsync(op->pcg, 0, bytes, s));
    double* rho_h = op->hist;
    double* sig_h = op->hist + op->hist_cap;
    double* rr_h = op->hist + 2 * op->hist_cap;
    StencilArgs a{};
    a.g = op->geo;
    a.chunk = op->chunk;
    a.kappa = halo_of(op, op->kappa, op->kg, 1);
    a.dinv = halo_of(op, op->dinv, op->dg, 1);
    a.c = op->c;
    a.curv = op->curv;
    a.st = op->st;
    a.rho_hist = rho_h;
    a.sigma_hist = sig_h;
    a.rr_hist = rr_h;
    a.scr = op->scr;
    a.host_flag = op->host_flag_dev;
    // P2P transport: every kernel publishes its 3 partial sums to every rank's
    // mailbox and the next one sums them there (no host-side allreduce)
    a.p2p = p2p_args(op);
    // a3: r0 = f - L x0 and <f,f>, <r0,r0> (k_stencil<RESID>, as the standard loop)
    if (comm) ST(comm_seams(comm, xd, nc, op->g->nl, plane, op->xg, op->xg + nc * plane, s));
    StencilArgs r0 = a;
    r0.u = halo_of(op, xd, op->xg, nc);
    r0.f = fd;
    r0.out = op->r;
    if (p2p) ST(comm_vsync(comm, s));  // virtual P2P ranks: every rank's previous solve done
    CU(launch_stencil(MODE_RESID, nc, r0, s));  // (P2P: publishes rho, rr, ff to slot B)
    op->launches++;
    if (comm && !p2p) {  // the init sums over the ranks; r0's edge planes for the init kernel
        ST(comm_allreduce(comm, &op->st->pend_rho, 3, s));  // rho, rr, ff
        ST(comm_seams(comm, op->r, nc, op->g->nl, plane, op->rg, op->rg + nc * plane, s));
    }
    a.x = xd;
    const bool graph = !op->prof && op->use_graph && (!comm || (p2p && !comm_is_virtual(comm)));
    if (graph) {
        ST(cg1_graph(op, a));
        CU(cudaGraphLaunch(op->gexec1, s));
    } else {
        // host-driven: launch n = 1 is the init, n = k + 1 is kernel k; stop
        // enqueueing once the device reports a decision taken by launch <= n-1.
        // Kernel maxit + 1 (launch maxit + 2) takes the maxit decision.
        for (int n = 1; n <= maxit + 2; n++) {
            cudaEvent_t* pe = nullptr;
            if (op->prof) {
                ST(ensure_prof_events(op, n));
                pe = &op->pev[6 * (size_t)(n - 1)];
                CU(cudaEventRecord(pe[0], s));
            }
            // virtual P2P ranks share one GPU: every rank's previous kernel done
            // before a kernel that waits on their mailbox entries is launched
            if (p2p) ST(comm_vsync(comm, s));
            if (n == 1) {
                StencilArgs a0 = a;
                a0.u = p2p ? peer_halo(op, op->r, op->nb_r[0], op->nb_r[1]) : halo_of(op, op->r, op->rg, nc);
                a0.out = op->q;
                CU(launch_stencil(MODE_CG1, nc, a0, s, true));
            } else {
                if (!p2p) ST(cg1_seams(op, n - 1, s));
                if (pe) CU(cudaEventRecord(pe[0], s));
                cg1_args(op, n - 1, a);
                CU(launch_stencil(MODE_CG1, nc, a, s));
            }
            op->launches++;
            if (pe) CU(cudaEventRecord(pe[1], s));
            // the one allreduce of the iteration: (gamma, delta, ||r||^2) in place
            if (comm && !p2p) ST(comm_allreduce(comm, &op->st->pend_sigma, 3, s));
            CU(cudaEventRecord(op->ev[n & 1], s));
            if (n >= 2) {
                ST(comm_wait_event(comm, op->ev[(n - 1) & 1]));
                const int flag = *(volatile int*)op->host_flag;
                if (flag > 0 && flag <= n - 1) break;
            }
        }
    }
    ST(comm_sync_stream(comm, s));
    // P2P: no rank may publish the next solve's partials while another rank's
    // kernels of this solve can still read its mailbox
    if (p2p && comm) ST(comm_barrier(comm, s));
    PcgState fin{};
    CU(cudaMemcpy(&fin, op->st, sizeof(fin), cudaMemcpyDeviceToHost));
    if (!fin.stopped) {
        set_last_error("internal: single-reduction loop ended without a stop decision");
        return MAS_ERR_CUDA;
    }
    *iters = fin.iters;
    *relres = fin.relres;
    if (graph) {  // the init + whole bodies of 2 kernels up to the deciding kernel (iters + 1)
        const int d = fin.status == MAS_ERR_BREAKDOWN && fin.iters == 1 ? 1 : fin.iters + 1;
        op->launches += 1 + 2 * ((d + 1) / 2);
    }
    if (res_hist) {
        const int nh = (fin.status == MAS_ERR_BREAKDOWN && fin.iters == 1) ? 1 : fin.iters + 1;
        std::vector<double> rr(nh);
        CU(cudaMemcpy(rr.data(), rr_h, rr.size() * sizeof(double), cudaMemcpyDeviceToHost));
        for (int k = 0; k < nh; k++) res_hist[k] = std::sqrt(rr[k]);
    }
    if (op->prof) {  // average device time of kernels 1..iters (the init excluded)
        double sa = 0.0;
        int n = 0;
        for (int k = 2; k <= fin.iters + 1 && 6 * (size_t)k <= op->pev.size(); k++, n++) {
            float t = 0.f;
            CU(cudaEventElapsedTime(&t, op->pev[6 * (size_t)(k - 1)], op->pev[6 * (size_t)(k - 1) + 1]));
            sa += t;
        }
        op->prof_a_ms = n ? sa / n : 0.0;
        op->prof_b_ms = 0.0;
        op->prof_c_ms = 0.0;
        op->prof_n = n;
    }
    return (mas_status_t)fin.status;
}

static mas_status_t ensure_stage(mas_op* op) {
    if (op->stage_a) return MAS_OK;
    ST(dmalloc(&op->stage_a, op->ncomp * op->Nl));
    ST(dmalloc(&op->stage_b, op->ncomp * op->Nl));
    return MAS_OK;
}

extern "C" {

mas_status_t mas_op_setup(mas_grid_t* g, int ncomp, const double* kappa, const double* mass,
                          mas_bc_t bc_r_inner, mas_bc_t bc_r_outer, cudaStream_t stream,
                          mas_op_t** out) {
    return mas_op_setup_placed(g, ncomp, MAS_PLACE_CELL, kappa, mass, bc_r_inner, bc_r_outer, stream, out);
}

mas_status_t mas_op_setup_placed(mas_grid_t* g, int ncomp, int placement, const double* kappa,
                                 const double* mass, mas_bc_t bc_r_inner, mas_bc_t bc_r_outer,
                                 cudaStream_t stream, mas_op_t** out) {
    NvtxRange nvtx("mas_op_setup");
    if (!out) return arg_error("null out");
    *out = nullptr;
    if (!g || !kappa) return arg_error("null grid or kappa");
    if (ncomp != 1 && ncomp != 3) return arg_error("ncomp must be 1 or 3");
    if (placement < MAS_PLACE_CELL || placement > MAS_PLACE_PHI_NODE) return arg_error("unknown placement");
    if (placement == MAS_PLACE_THETA_NODE && !g->d_tab_tn)
        return arg_error("theta-node placement needs both pole flags, nt >= 2 and ptheta == 1");
    if (placement == MAS_PLACE_R_NODE && !g->d_tab_rn)
        return arg_error("r-node placement needs one rank and nr >= 2");
    if ((bc_r_inner != MAS_BC_DIRICHLET && bc_r_inner != MAS_BC_NEUMANN) ||
        (bc_r_outer != MAS_BC_DIRICHLET && bc_r_outer != MAS_BC_NEUMANN))
        return arg_error("bad boundary condition");
    mas_op* op = new (std::nothrow) mas_op();
    if (!op) return MAS_ERR_NOMEM;
    op->g = g;
    op->ncomp = ncomp;
    op->bci = bc_r_inner;
    op->bco = bc_r_outer;
    op->tnode = placement == MAS_PLACE_THETA_NODE;
    op->placement = placement;
    // local block [nl][ntl][np]; theta nodes: [nl][nt+1][np]; r nodes: [nr-1][nt][np]
    const int nl = placement == MAS_PLACE_R_NODE ? g->nr - 1 : g->nl;
    const int nt = op->tnode ? g->nt + 1 : g->ntl, np = g->np;
    // this block holds the global outer r-boundary (r nodes: one rank, always)
    const bool owns_top = placement == MAS_PLACE_R_NODE || g->i0 + g->nl == g->nr;
    const long long plane = (long long)nt * np;
    op->Nl = (long long)nl * plane;
    if ((long long)ncomp * op->Nl >= (1LL << 31)) {  // the stencil kernels index with 32-bit offsets
        delete op;
        return arg_error("local slab too large: ncomp * cells must be < 2^31 per rank");
    }
    const bool multi = g->comm != nullptr;
    mas_status_t s;
#define TRY(x)                         \
    do {                               \
        s = (x);                       \
        if (s != MAS_OK) {             \
            op_free(op);               \
            return s;                  \
        }                              \
    } while (0)
    TRY(dmalloc(&op->kappa, op->Nl));
    TRY(dmalloc(&op->c, op->Nl));
    TRY(dmalloc(&op->dinv, op->Nl));
    TRY(dmalloc(&op->wR, 2 * (size_t)nl));
    TRY(dmalloc(&op->r, ncomp * op->Nl));
    TRY(dmalloc(&op->p[0], ncomp * op->Nl));
    TRY(dmalloc(&op->p[1], ncomp * op->Nl));
    TRY(dmalloc(&op->q, ncomp * op->Nl));
    if (multi) {
        TRY(dmalloc(&op->kg, 2 * plane));
        TRY(dmalloc(&op->dg, 2 * plane));
        TRY(dmalloc(&op->rg, 2 * ncomp * plane));
        TRY(dmalloc(&op->pg[0], 2 * ncomp * plane));
        TRY(dmalloc(&op->pg[1], 2 * ncomp * plane));
        TRY(dmalloc(&op->xg, 2 * ncomp * plane));
    }
    if (g->ptheta > 1) {  // theta neighbours: rank -/+ 1 within the same r-slab
        op->tlo = g->trank > 0 ? g->rank - 1 : -1;
        op->thi = g->trank < g->ptheta - 1 ? g->rank + 1 : -1;
        const size_t rows = (size_t)nl * np;
        TRY(dmalloc(&op->kgt, 2 * rows));
        TRY(dmalloc(&op->dgt, 2 * rows));
        TRY(dmalloc(&op->xgt, 2 * ncomp * rows));
        TRY(dmalloc(&op->rgt, 2 * ncomp * rows));
        TRY(dmalloc(&op->pgt[0], 2 * ncomp * rows));
        TRY(dmalloc(&op->pgt[1], 2 * ncomp * rows));
        TRY(dmalloc(&op->tpack, 2 * ncomp * rows));
    }
    TRY(dmalloc(&op->st, 1));
    TRY(dmalloc(&op->dot_out, 1));
    TRY(dmalloc(&op->bad, 1));
    TRY(ensure_hist(op, 64));
    if (multi && (cudaStreamCreateWithFlags(&op->cs, cudaStreamNonBlocking) != cudaSuccess ||
                  cudaEventCreateWithFlags(&op->ev_ready, cudaEventDisableTiming) != cudaSuccess ||
                  cudaEventCreateWithFlags(&op->ev_seam, cudaEventDisableTiming) != cudaSuccess)) {
        cudaGetLastError();
        op_free(op);
        set_last_error("comm stream setup failed");
        return MAS_ERR_CUDA;
    }
    // geometry with the boundary conditions folded into the radial tables:
    // a Neumann face gets weight 0; a Dirichlet face keeps its weight and the
    // kernels use kappa_ghost = kappa_P, u_ghost = 0 (R3).
    {
        std::vector<double> w(2 * nl);
        const bool rn = placement == MAS_PLACE_R_NODE;  // r nodes: the rnode_tables weights
        for (int il = 0; il < nl; il++) {
            w[il] = rn ? g->rn_host[il] : g->tab.wRm[il];
            w[nl + il] = rn ? g->rn_host[nl + il] : g->tab.wRp[il];
        }
        if (g->i0 == 0 && bc_r_inner == MAS_BC_NEUMANN) w[0] = 0.0;
        if (owns_top && bc_r_outer == MAS_BC_NEUMANN) w[2 * nl - 1] = 0.0;
        if (cudaMemcpy(op->wR, w.data(), w.size() * sizeof(double), cudaMemcpyHostToDevice) !=
            cudaSuccess) {
            op_free(op);
            set_last_error("cudaMemcpy wR");
            return MAS_ERR_CUDA;
        }
    }
    Geo& G = op->geo;
    G.nl = nl; G.nt = nt; G.np = np; G.plane = plane;
    G.glob_lo = g->i0 == 0;
    G.glob_hi = owns_top;
    G.wRm = op->wR;
    G.wRp = op->wR + nl;
    const double* t = g->d_tab;  // the grid's (cell-centred) tables: [irc2 vr](g->nl) [theta](ntl) [phi](np)
    G.irc2 = t; t += g->nl;
    G.vr = t; t += g->nl;
    G.wTm = t; t += g->ntl;
    G.wTp = t; t += g->ntl;
    G.isc2 = t; t += g->ntl;
    G.vt = t; t += g->ntl;
    if (op->tnode) {  // the theta part of the geometry: the theta-node rows (NEXT-2)
        G.wTm = g->d_tab_tn;
        G.wTp = g->d_tab_tn + nt;
        G.isc2 = g->d_tab_tn + 2 * nt;
        G.vt = g->d_tab_tn + 3 * nt;
    }
    if (placement == MAS_PLACE_R_NODE) {  // the dual r cells (NEXT-2, R32); wR above
        G.irc2 = g->d_tab_rn + 2 * nl;
        G.vr = g->d_tab_rn + 3 * nl;
    }
    G.wPm = t; t += np;
    G.wPp = t; t += np;
    G.vp = t;
    if (placement == MAS_PLACE_PHI_NODE) {  // the dual phi cells (NEXT-2, R33)
        G.wPm = g->d_tab_pn;
        G.wPp = g->d_tab_pn + np;
        G.vp = g->d_tab_pn + 2 * np;
    }
    const char* g_env = getenv("MAS_NO_GRAPH");  // experiment hook: host-driven loop
    op->use_graph = !(g_env && atoi(g_env));
    const char* gp_env = getenv("MAS_GRAPH_PRE");  // experiment hook (round-1 graph form)
    op->graph_pre = gp_env && atoi(gp_env);
    // experiment hook: the iteration's L_par inside kernel A (correct, but
    // measured slower than the separate k_aniso: profiles/README.md r3l)
    const char* lf_env = getenv("MAS_LPAR_FUSED");
    op->lpar_fused = lf_env && atoi(lf_env) == 1;
    const char* ch_env = getenv("MAS_CHUNK");  // experiment hook
    op->chunk = ch_env ? atoi(ch_env) : (nl >= 128 ? 32 : nl >= 64 ? 16 : (nl >= 16 ? 8 : 4));
    if (!ch_env && multi && nl >= 12) {
        // at least 3 chunks so that the interior ones can overlap the seams
        op->chunk = nl / 4 < 4 ? 4 : (nl / 4 > 32 ? 32 : nl / 4);
    }
    if (op->chunk < 1 || op->chunk > 64) op->chunk = 16;
    op->max_blocks = stencil_blocks(G, op->chunk);
    const char* bb_env = getenv("MAS_BBLOCKS");  // experiment hook
    // kernel B: 4 blocks per SM (a sweep over 3..8 per SM: 4 and 8 are best at
    // C3, 4 is 13% faster than 8 at C2, profiles/README.md r1g)
    int sms = 148, dev = 0;
    if (cudaGetDevice(&dev) == cudaSuccess)
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    if (sms <= 0) sms = 148;
    op->b_blocks = bb_env ? atoi(bb_env) : 4 * sms;
    if (op->b_blocks > op->max_blocks) op->max_blocks = op->b_blocks;
    TRY(dmalloc(&op->scr.partials, 4 * (size_t)op->max_blocks));
    TRY(dmalloc(&op->scr.ticket, 8));
    if (cudaMemset(op->scr.ticket, 0, 8 * sizeof(unsigned)) != cudaSuccess ||
        cudaHostAlloc(reinterpret_cast<void**>(&op->host_flag), sizeof(int), cudaHostAllocMapped) !=
            cudaSuccess ||
        cudaHostGetDevicePointer(reinterpret_cast<void**>(&op->host_flag_dev), op->host_flag, 0) !=
            cudaSuccess ||
        cudaEventCreateWithFlags(&op->ev[0], cudaEventDisableTiming) != cudaSuccess ||
        cudaEventCreateWithFlags(&op->ev[1], cudaEventDisableTiming) != cudaSuccess) {
        cudaGetLastError();
        op_free(op);
        set_last_error("device scratch setup failed");
        return MAS_ERR_CUDA;
    }
    TRY(op_load(op, kappa, mass, stream, nullptr));
#undef TRY
    *out = op;
    return MAS_OK;
}

mas_status_t mas_op_update(mas_op_t* op, const double* kappa, const double* mass,
                           cudaStream_t stream) {
    NvtxRange nvtx("mas_op_update");
    if (!op || !kappa) return arg_error("null op or kappa");
    return op_load(op, kappa, mass, stream, nullptr);
}

mas_status_t mas_op_diag(const mas_op_t* op_c, double* D, cudaStream_t stream) {
    mas_op* op = const_cast<mas_op*>(op_c);
    if (!op || !D) return arg_error("null argument");
    double* Dd = D;
    const bool host = !is_device_ptr(D);
    if (host) {
        ST(ensure_stage(op));
        Dd = op->stage_b;
    }
    CU(cudaMemsetAsync(op->bad, 0, sizeof(int), stream));
    ST(op_diag(op, Dd, stream));
    if (host) {
        CU(cudaMemcpyAsync(D, Dd, op->Nl * sizeof(double), cudaMemcpyDeviceToHost, stream));
        CU(cudaStreamSynchronize(stream));
    }
    return MAS_OK;
}

mas_status_t mas_op_apply(const mas_op_t* op_c, const double* x, double* y, cudaStream_t stream) {
    mas_op* op = const_cast<mas_op*>(op_c);
    if (!op || !x || !y) return arg_error("null argument");
    const size_t bytes = op->ncomp * op->Nl * sizeof(double);
    const double* xd = x;
    double* yd = y;
    const bool hx = !is_device_ptr(x), hy = !is_device_ptr(y);
    if (hx || hy) ST(ensure_stage(op));
    if (hx) {
        CU(cudaMemcpyAsync(op->stage_a, x, bytes, cudaMemcpyHostToDevice, stream));
        xd = op->stage_a;
    }
    if (hy) yd = op->stage_b;
    const long long plane = op->geo.plane;
    if (op->g->comm)
        ST(comm_seams(op->g->comm, xd, op->ncomp, op->g->nl, plane, op->xg,
                      op->xg + op->ncomp * plane, stream, rstride(op)));
    ST(tseams(op, xd, op->ncomp, op->xgt, stream));
    StencilArgs a{};
    a.g = op->geo;
    a.chunk = op->chunk;
    a.u = halo_of(op, xd, op->xg, op->ncomp);
    a.kappa = halo_of(op, op->kappa, op->kg, 1);
    a.tu = packed_rows(op, op->xgt, op->ncomp);
    a.tkappa = packed_rows(op, op->kgt, 1);
    a.c = op->c;
    a.curv = op->curv;
    a.out = yd;
    a.scr = op->scr;
    CU(launch_stencil(MODE_APPLY, op->ncomp, a, stream));
    if (op->aniso)
        CU(launch_aniso(MODE_APPLY, aniso_args(op, MODE_APPLY, halo_of(op, xd, op->xg, 1), yd), stream));
    ST(pole_pass(op, yd, op->ncomp, stream));
    if (hy) {
        CU(cudaMemcpyAsync(y, yd, bytes, cudaMemcpyDeviceToHost, stream));
        CU(cudaStreamSynchronize(stream));
    }
    return MAS_OK;
}

mas_status_t mas_op_dirichlet_rhs(const mas_op_t* op_c, const double* ub_inner,
                                  const double* ub_outer, double* f_inout, cudaStream_t stream) {
    mas_op* op = const_cast<mas_op*>(op_c);
    if (!op || !f_inout) return arg_error("null argument");
    const long long plane = op->geo.plane;
    const size_t fbytes = op->ncomp * op->Nl * sizeof(double);
    const size_t bbytes = op->ncomp * plane * sizeof(double);
    const bool hf = !is_device_ptr(f_inout);
    if (hf) ST(ensure_stage(op));
    double* fd = hf ? op->stage_a : f_inout;
    if (hf) CU(cudaMemcpyAsync(fd, f_inout, fbytes, cudaMemcpyHostToDevice, stream));
    double* ubuf = nullptr;
    for (int side = 0; side < 2; side++) {
        const double* ub = side ? ub_outer : ub_inner;
        const bool owns = side ? op->geo.glob_hi : op->geo.glob_lo;
        const bool dir = (side ? op->bco : op->bci) == MAS_BC_DIRICHLET;
        if (!ub || !owns || !dir) continue;
        const double* ubd = ub;
        if (!is_device_ptr(ub)) {
            if (!ubuf) ST(dmalloc(&ubuf, op->ncomp * plane));
            CU(cudaMemcpyAsync(ubuf, ub, bbytes, cudaMemcpyHostToDevice, stream));
            ubd = ubuf;
        }
        CU(launch_dirichlet(op->geo, op->ncomp, op->kappa, ubd, side, fd, stream));
        if (op->tnode)  // the cap's boundary term: phi average over the pole row's slices
            CU(launch_pole_avg(op->geo, op->ncomp, fd, nullptr, side ? op->geo.nl - 1 : 0, 1, stream));
    }
    if (hf) CU(cudaMemcpyAsync(f_inout, fd, fbytes, cudaMemcpyDeviceToHost, stream));
    if (ubuf || hf) CU(cudaStreamSynchronize(stream));
    if (ubuf) cudaFree(ubuf);
    return MAS_OK;
}

mas_status_t mas_op_dot(const mas_op_t* op_c, const double* a, const double* b, double* out,
                        cudaStream_t stream) {
    mas_op* op = const_cast<mas_op*>(op_c);
    if (!op || !a || !b || !out) return arg_error("null argument");
    const size_t bytes = op->ncomp * op->Nl * sizeof(double);
    const double *ad = a, *bd = b;
    if (!is_device_ptr(a) || !is_device_ptr(b)) {
        ST(ensure_stage(op));
        if (!is_device_ptr(a)) {
            CU(cudaMemcpyAsync(op->stage_a, a, bytes, cudaMemcpyHostToDevice, stream));
            ad = op->stage_a;
        }
        if (!is_device_ptr(b)) {
            CU(cudaMemcpyAsync(op->stage_b, b, bytes, cudaMemcpyHostToDevice, stream));
            bd = op->stage_b;
        }
    }
    CU(launch_dot(op->geo, op->ncomp, ad, bd, op->scr, op->dot_out, op->b_blocks, stream));
    if (op->g->comm) ST(comm_allreduce(op->g->comm, op->dot_out, 1, stream));
    CU(cudaMemcpyAsync(out, op->dot_out, sizeof(double), cudaMemcpyDeviceToHost, stream));
    CU(cudaStreamSynchronize(stream));
    return MAS_OK;
}

mas_status_t mas_op_radial_sums(const mas_op_t* op_c, const double* x, const double* w, double* out,
                                cudaStream_t stream) {
    mas_op* op = const_cast<mas_op*>(op_c);
    if (!op || !x || !w || !out) return arg_error("null argument");
    if (op->g->ptheta > 1) return arg_error("radial sums: r-slab decompositions only (ptheta == 1)");
    const size_t plane = (size_t)op->geo.plane;
    const size_t nout = (size_t)op->ncomp * op->g->nl;
    const double *xd = x, *wd = w;
    if (!is_device_ptr(x)) {
        ST(ensure_stage(op));
        CU(cudaMemcpyAsync(op->stage_a, x, op->ncomp * op->Nl * sizeof(double), cudaMemcpyHostToDevice,
                           stream));
        xd = op->stage_a;
    }
    if (!is_device_ptr(w)) {
        if (!op->rs_w) ST(dmalloc(&op->rs_w, plane));
        CU(cudaMemcpyAsync(op->rs_w, w, plane * sizeof(double), cudaMemcpyHostToDevice, stream));
        wd = op->rs_w;
    }
    const bool hout = !is_device_ptr(out);
    double* od = out;
    if (hout) {
        if (!op->rs_out) ST(dmalloc(&op->rs_out, nout));
        od = op->rs_out;
    }
    CU(launch_radial_sums(op->geo, op->ncomp, xd, wd, od, stream));
    if (hout) {
        CU(cudaMemcpyAsync(out, od, nout * sizeof(double), cudaMemcpyDeviceToHost, stream));
        CU(cudaStreamSynchronize(stream));
    }
    return MAS_OK;
}

// Collective: switch the iteration loop of this op to the P2P transport.
// Every rank exports (CUDA IPC) its r, p[0], p[1] and mailbox; the records
// are all-gathered once; each rank maps its r-neighbours' r / p arrays and
// every rank's mailbox.  Virtual ranks (one process) share raw pointers.
mas_status_t mas_op_enable_p2p(mas_op_t* op, cudaStream_t s) {
    if (!op) return arg_error("null op");
    if (op->p2p) return MAS_OK;
    if (op->placement != MAS_PLACE_CELL)
        return arg_error("P2P transport: cell-centred placement only (the other placements keep NCCL)");
    if (op->cg1 && op->g->ptheta > 1) return arg_error("P2P transport with single reduction: r-slabs only");
    Comm* comm = op->g->comm;
    const int P = comm_nranks(comm), rank = comm_rank(comm);
    const bool virt = comm_is_virtual(comm);
    ST(dmalloc(&op->mbox, MB_SLOTS * (size_t)P));
    CU(cudaMemset(op->mbox, 0, MB_SLOTS * (size_t)P * sizeof(Mail)));
    struct Rec {
        cudaIpcMemHandle_t h[7];
        unsigned long long raw[7];
        int nl, ntl;
        int ok;
    };
    Rec mine;
    memset(&mine, 0, sizeof(mine));
    // r, p[0], p[1], the mailbox; with the single-reduction loop on also its
    // ping-pong buffers r2, w = q, w2 (r-neighbours' halos read in place)
    const bool cg = op->cg1 != 0;
    const void* bufs[7] = {op->r, op->p[0], op->p[1], op->mbox, cg ? op->r2 : nullptr, cg ? op->q : nullptr,
                           cg ? op->w2 : nullptr};
    mine.nl = op->g->nl;
    mine.ntl = op->g->ntl;
    mine.ok = 1;
    for (int b = 0; b < 7; b++) {
        if (!bufs[b]) continue;
        mine.raw[b] = (unsigned long long)(uintptr_t)bufs[b];
        if (P > 1 && !virt && cudaIpcGetMemHandle(&mine.h[b], const_cast<void*>(bufs[b])) != cudaSuccess) {
            cudaGetLastError();
            mine.ok = 0;
        }
    }
    std::vector<Rec> all(P);
    ST(comm_allgather_bytes(comm, &mine, all.data(), sizeof(Rec), s));
    bool ok = true;
    for (int q = 0; q < P; q++) ok = ok && all[q].ok;
    std::string why = ok ? "" : "cudaIpcGetMemHandle failed on some rank";
    auto map = [&](int q, int b) -> void* {
        if (q == rank || virt) return (void*)(uintptr_t)all[q].raw[b];
        void* p = nullptr;
        if (cudaIpcOpenMemHandle(&p, all[q].h[b], cudaIpcMemLazyEnablePeerAccess) != cudaSuccess) {
            why = std::string("cudaIpcOpenMemHandle: ") + cudaGetErrorString(cudaGetLastError());
            ok = false;
            return nullptr;
        }
        op->ipc_opened.push_back(p);
        return p;
    };
    std::vector<Mail*> peers(P, nullptr);
    for (int q = 0; q < P && ok; q++) peers[q] = (Mail*)map(q, 3);
    const int pt = op->g->ptheta;
    for (int side = 0; side < 2 && ok; side++) {  // r-neighbours: rank -/+ ptheta
        const int q = side == 0 ? rank - pt : rank + pt;
        if (q < 0 || q >= P) continue;
        op->nb_r[side] = (const double*)map(q, 0);
        op->nb_p[0][side] = (const double*)map(q, 1);
        op->nb_p[1][side] = (const double*)map(q, 2);
        op->nb_nl[side] = all[q].nl;
        for (int b = 0; b < 3 && cg && ok; b++) op->nb_cg[b][side] = (const double*)map(q, 4 + b);
    }
    for (int side = 0; side < 2 && ok; side++) {  // theta neighbours (same r-slab)
        const int q = side == 0 ? op->tlo : op->thi;
        if (q < 0) continue;
        op->nbt_r[side] = (const double*)map(q, 0);
        op->nbt_p[0][side] = (const double*)map(q, 1);
        op->nbt_p[1][side] = (const double*)map(q, 2);
        op->nbt_ntl[side] = all[q].ntl;
    }
    if (ok && dmalloc(&op->d_peers, (size_t)P) == MAS_OK &&
        cudaMemcpy(op->d_peers, peers.data(), P * sizeof(Mail*), cudaMemcpyHostToDevice) != cudaSuccess) {
        cudaGetLastError();
        ok = false;
        why = "peer table copy";
    }
    if (comm && P > 1) {  // every rank adopts the transport, or none does
        double* d = op->dot_out;
        double flag = ok ? 0.0 : 1.0;
        CU(cudaMemcpyAsync(d, &flag, sizeof(double), cudaMemcpyHostToDevice, s));
        ST(comm_allreduce(comm, d, 1, s));
        CU(cudaMemcpyAsync(&flag, d, sizeof(double), cudaMemcpyDeviceToHost, s));
        CU(cudaStreamSynchronize(s));
        if (flag != 0.0 && ok) {
            ok = false;
            why = "P2P setup failed on another rank";
        }
    }
    if (!ok) {
        for (void* p : op->ipc_opened) cudaIpcCloseMemHandle(p);
        op->ipc_opened.clear();
        cudaFree(op->mbox);
        op->mbox = nullptr;
        if (op->d_peers) cudaFree(op->d_peers);
        op->d_peers = nullptr;
        op->nb_r[0] = op->nb_r[1] = nullptr;
        op->nbt_r[0] = op->nbt_r[1] = nullptr;
        op->nbt_p[0][0] = op->nbt_p[0][1] = op->nbt_p[1][0] = op->nbt_p[1][1] = nullptr;
        op->nb_p[0][0] = op->nb_p[0][1] = op->nb_p[1][0] = op->nb_p[1][1] = nullptr;
        for (auto& v : op->nb_cg) v[0] = v[1] = nullptr;
        set_last_error("P2P transport unavailable: " + why);
        return MAS_ERR_CUDA;
    }
    op->p2p = 1;
    op->p2p_cg1 = cg ? 1 : 0;
    if (op->gexec) {  // the loop graph reads the ghost planes differently now
        cudaGraphExecDestroy(op->gexec);
        op->gexec = nullptr;
    }
    if (op->gexec1) {
        cudaGraphExecDestroy(op->gexec1);
        op->gexec1 = nullptr;
    }
    return MAS_OK;
}

int mas_op_transport(const mas_op_t* op) { return !op ? -1 : op->p2p ? 1 : 0; }

mas_status_t mas_op_set_single_reduction(mas_op_t* op, int on) {
    if (!op) return arg_error("null op");
    if (!on) {
        op->cg1 = 0;
        return MAS_OK;
    }
    if (op->p2p && !op->p2p_cg1)
        return arg_error("single-reduction PCG over the P2P transport: switch it on before mas_op_enable_p2p");
    if (op->g->ptheta > 1) return arg_error("single-reduction PCG: r-slab decompositions only (ptheta == 1)");
    if (op->aniso) return arg_error("single-reduction PCG: isotropic operator only (no mas_op_set_aniso)");
    if (op->placement != MAS_PLACE_CELL) return arg_error("single-reduction PCG: cell-centred placement only");
    if (op->curv) return arg_error("single-reduction PCG: without the curvature terms");
    const size_t n = op->ncomp * (size_t)op->Nl;
    if (!op->r2) ST(dmalloc(&op->r2, n));
    if (!op->w2) ST(dmalloc(&op->w2, n));
    if (!op->pcg) ST(dmalloc(&op->pcg, n));
    op->cg1 = 1;
    return MAS_OK;
}

int mas_op_single_reduction(const mas_op_t* op) { return op ? op->cg1 : -1; }

int mas_op_aniso_fused(const mas_op_t* op) { return !op ? -1 : lpar_in_a(op) ? 1 : 0; }

// Kernel-replay timing: reps launches of one kernel captured in a CUDA graph,
// each preceded by an L2 flush (a read-only sweep over twice the L2 size) and a
// reset of the PCG state to a mid-solve iteration.  A second graph holds the
// flushes and resets alone; the time per launch is the difference of the two
// graphs' event-timed durations over reps (device time, cold L2, no host
// dispatch between launches).
static mas_status_t time_graph(cudaStream_t cap, cudaStream_t s, int reps, void* flush, size_t flush_bytes,
                               PcgState* st, const PcgState* st_init,
                               const std::function<cudaError_t(cudaStream_t)>* launch, float* ms) {
    cudaGraph_t g;
    cudaError_t e = cudaStreamBeginCapture(cap, cudaStreamCaptureModeThreadLocal);
    for (int i = 0; i < reps && e == cudaSuccess; i++) {
        e = launch_l2_sweep(static_cast<const double*>(flush), (long long)(flush_bytes / sizeof(double)),
                            static_cast<double*>(flush), cap);
        if (e == cudaSuccess) e = cudaMemcpyAsync(st, st_init, sizeof(PcgState), cudaMemcpyDeviceToDevice, cap);
        if (e == cudaSuccess && launch) e = (*launch)(cap);
    }
    cudaError_t e2 = cudaStreamEndCapture(cap, &g);
    if (e != cudaSuccess || e2 != cudaSuccess) {
        if (e2 == cudaSuccess) cudaGraphDestroy(g);
        cudaGetLastError();
        set_last_error(std::string("kernel replay capture: ") + cudaGetErrorString(e != cudaSuccess ? e : e2));
        return MAS_ERR_CUDA;
    }
    cudaGraphExec_t ge;
    e = cudaGraphInstantiate(&ge, g, 0);
    cudaGraphDestroy(g);
    if (e != cudaSuccess) {
        cudaGetLastError();
        set_last_error(std::string("kernel replay instantiate: ") + cudaGetErrorString(e));
        return MAS_ERR_CUDA;
    }
    cudaEvent_t e0 = nullptr, e1 = nullptr;
    e = cudaEventCreate(&e0);
    if (e == cudaSuccess) e = cudaEventCreate(&e1);
    if (e == cudaSuccess) e = cudaGraphLaunch(ge, s);  // warm-up
    if (e == cudaSuccess) e = cudaEventRecord(e0, s);
    if (e == cudaSuccess) e = cudaGraphLaunch(ge, s);
    if (e == cudaSuccess) e = cudaEventRecord(e1, s);
    if (e == cudaSuccess) e = cudaEventSynchronize(e1);
    if (e == cudaSuccess) e = cudaEventElapsedTime(ms, e0, e1);
    if (e0) cudaEventDestroy(e0);
    if (e1) cudaEventDestroy(e1);
    cudaGraphExecDestroy(ge);
    if (e != cudaSuccess) {
        cudaGetLastError();
        set_last_error(std::string("kernel replay: ") + cudaGetErrorString(e));
        return MAS_ERR_CUDA;
    }
    return MAS_OK;
}

static mas_status_t replay_time(cudaStream_t cap, cudaStream_t s, int reps, double* ms, void* flush,
                                size_t flush_bytes, PcgState* st, const PcgState* st_init,
                                const std::function<cudaError_t(cudaStream_t)>& launch) {
    float with = 0.f, without = 0.f;
    ST(time_graph(cap, s, reps, flush, flush_bytes, st, st_init, &launch, &with));
    ST(time_graph(cap, s, reps, flush, flush_bytes, st, st_init, nullptr, &without));
    *ms = (double)(with - without) / reps;
    return MAS_OK;
}

mas_status_t mas_op_kernel_bench(mas_op_t* op, int reps, double* a_ms, double* b_ms, double* c_ms,
                                 cudaStream_t s) {
    if (!op || !a_ms || !b_ms || !c_ms || reps < 1) return arg_error("bad argument");
    if (op->g->comm) return arg_error("kernel replay timing: one GPU (no mas_dist_t)");
    *a_ms = *b_ms = *c_ms = 0.0;
    const int nc = op->ncomp;
    const long long n = nc * op->Nl;
    ST(ensure_stage(op));
    ST(ensure_hist(op, 2 * reps + 8));
    if (op->cg1) {
        if (!op->r2) return arg_error("single-reduction buffers missing");
    }
    for (double* v : {op->r, op->p[0], op->p[1], op->q}) CU(launch_fill_test(v, n, s));
    if (op->cg1)
        for (double* v : {op->r2, op->w2, op->pcg}) CU(launch_fill_test(v, n, s));
    CU(cudaMemsetAsync(op->stage_b, 0, n * sizeof(double), s));
    // the PCG state every replay starts from: iteration 2, tol 0, no stop
    // (for the single-reduction kernel: delta - beta gamma / alpha = 2 - 1 > 0)
    PcgState init{};
    init.tol = 0.0;
    init.maxit = 1 << 30;
    init.k = 2;
    init.pend_rho = init.rho_prev = init.sigma_prev = init.pend_rr = init.pend_ff = 1.0;
    init.pend_sigma = 2.0;
    init.cg_alpha = init.cg_gamma = 1.0;
    init.status = MAS_NOT_CONVERGED;
    PcgState* st_init = nullptr;
    ST(dmalloc(reinterpret_cast<double**>(&st_init), (sizeof(PcgState) + 7) / 8));
    void* flush = nullptr;
    int l2 = 0, dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, dev);
    const size_t flush_bytes = 2 * (size_t)(l2 > 0 ? l2 : 128 << 20);
    if (cudaMalloc(&flush, flush_bytes) != cudaSuccess) {
        cudaGetLastError();
        cudaFree(st_init);
        set_last_error("kernel replay: flush buffer");
        return MAS_ERR_NOMEM;
    }
    struct Free {
        void* a;
        void* b;
        ~Free() {
            cudaFree(a);
            cudaFree(b);
        }
    } free_on_exit{flush, st_init};
    CU(cudaMemcpyAsync(st_init, &init, sizeof(init), cudaMemcpyHostToDevice, s));
    CU(cudaMemsetAsync(flush, 0, flush_bytes, s));  // the sweep reads zeros
    if (!op->cap_stream) CU(cudaStreamCreateWithFlags(&op->cap_stream, cudaStreamNonBlocking));
    CU(cudaStreamSynchronize(s));
    StencilArgs a{};
    a.g = op->geo;
    a.chunk = op->chunk;
    a.kappa = halo_of(op, op->kappa, nullptr, 1);
    a.dinv = halo_of(op, op->dinv, nullptr, 1);
    a.c = op->c;
    a.curv = op->curv;
    a.st = op->st;
    a.rho_hist = op->hist;
    a.sigma_hist = op->hist + op->hist_cap;
    a.rr_hist = op->hist + 2 * op->hist_cap;
    a.scr = op->scr;
    a.x = op->stage_b;
    if (op->cg1) {  // the single-reduction kernel, iteration 2
        cg1_args(op, 2, a);
        ST(replay_time(op->cap_stream, s, reps, a_ms, flush, flush_bytes, op->st, st_init,
                       [&](cudaStream_t cs) { return launch_stencil(MODE_CG1, nc, a, cs); }));
        return MAS_OK;
    }
    a.u = halo_of(op, op->r, nullptr, nc);
    a.pold = halo_of(op, op->p[1], nullptr, nc);
    a.pnew = op->p[0];
    a.out = op->q;
    set_lpar_args(op, a);
    ST(replay_time(op->cap_stream, s, reps, a_ms, flush, flush_bytes, op->st, st_init,
                   [&](cudaStream_t cs) { return launch_stencil(MODE_PCGA, nc, a, cs); }));
    if (op->aniso && !lpar_in_a(op)) {
        AnisoArgs an = aniso_args(op, MODE_PCGA, Halo{op->p[0], nullptr, nullptr, 0, 0}, op->q);
        ST(replay_time(op->cap_stream, s, reps, c_ms, flush, flush_bytes, op->st, st_init,
                       [&](cudaStream_t cs) { return launch_aniso(MODE_PCGA, an, cs); }));
    }
    StreamArgs b{};
    b.g = op->geo;
    b.ncomp = nc;
    b.r = op->r;
    b.q = op->q;
    b.dinv = op->dinv;
    b.tnode = op->tnode;
    b.st = op->st;
    b.rho_hist = a.rho_hist;
    b.sigma_hist = a.sigma_hist;
    b.rr_hist = a.rr_hist;
    b.scr = op->scr;
    ST(replay_time(op->cap_stream, s, reps, b_ms, flush, flush_bytes, op->st, st_init,
                   [&](cudaStream_t cs) { return launch_pcg_b(b, op->b_blocks, cs); }));
    return MAS_OK;
}

mas_status_t mas_op_set_curvature(mas_op_t* op, int on) {
    if (!op) return arg_error("null op");
    if (on && op->ncomp != 3) return arg_error("curvature terms: the 3-component (viscosity) operator only");
    if (on && op->placement != MAS_PLACE_CELL) return arg_error("curvature terms: cell-centred placement only");
    if (on && op->cg1) return arg_error("curvature terms: the two-kernel loop only (single reduction is on)");
    op->curv = on ? 1 : 0;
    return MAS_OK;
}

mas_status_t mas_op_comm_bench(mas_op_t* op, int reps, double* seam_us, double* allreduce_us,
                               double* seam_bytes, cudaStream_t s) {
    if (!op || !seam_us || !allreduce_us || !seam_bytes || reps < 1) return arg_error("bad argument");
    Comm* comm = op->g->comm;
    const int nc = op->ncomp;
    const long long plane = op->geo.plane;
    const int pt = op->g->ptheta;
    const int nb = (comm_rank(comm) - pt >= 0) + (comm_rank(comm) + pt < comm_nranks(comm));
    *seam_bytes = comm ? 2.0 * nb * 2.0 * nc * plane * sizeof(double) : 0.0;  // r and p, sent + received
    *seam_us = *allreduce_us = 0.0;
    if (!comm) return MAS_OK;
    cudaEvent_t e0, e1;
    CU(cudaEventCreate(&e0));
    CU(cudaEventCreate(&e1));
    float ms = 0.f;
    mas_status_t st = MAS_OK;
    // the per-iteration seams of the NCCL loop: r and p_{k-1} edge planes (r-slabs)
    ST(comm_seams(comm, op->r, nc, op->g->nl, plane, op->rg, op->rg + nc * plane, s, rstride(op)));
    CU(cudaEventRecord(e0, s));
    for (int i = 0; i < reps && st == MAS_OK; i++) {
        st = comm_seams(comm, op->r, nc, op->g->nl, plane, op->rg, op->rg + nc * plane, s, rstride(op));
        if (st == MAS_OK)
            st = comm_seams(comm, op->p[0], nc, op->g->nl, plane, op->pg[0], op->pg[0] + nc * plane, s,
                            rstride(op));
    }
    CU(cudaEventRecord(e1, s));
    if (st == MAS_OK) st = comm_sync_stream(comm, s);
    if (st == MAS_OK && cudaEventElapsedTime(&ms, e0, e1) == cudaSuccess) *seam_us = 1e3 * ms / reps;
    // the 2-double allreduce of kernel B's (rho, ||r||^2)
    CU(cudaMemsetAsync(op->scr.partials, 0, 2 * sizeof(double), s));
    CU(cudaEventRecord(e0, s));
    for (int i = 0; i < reps && st == MAS_OK; i++) st = comm_allreduce(comm, op->scr.partials, 2, s);
    CU(cudaEventRecord(e1, s));
    if (st == MAS_OK) st = comm_sync_stream(comm, s);
    if (st == MAS_OK && cudaEventElapsedTime(&ms, e0, e1) == cudaSuccess) *allreduce_us = 1e3 * ms / reps;
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    return st;
}

long long mas_op_launch_count(const mas_op_t* op) { return op ? op->launches : -1; }

mas_status_t mas_op_set_profiling(mas_op_t* op, int on) {
    if (!op) return arg_error("null op");
    op->prof = on ? 1 : 0;
    return MAS_OK;
}

mas_status_t mas_op_kernel_times(const mas_op_t* op, double* a_ms, double* b_ms, int* n) {
    if (!op || !a_ms || !b_ms || !n) return arg_error("null argument");
    *a_ms = op->prof_a_ms;
    *b_ms = op->prof_b_ms;
    *n = op->prof_n;
    return MAS_OK;
}

mas_status_t mas_op_aniso_time(const mas_op_t* op, double* ms) {
    if (!op || !ms) return arg_error("null argument");
    *ms = op->prof_c_ms;
    return MAS_OK;
}

mas_status_t mas_op_set_aniso(mas_op_t* op, const double* kpar, const double* bhat,
                              cudaStream_t stream) {
    NvtxRange nvtx("mas_op_set_aniso");
    if (!op) return arg_error("null op");
    if (!kpar) {  // switch the term off
        op->aniso = 0;
        CU(cudaMemsetAsync(op->bad, 0, sizeof(int), stream));
        ST(op_diag(op, nullptr, stream));
        if (op->g->comm)
            ST(comm_seams(op->g->comm, op->dinv, 1, op->g->nl, op->geo.plane, op->dg,
                          op->dg + op->geo.plane, stream, rstride(op)));
        return MAS_OK;
    }
    if (!bhat) return arg_error("null bhat");
    if (op->cg1) return arg_error("field-aligned conduction: switch the single-reduction loop off first");
    if (op->placement != MAS_PLACE_CELL) return arg_error("field-aligned conduction: cell-centred placement only");
    if (op->ncomp != 1) return arg_error("field-aligned conduction needs ncomp == 1");
    if (op->g->ptheta > 1)
        return arg_error("field-aligned conduction: r-slab decompositions only (ptheta == 1)");
    mas_grid* g = op->g;
    const int nl = g->nl, nt = g->ntl, np = g->np;
    const long long N = op->Nl;
    if (!op->atab) {  // 1-D corner metrics (R22, R23), 0 on dead corners (R24)
        std::vector<double> t(3 * (size_t)nl + 2 * (size_t)nt + np, 0.0);
        double *rF = t.data(), *hr = rF + nl, *sF = hr + nl, *ht = sF + nt, *hp = ht + nt;
        double* ivr = hp + np;
        for (int il = 0; il < nl; il++) {
            const int i = g->i0 + il;
            rF[il] = g->rF[i];
            hr[il] = i > 0 ? g->rC[i] - g->rC[i - 1] : 0.0;
            ivr[il] = 1.0 / g->tab.vr[il];
        }
        for (int j = 1; j < nt; j++) {
            sF[j] = std::sin(g->tF[j]);
            ht[j] = g->tC[j] - g->tC[j - 1];
        }
        hp[0] = g->pC[0] + 2.0 * M_PI - g->pC[np - 1];
        for (int k = 1; k < np; k++) hp[k] = g->pC[k] - g->pC[k - 1];
        ST(dmalloc(&op->atab, t.size()));
        CU(cudaMemcpy(op->atab, t.data(), t.size() * sizeof(double), cudaMemcpyHostToDevice));
        op->at.rF = op->atab;
        op->at.hr = op->atab + nl;
        op->at.sF = op->atab + 2 * nl;
        op->at.ht = op->atab + 2 * nl + nt;
        op->at.hp = op->atab + 2 * nl + 2 * nt;
        op->at.ivr = op->atab + 2 * nl + 2 * nt + np;
    }
    if (!op->ca) ST(dmalloc(&op->ca, 3 * (size_t)N));
    if (op->g->comm && !op->cag) {
        ST(dmalloc(&op->cag, 6 * (size_t)op->geo.plane));
        // the NCCL loop's p_k seam buffers (2 planes; unused once the op runs the
        // P2P transport, which reads the neighbours' p_k in place)
        ST(dmalloc(&op->pkg, 2 * (size_t)op->geo.plane));
    }
    const double *kd = kpar, *bd = bhat;
    // host inputs are staged through a library-owned device buffer (kept for
    // the next call: a time-stepping caller refreshes kpar and b every step)
    const bool hk = !is_device_ptr(kpar), hb = !is_device_ptr(bhat);
    double* tmp = nullptr;
    if (hk || hb) {
        if (!op->astage) ST(dmalloc(&op->astage, 4 * (size_t)N));
        tmp = op->astage;
        if (hk) {
            CU(cudaMemcpyAsync(tmp, kpar, N * sizeof(double), cudaMemcpyHostToDevice, stream));
            kd = tmp;
        }
        if (hb) {
            CU(cudaMemcpyAsync(tmp + N, bhat, 3 * N * sizeof(double), cudaMemcpyHostToDevice, stream));
            bd = tmp + N;
        }
    }
    CU(cudaMemsetAsync(op->bad, 0, sizeof(int), stream));
    CU(launch_aniso_coef(op->geo, op->at, kd, bd, op->ca, op->bad, stream));
    Comm* comm = op->g->comm;
    const long long plane = op->geo.plane;
    if (comm)  // the corner plane above the slab: rank+1's plane 0 of (a, b, e)
        ST(comm_seams(comm, op->ca, 3, op->g->nl, plane, op->cag, op->cag + 3 * plane, stream,
                      rstride(op)));
    op->aniso = 1;
    struct AnisoOff {  // an error return below leaves the term off
        mas_op* op;
        bool keep = false;
        ~AnisoOff() {
            if (!keep) op->aniso = 0;
        }
    } on_error{op};
    ST(op_diag(op, nullptr, stream));
    if (comm)
        ST(comm_seams(comm, op->dinv, 1, op->g->nl, plane, op->dg, op->dg + plane, stream, rstride(op)));
    int bad = 0;
    CU(cudaMemcpyAsync(&bad, op->bad, sizeof(int), cudaMemcpyDeviceToHost, stream));
    CU(cudaStreamSynchronize(stream));
    if (comm) {  // agree on the verdict across ranks
        double* d = op->dot_out;
        double hb = bad;
        CU(cudaMemcpyAsync(d, &hb, sizeof(double), cudaMemcpyHostToDevice, stream));
        ST(comm_allreduce(comm, d, 1, stream));
        CU(cudaMemcpyAsync(&hb, d, sizeof(double), cudaMemcpyDeviceToHost, stream));
        CU(cudaStreamSynchronize(stream));
        bad = hb != 0.0;
    }
    if (bad) {
        op->aniso = 0;
        op_diag(op, nullptr, stream);
        if (comm) comm_seams(comm, op->dinv, 1, op->g->nl, plane, op->dg, op->dg + plane, stream, rstride(op));
        return arg_error("kpar negative or non-finite, b non-finite, or Jacobi diagonal D <= 0");
    }
    on_error.keep = true;
    return MAS_OK;
}

mas_status_t mas_pcg_solve(const mas_op_t* op_c, const double* rhs, double* x, double tol,
                           int maxit, int* iters, double* relres, double* res_hist,
                           cudaStream_t s) {
    NvtxRange nvtx("mas_pcg_solve");
    mas_op* op = const_cast<mas_op*>(op_c);
    if (!op || !rhs || !x || !iters || !relres) return arg_error("null argument");
    if (!(tol >= 0.0) || maxit < 0) return arg_error("need tol >= 0 and maxit >= 0");
    const int nc = op->ncomp;
    const long long plane = op->geo.plane;
    const size_t bytes = nc * op->Nl * sizeof(double);
    Comm* comm = op->g->comm;
    ST(ensure_hist(op, maxit));
    op->launches = 0;

    // host buffers are staged through library-owned device memory
    const double* fd = rhs;
    double* xd = x;
    const bool hf = !is_device_ptr(rhs), hx = !is_device_ptr(x);
    if (hf || hx) ST(ensure_stage(op));
    if (hf) {
        CU(cudaMemcpyAsync(op->stage_a, rhs, bytes, cudaMemcpyHostToDevice, s));
        fd = op->stage_a;
    }
    if (hx) {
        CU(cudaMemcpyAsync(op->stage_b, x, bytes, cudaMemcpyHostToDevice, s));
        xd = op->stage_b;
    }

    if (op->cg1) {  // NEXT-1: single-reduction loop (one GPU, isotropic operator)
        mas_status_t st = cg1_solve(op, fd, xd, tol, maxit, iters, relres, res_hist, s);
        if (hx && (st == MAS_OK || st == MAS_NOT_CONVERGED || st == MAS_ERR_BREAKDOWN))
            CU(cudaMemcpy(x, xd, bytes, cudaMemcpyDeviceToHost));
        return st;
    }
    const bool p2p = op->p2p;
    PcgState init{};
    if (p2p) init.epoch = ++op->epoch;
    init.tol = tol;
    init.maxit = maxit;
    init.k = 1;
    init.stopped = 0;
    init.status = MAS_NOT_CONVERGED;
    CU(cudaMemcpyAsync(op->st, &init, sizeof(init), cudaMemcpyHostToDevice, s));
    *op->host_flag = 0;
    double* rho_h = op->hist;
    double* sig_h = op->hist + op->hist_cap;
    double* rr_h = op->hist + 2 * op->hist_cap;

    // a3: r = f - L x0 and the three initial dot products
    ST(pole_pass(op, xd, nc, s));  // theta nodes: x0's pole rows are one value each (their average)
    if (comm) ST(comm_seams(comm, xd, nc, op->g->nl, plane, op->xg, op->xg + nc * plane, s, rstride(op)));
    ST(tseams(op, xd, nc, op->xgt, s));
    StencilArgs a{};
    a.g = op->geo;
    a.chunk = op->chunk;
    a.u = halo_of(op, xd, op->xg, nc);
    a.kappa = halo_of(op, op->kappa, op->kg, 1);
    a.dinv = halo_of(op, op->dinv, op->dg, 1);
    a.tu = packed_rows(op, op->xgt, nc);
    a.tkappa = packed_rows(op, op->kgt, 1);
    a.tdinv = packed_rows(op, op->dgt, 1);
    a.c = op->c;
    a.curv = op->curv;
    a.f = fd;
    a.out = op->r;
    a.st = op->st;
    a.rho_hist = rho_h;
    a.sigma_hist = sig_h;
    a.rr_hist = rr_h;
    a.scr = op->scr;
    a.host_flag = op->host_flag_dev;
    a.p2p = p2p_args(op);
    a.nopub = op->aniso && p2p;  // k_aniso<RESID> publishes the corrected init sums
    CU(launch_stencil(MODE_RESID, nc, a, s));
    op->launches++;
    AnisoArgs an{};
    if (op->aniso) {  // r -= L_par x0 and the three initial dots again (rank-local sums)
        an = aniso_args(op, MODE_RESID, halo_of(op, xd, op->xg, 1), op->r);
        an.f = fd;
        an.dinv = op->dinv;
        CU(launch_aniso(MODE_RESID, an, s));
        op->launches++;
        an = aniso_args(op, MODE_PCGA, Halo{}, op->q);
    }
    if (op->tnode) {  // the caps' residuals, then the three sums again
        ST(pole_pass(op, op->r, nc, s));
        CU(launch_init_dots(op->geo, nc, fd, op->r, op->dinv, op->scr, op->st, op->b_blocks, s));
        op->launches += 2;
    }
    if (comm && !p2p) ST(comm_allreduce(comm, &op->st->pend_rho, 3, s));  // rho, rr, ff

    StreamArgs b{};
    b.g = op->geo;
    b.ncomp = nc;
    b.r = op->r;
    b.q = op->q;
    b.dinv = op->dinv;
    b.tnode = op->tnode;
    b.st = op->st;
    b.rho_hist = rho_h;
    b.sigma_hist = sig_h;
    b.rr_hist = rr_h;
    b.scr = op->scr;
    b.host_flag = op->host_flag_dev;
    b.p2p = p2p_args(op);
    b.aniso = op->aniso && !lpar_in_a(op);  // P2P: sigma's L_par part in its own slot (MB_C)
    b.x = xd;  // a breakdown at an even k completes x's two-iteration update
    b.p[0] = op->p[0];
    b.p[1] = op->p[1];
    {  // test hook: a breakdown forced in B(k) (tests of the breakdown paths)
        const char* t = getenv("MAS_TEST_TRANSPORTS");
        const char* k = getenv("MAS_TEST_BREAKDOWN_AT");
        b.brk_at = (t && atoi(t) == 1 && k) ? atoi(k) : 0;
    }

    // a4: iterations.  Kernel A(k) reads k, alpha, beta and the convergence
    // decision from PcgState; the host only keeps two iterations in flight
    // and stops enqueueing once the device reports the stop (a decision all
    // ranks take identically, so the collectives stay matched).
    a.u = r_halo(op);
    a.tu = r_trows(op);
    a.out = op->q;
    a.x = xd;
    a.f = nullptr;
    set_lpar_args(op, a);  // the field-aligned term inside kernel A (fused)
    // no host involvement per iteration on one GPU and with the P2P transport
    // (virtual P2P ranks share one GPU and need host ordering: comm_vsync)
    const bool graph = !op->prof && op->use_graph && (!comm || (p2p && !comm_is_virtual(comm)));
    if (graph) {
        const bool pre = op->graph_pre != 0;
        ST(loop_graph(op, a, b, an, pre));
        if (pre) {
            a.pold = pold_halo(op, 1);  // iteration 1 (not read)
            a.tpold = pold_trows(op, 1);
            a.pnew = op->p[1];
            CU(launch_stencil(MODE_PCGA, nc, a, s, true));
            if (op->aniso && !lpar_in_a(op)) {
                an.u = aniso_p_halo(op, 1);
                CU(launch_aniso(MODE_PCGA, an, s));
            }
            CU(launch_pcg_b(b, op->b_blocks, s));  // (theta nodes: with the pole pass on q)
        }
        CU(cudaGraphLaunch(op->gexec, s));
    }
    int stop_seen_at = -1;
    for (int k = 1; !graph && k <= maxit + 1; k++) {
        NvtxRange nvtx_it("pcg iteration (A, [seams, allreduce], B)");
        double* pold = op->p[(k + 1) & 1];
        double* pnew = op->p[k & 1];
        a.pold = pold_halo(op, k);
        a.tpold = pold_trows(op, k);
        a.pnew = pnew;
        cudaEvent_t* pe = nullptr;
        if (op->prof) {
            ST(ensure_prof_events(op, k));
            pe = &op->pev[6 * (size_t)(k - 1)];
        }
        if (comm && !p2p && split_theta(op)) {
            // (r, theta) decomposition over NCCL: r-plane seams and packed
            // theta rows of r and p_{k-1} on the solve stream, then kernel A
            ST(comm_seams(comm, op->r, nc, op->g->nl, plane, op->rg, op->rg + nc * plane, s,
                          rstride(op)));
            ST(tseams(op, op->r, nc, op->rgt, s));
            if (k > 1) {
                ST(comm_seams(comm, pold, nc, op->g->nl, plane, op->pg[(k + 1) & 1],
                              op->pg[(k + 1) & 1] + nc * plane, s, rstride(op)));
                ST(tseams(op, pold, nc, op->pgt[(k + 1) & 1], s));
            }
            if (pe) CU(cudaEventRecord(pe[0], s));
            CU(launch_stencil(MODE_PCGA, nc, a, s, k == 1));
            op->launches++;
        } else if (comm && !p2p) {
            // seams of r and p_{k-1} on the comm stream, overlapped with kernel
            // A on the interior chunks; the two edge chunks wait for them
            CU(cudaEventRecord(op->ev_ready, s));
            CU(cudaStreamWaitEvent(op->cs, op->ev_ready, 0));
            ST(comm_seams(comm, op->r, nc, op->g->nl, plane, op->rg, op->rg + nc * plane, op->cs,
                          rstride(op)));
            if (k > 1)
                ST(comm_seams(comm, pold, nc, op->g->nl, plane, op->pg[(k + 1) & 1],
                              op->pg[(k + 1) & 1] + nc * plane, op->cs, rstride(op)));
            CU(cudaEventRecord(op->ev_seam, op->cs));
            if (pe) CU(cudaEventRecord(pe[0], s));
            const int nchunk = (op->g->nl + op->chunk - 1) / op->chunk;
            if (nchunk >= 3) {
                a.part = 1;
                CU(launch_stencil(MODE_PCGA, nc, a, s, k == 1));
                CU(cudaStreamWaitEvent(s, op->ev_seam, 0));
                a.part = 2;
                CU(launch_stencil(MODE_PCGA, nc, a, s, k == 1));
                a.part = 0;
                op->launches += 2;
            } else {
                CU(cudaStreamWaitEvent(s, op->ev_seam, 0));
                CU(launch_stencil(MODE_PCGA, nc, a, s, k == 1));
                op->launches++;
            }
        } else {
            if (p2p) ST(comm_vsync(comm, s));  // virtual P2P ranks: all B(k-1) done
            if (pe) CU(cudaEventRecord(pe[0], s));
            CU(launch_stencil(MODE_PCGA, nc, a, s, k == 1));
            op->launches++;
        }
        if (pe) CU(cudaEventRecord(pe[1], s));
        if (op->aniso && !lpar_in_a(op)) {  // q += L_par p_k, sigma += <p_k, L_par p_k> (rank-local)
            if (comm && !p2p)  // the p_k planes of the r-neighbours (kernel A(k) just wrote them)
                ST(comm_seams(comm, pnew, 1, op->g->nl, plane, op->pkg, op->pkg + plane, s,
                              rstride(op)));
            if (p2p) ST(comm_vsync(comm, s));  // virtual P2P ranks: all A(k) done
            an.u = aniso_p_halo(op, k);
            if (pe) CU(cudaEventRecord(pe[4], s));
            CU(launch_aniso(MODE_PCGA, an, s));
            if (pe) CU(cudaEventRecord(pe[5], s));
            op->launches++;
        }
        if (comm && !p2p) ST(comm_allreduce(comm, &op->st->pend_sigma, 1, s));
        if (k <= maxit) {
            // virtual P2P ranks: all A(k) and k_aniso(k) done (B(k) reads slots A and C)
            if (p2p) ST(comm_vsync(comm, s));
            // (theta nodes, NEXT-2: kernel B forms the caps of q = L p itself)
            if (pe) CU(cudaEventRecord(pe[2], s));
            CU(launch_pcg_b(b, op->b_blocks, s));
            op->launches++;
            if (pe) CU(cudaEventRecord(pe[3], s));
            if (comm && !p2p) ST(comm_allreduce(comm, &op->st->pend_rho, 2, s));
        }
        CU(cudaEventRecord(op->ev[k & 1], s));
        if (k >= 2) {
            // wait for iteration k-1 to finish, then stop if the device
            // decided at or before iteration k-1 (every rank sees the same
            // decision at the same point, so the collectives stay matched)
            ST(comm_wait_event(comm, op->ev[(k - 1) & 1]));
            const int flag = *(volatile int*)op->host_flag;
            if (flag > 0 && flag <= k - 1) {
                stop_seen_at = k;
                break;
            }
        }
    }
    (void)stop_seen_at;
    ST(comm_sync_stream(comm, s));
    // P2P: no rank may publish the next solve's partials while another rank's
    // kernels of this solve can still read its mailbox
    if (p2p && comm) ST(comm_barrier(comm, s));
    PcgState fin{};
    CU(cudaMemcpy(&fin, op->st, sizeof(fin), cudaMemcpyDeviceToHost));
    if (!fin.stopped) {
        set_last_error("internal: PCG loop ended without a stop decision");
        return MAS_ERR_CUDA;
    }
    *iters = fin.iters;
    *relres = fin.relres;
    if (graph) {  // iteration 1 + 4 kernels per executed loop body (iterations 2k, 2k+1)
        const int last_a = fin.status == MAS_ERR_BREAKDOWN ? fin.iters : fin.iters + 1;
        const int bodies = last_a <= 2 ? 1 : last_a / 2;
        const int per = 2 + (op->aniso && !lpar_in_a(op) ? 1 : 0);  // kernels per iteration
        op->launches += per + 2LL * per * bodies;
    }
    if (res_hist) {
        // after a breakdown at iteration k only ||r_0..r_{k-1}|| exist
        const int nh = fin.status == MAS_ERR_BREAKDOWN ? fin.iters : fin.iters + 1;
        std::vector<double> rr(nh);
        CU(cudaMemcpy(rr.data(), rr_h, rr.size() * sizeof(double), cudaMemcpyDeviceToHost));
        for (int k = 0; k < nh; k++) res_hist[k] = std::sqrt(rr[k]);
    }
    if (op->prof) {  // average device time of the working launches 1..iters
        double sa = 0.0, sb = 0.0, sc = 0.0;
        int n = 0;
        for (int k = 1; k <= fin.iters && 6 * (size_t)k <= op->pev.size(); k++, n++) {
            float ta = 0.f, tb = 0.f, tc = 0.f;
            const cudaEvent_t* e = &op->pev[6 * (size_t)(k - 1)];
            CU(cudaEventElapsedTime(&ta, e[0], e[1]));
            CU(cudaEventElapsedTime(&tb, e[2], e[3]));
            if (op->aniso && !lpar_in_a(op)) CU(cudaEventElapsedTime(&tc, e[4], e[5]));
            sa += ta;
            sb += tb;
            sc += tc;
        }
        op->prof_c_ms = n ? sc / n : 0.0;
        op->prof_n = n;
        op->prof_a_ms = n ? sa / n : 0.0;
        op->prof_b_ms = n ? sb / n : 0.0;
    }
    if (hx) CU(cudaMemcpy(x, xd, bytes, cudaMemcpyDeviceToHost));
    return (mas_status_t)fin.status;
}

// ---------------------------------------------------------------------------
// stacked solve: one PCG on the stacked vector of several operators (NEXT-2,
// reading R34).  Each block runs its own kernels A and B on
// its own PcgState exactly as a rank of the r-slab NCCL loop does; where that
// loop allreduces the partial sums over the ranks, k_stack_sum sums them over
// the blocks (in block order) and writes the sum back to every block's state.
// Every block then takes the same alpha, beta and stop decision.
// ---------------------------------------------------------------------------
static_assert(offsetof(PcgState, pend_sigma) == 0 && offsetof(PcgState, pend_rho) == 8 &&
                  offsetof(PcgState, pend_rr) == 16 && offsetof(PcgState, pend_ff) == 24,
              "k_stack_sum offsets (0 sigma; 1 rho, 2 rr, 3 ff)");
}  // extern "C"

struct mas_stack {
    std::vector<mas_op*> ops;
    cudaGraphExec_t gexec = nullptr;   // the loop graph (iteration 1, then the while node)
    std::vector<const double*> g_x, g_hist;
    cudaStream_t cap = nullptr;
    cudaEvent_t ev[2] = {nullptr, nullptr};
};

extern "C" {

static StackStates stack_states(const mas_stack* sk) {
    StackStates ss{};
    ss.n = (int)sk->ops.size();
    for (int m = 0; m < ss.n; m++) ss.st[m] = sk->ops[m]->st;
    return ss;
}

// iteration k of every block: kernels A, the sigma sum, [q's pole rows,]
// kernels B, the rho / ||r||^2 sum
static cudaError_t stack_iteration(const mas_stack* sk, std::vector<StencilArgs>& a,
                                   std::vector<StreamArgs>& b, int k, bool first, bool with_b,
                                   cudaStream_t s) {
    const StackStates ss = stack_states(sk);
    cudaError_t e = cudaSuccess;
    for (size_t m = 0; m < sk->ops.size() && e == cudaSuccess; m++) {
        const mas_op* op = sk->ops[m];
        a[m].pold = pold_halo(op, k);
        a[m].tpold = pold_trows(op, k);
        a[m].pnew = op->p[k & 1];
        e = launch_stencil(MODE_PCGA, op->ncomp, a[m], s, first);
    }
    if (e == cudaSuccess) e = launch_stack_sum(ss, 0, 1, s);  // sigma_k
    if (!with_b) return e;
    for (size_t m = 0; m < sk->ops.size() && e == cudaSuccess; m++) {
        const mas_op* op = sk->ops[m];
        e = launch_pcg_b(b[m], op->b_blocks, s);  // (theta nodes: with the pole pass on q)
    }
    if (e == cudaSuccess) e = launch_stack_sum(ss, 1, 2, s);  // rho_k, ||r_k||^2
    return e;
}

// the single-GPU loop graph of a stack (loop_graph's structure): iteration 1
// as a chain of kernel nodes, then a device-side while node whose body runs
// iterations 2k and 2k+1; rebuilt when an x or history buffer moves
static mas_status_t stack_graph(mas_stack* sk, std::vector<StencilArgs> a, std::vector<StreamArgs> b) {
    const size_t n = sk->ops.size();
    bool same = sk->gexec && sk->g_x.size() == n;
    for (size_t m = 0; same && m < n; m++) same = sk->g_x[m] == a[m].x && sk->g_hist[m] == a[m].rho_hist;
    if (same) return MAS_OK;
    if (sk->gexec) {
        cudaGraphExecDestroy(sk->gexec);
        sk->gexec = nullptr;
    }
    if (!sk->cap) CU(cudaStreamCreateWithFlags(&sk->cap, cudaStreamNonBlocking));
    cudaGraph_t g;
    CU(cudaGraphCreate(&g, 0));
    cudaError_t e = cudaStreamBeginCaptureToGraph(sk->cap, g, nullptr, nullptr, 0, cudaStreamCaptureModeThreadLocal);
    if (e == cudaSuccess) {
        e = stack_iteration(sk, a, b, 1, true, true, sk->cap);
        cudaGraph_t out = g;
        const cudaError_t e2 = cudaStreamEndCapture(sk->cap, &out);
        if (e == cudaSuccess) e = e2;
    }
    std::vector<cudaGraphNode_t> deps;
    size_t nn = 0;
    if (e == cudaSuccess) e = cudaGraphGetNodes(g, nullptr, &nn);
    std::vector<cudaGraphNode_t> nodes(nn);
    if (e == cudaSuccess && nn) e = cudaGraphGetNodes(g, nodes.data(), &nn);
    for (size_t i = 0; i < nn && e == cudaSuccess; i++) {
        size_t nd = 0;
        e = cudaGraphNodeGetDependentNodes(nodes[i], nullptr, &nd);
        if (e == cudaSuccess && nd == 0) deps.push_back(nodes[i]);
    }
    if (e == cudaSuccess && deps.size() != 1) e = cudaErrorInvalidValue;
    cudaGraphConditionalHandle h;
    if (e == cudaSuccess) e = cudaGraphConditionalHandleCreate(&h, g, 1, cudaGraphCondAssignDefault);
    cudaGraphNodeParams p = {};
    p.type = cudaGraphNodeTypeConditional;
    p.conditional.handle = h;
    p.conditional.type = cudaGraphCondTypeWhile;
    p.conditional.size = 1;
    cudaGraphNode_t node;
    if (e == cudaSuccess) e = cudaGraphAddNode(&node, g, deps.data(), deps.size(), &p);
    if (e == cudaSuccess) {
        cudaGraph_t body = p.conditional.phGraph_out[0];
        e = cudaStreamBeginCaptureToGraph(sk->cap, body, nullptr, nullptr, 0, cudaStreamCaptureModeThreadLocal);
        if (e == cudaSuccess) {
            for (size_t m = 0; m < n; m++) a[m].cond = b[m].cond = (unsigned long long)h;
            for (int kk = 2; kk <= 3 && e == cudaSuccess; kk++) e = stack_iteration(sk, a, b, kk, false, true, sk->cap);
            cudaGraph_t out = body;
            const cudaError_t e2 = cudaStreamEndCapture(sk->cap, &out);
            if (e == cudaSuccess) e = e2;
        }
    }
    if (e == cudaSuccess) e = cudaGraphInstantiate(&sk->gexec, g, 0);
    cudaGraphDestroy(g);
    if (e != cudaSuccess) {
        cudaGetLastError();
        sk->gexec = nullptr;
        set_last_error(std::string("stack loop graph: ") + cudaGetErrorString(e));
        return MAS_ERR_CUDA;
    }
    sk->g_x.resize(n);
    sk->g_hist.resize(n);
    for (size_t m = 0; m < n; m++) {
        sk->g_x[m] = a[m].x;
        sk->g_hist[m] = a[m].rho_hist;
    }
    return MAS_OK;
}

mas_status_t mas_stack_create(mas_op_t* const* ops, int nops, mas_stack_t** out) {
    if (!out) return arg_error("null out");
    *out = nullptr;
    if (!ops || nops < 1 || nops > kMaxStack) return arg_error("need 1 <= nops <= 8 operators");
    for (int m = 0; m < nops; m++) {
        const mas_op* op = ops[m];
        if (!op) return arg_error("null operator");
        for (int q = 0; q < m; q++)
            if (ops[q] == op) return arg_error("the same operator twice in a stack");
        if (op->g->comm) return arg_error("stacked solve: one GPU without a mas_dist_t");
        if (op->p2p) return arg_error("stacked solve: no P2P transport");
        if (op->cg1) return arg_error("stacked solve: the two-kernel loop (single reduction is on)");
        if (op->aniso) return arg_error("stacked solve: isotropic operators (no mas_op_set_aniso)");
    }
    mas_stack* sk = new mas_stack;
    sk->ops.assign(ops, ops + nops);
    for (int q = 0; q < 2; q++)
        if (cudaEventCreateWithFlags(&sk->ev[q], cudaEventDisableTiming) != cudaSuccess) {
            cudaGetLastError();
            mas_stack_destroy(sk);
            set_last_error("stack events");
            return MAS_ERR_CUDA;
        }
    *out = sk;
    return MAS_OK;
}

mas_status_t mas_stack_destroy(mas_stack_t* sk) {
    if (!sk) return MAS_OK;
    if (sk->gexec) cudaGraphExecDestroy(sk->gexec);
    if (sk->cap) cudaStreamDestroy(sk->cap);
    for (cudaEvent_t e : sk->ev)
        if (e) cudaEventDestroy(e);
    delete sk;
    return MAS_OK;
}

mas_status_t mas_stack_solve(mas_stack_t* sk, const double* const* rhs, double* const* x, double tol,
                             int maxit, int* iters, double* relres, double* res_hist, cudaStream_t s) {
    NvtxRange nvtx("mas_stack_solve");
    if (!sk || !rhs || !x || !iters || !relres) return arg_error("null argument");
    if (!(tol >= 0.0) || maxit < 0) return arg_error("need tol >= 0 and maxit >= 0");
    const size_t n = sk->ops.size();
    // host arrays are staged through each op's library-owned device buffers
    // (as mas_pcg_solve does); device arrays are used in place
    std::vector<const double*> fd(n);
    std::vector<double*> xd(n);
    std::vector<bool> hx(n, false);
    for (size_t m = 0; m < n; m++) {
        if (!rhs[m] || !x[m]) return arg_error("null rhs or x");
        mas_op* op = sk->ops[m];
        const size_t bytes = op->ncomp * op->Nl * sizeof(double);
        fd[m] = rhs[m];
        xd[m] = x[m];
        const bool hf = !is_device_ptr(rhs[m]);
        hx[m] = !is_device_ptr(x[m]);
        if (hf || hx[m]) ST(ensure_stage(op));
        if (hf) {
            CU(cudaMemcpyAsync(op->stage_a, rhs[m], bytes, cudaMemcpyHostToDevice, s));
            fd[m] = op->stage_a;
        }
        if (hx[m]) {
            CU(cudaMemcpyAsync(op->stage_b, x[m], bytes, cudaMemcpyHostToDevice, s));
            xd[m] = op->stage_b;
        }
    }
    const StackStates ss = stack_states(sk);
    std::vector<StencilArgs> a(n);
    std::vector<StreamArgs> b(n);
    // init: every block's state, r = f - L x0 and its three partial sums
    for (size_t m = 0; m < n; m++) {
        mas_op* op = sk->ops[m];
        ST(ensure_hist(op, maxit));
        op->launches = 0;
        PcgState init{};
        init.tol = tol;
        init.maxit = maxit;
        init.k = 1;
        init.status = MAS_NOT_CONVERGED;
        CU(cudaMemcpyAsync(op->st, &init, sizeof(init), cudaMemcpyHostToDevice, s));
        *op->host_flag = 0;
        const int nc = op->ncomp;
        ST(pole_pass(op, xd[m], nc, s));
        StencilArgs& A = a[m];
        A.g = op->geo;
        A.chunk = op->chunk;
        A.u = halo_of(op, xd[m], op->xg, nc);
        A.kappa = halo_of(op, op->kappa, op->kg, 1);
        A.dinv = halo_of(op, op->dinv, op->dg, 1);
        A.tu = packed_rows(op, op->xgt, nc);
        A.tkappa = packed_rows(op, op->kgt, 1);
        A.tdinv = packed_rows(op, op->dgt, 1);
        A.c = op->c;
        A.curv = op->curv;
        A.f = fd[m];
        A.out = op->r;
        A.st = op->st;
        A.rho_hist = op->hist;
        A.sigma_hist = op->hist + op->hist_cap;
        A.rr_hist = op->hist + 2 * op->hist_cap;
        A.scr = op->scr;
        A.host_flag = op->host_flag_dev;
        CU(launch_stencil(MODE_RESID, nc, A, s));
        if (op->tnode) {  // the caps' residuals, then the three sums again
            ST(pole_pass(op, op->r, nc, s));
            CU(launch_init_dots(op->geo, nc, fd[m], op->r, op->dinv, op->scr, op->st, op->b_blocks, s));
        }
        // the iteration arguments (kernel A: p from r; kernel B)
        A.u = r_halo(op);
        A.tu = r_trows(op);
        A.out = op->q;
        A.x = xd[m];
        A.f = nullptr;
        StreamArgs& B = b[m];
        B.g = op->geo;
        B.ncomp = nc;
        B.r = op->r;
        B.q = op->q;
        B.dinv = op->dinv;
        B.tnode = op->tnode;
        B.st = op->st;
        B.rho_hist = A.rho_hist;
        B.sigma_hist = A.sigma_hist;
        B.rr_hist = A.rr_hist;
        B.scr = op->scr;
        B.host_flag = op->host_flag_dev;
        B.x = xd[m];
        B.p[0] = op->p[0];
        B.p[1] = op->p[1];
    }
    CU(launch_stack_sum(ss, 1, 3, s));  // rho_0, ||r_0||^2, ||f||^2 of the stacked vector
    bool graph = true;
    for (const mas_op* op : sk->ops) graph = graph && op->use_graph && !op->prof;
    if (graph) {
        ST(stack_graph(sk, a, b));
        CU(cudaGraphLaunch(sk->gexec, s));
    }
    for (int k = 1; !graph && k <= maxit + 1; k++) {
        CU(stack_iteration(sk, a, b, k, k == 1, k <= maxit, s));
        CU(cudaEventRecord(sk->ev[k & 1], s));
        if (k >= 2) {  // stop once block 0 reports a decision at or before iteration k-1
            CU(cudaEventSynchronize(sk->ev[(k - 1) & 1]));
            const int flag = *(volatile int*)sk->ops[0]->host_flag;
            if (flag > 0 && flag <= k - 1) break;
        }
    }
    CU(cudaStreamSynchronize(s));
    PcgState fin{};
    for (size_t m = 0; m < n; m++) {
        PcgState f{};
        CU(cudaMemcpy(&f, sk->ops[m]->st, sizeof(f), cudaMemcpyDeviceToHost));
        if (!f.stopped) {
            set_last_error("internal: stacked loop ended without a stop decision");
            return MAS_ERR_CUDA;
        }
        if (m == 0) {
            fin = f;
        } else if (f.iters != fin.iters || f.status != fin.status) {
            set_last_error("internal: the blocks of a stack took different stop decisions");
            return MAS_ERR_CUDA;
        }
    }
    *iters = fin.iters;
    *relres = fin.relres;
    if (res_hist) {
        const int nh = fin.status == MAS_ERR_BREAKDOWN ? fin.iters : fin.iters + 1;
        std::vector<double> rr(nh);
        const mas_op* op0 = sk->ops[0];
        CU(cudaMemcpy(rr.data(), op0->hist + 2 * op0->hist_cap, rr.size() * sizeof(double),
                      cudaMemcpyDeviceToHost));
        for (int k = 0; k < nh; k++) res_hist[k] = std::sqrt(rr[k]);
    }
    for (size_t m = 0; m < n; m++)
        if (hx[m])
            CU(cudaMemcpy(x[m], xd[m], sk->ops[m]->ncomp * sk->ops[m]->Nl * sizeof(double), cudaMemcpyDeviceToHost));
    return (mas_status_t)fin.status;
}

mas_status_t mas_op_destroy(mas_op_t* op) {
    op_free(op);
    return MAS_OK;
}

}  // extern "C"
