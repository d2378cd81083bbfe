// mas_internal.h — structures shared by the host driver (C++) and the CUDA
// kernels of the B200 MAS-PCG library.  Not part of the ABI.
#pragma once

#include <cuda_runtime.h>

#include <atomic>
#include <cstdint>
#include <string>

#include "../../include/mas_pcg.h"

namespace mas {

// ---------------------------------------------------------------------------
// Geometry: 1-D coefficient tables (device pointers), computed once on the
// host from the node/half meshes (grid.cpp).  With them the per-cell operator
// of DESIGN.md §5.1 is
//   (L u)_P = c u + aRm (u-u_{i-1}) + aRp (u-u_{i+1}) + aTm (u-u_{j-1})
//           + aTp (u-u_{j+1}) + aPm (u-u_{k-1}) + aPp (u-u_{k+1})
//   aRm = wRm[i] kf,   aTm = irc2[i] wTm[j] kf,   aPm = irc2[i] isc2[j] wPm[k] kf
// with kf = (kappa_P + kappa_N)/2 of that face.  V_P = vr[i] vt[j] vp[k].
// ---------------------------------------------------------------------------
struct Geo {
    int nl, nt, np;        // local r-planes, local theta rows, phi
    long long plane;       // nt*np
    int glob_lo, glob_hi;  // this slab owns the global inner / outer r-boundary
    const double* wRm;     // [nl] r-face i   / V  (0 on a global Neumann face)
    const double* wRp;     // [nl] r-face i+1 / V
    const double* irc2;    // [nl] 1/rC^2
    const double* vr;      // [nl] rC^2 dr
    const double* wTm;     // [nt] theta-face j   / (V/r^2)   (0 at pole/wall)
    const double* wTp;     // [nt] theta-face j+1 / (V/r^2)
    const double* isc2;    // [nt] 1/sin^2(tC)
    const double* vt;      // [nt] sin(tC) dt
    const double* wPm;     // [np] phi-face k   / (V/(r^2 sin^2))
    const double* wPp;     // [np] phi-face k+1 / (V/(r^2 sin^2))
    const double* vp;      // [np] dp
};

// A field read with an r-halo: interior planes plus optional ghost planes
// (multi-GPU seams).  ghost == nullptr at a global boundary or on one GPU.
struct Halo {
    const double* in;   // [ncomp][nl][nt][np]
    const double* glo;  // plane i0-1 of component 0: a ghost copy [ncomp][nt][np], or (P2P
                        // transport) the last plane of rank-1's own array, read over NVLink
    const double* ghi;  // plane i0+nl of component 0 (ghost copy, or rank+1's first plane)
    int slo, shi;       // component strides of glo / ghi (plane for a ghost copy,
                        // nl_neighbour * plane for a neighbour's array)
};

// The theta-ghost rows of a field under an (r, theta) decomposition (NEXT-3):
// rows j = -1 and j = nt_local of every local plane, taken from the theta
// neighbours.  Either a packed copy [ncomp][nl][np] (static kappa / 1/D rows,
// x at init, the NCCL loop) or, under the P2P transport, the neighbour's own
// array read in place.  lo / hi == nullptr: no neighbour on that side (pole or
// theta wall: the face carries no flux, the halo holds zeros).
struct TRows {
    const double* lo;  // row j = -1, component 0, plane 0
    const double* hi;  // row j = nt_local
    int cs_lo, ps_lo;  // component / plane strides of lo
    int cs_hi, ps_hi;
};

// ---------------------------------------------------------------------------
// P2P transport (multi-GPU over NVLink / NVSwitch peer memory): the two
// per-iteration scalar allreduces become one-shot mailbox writes fused into
// the reducing kernel's last block, and kernel A reads the r-neighbours'
// edge planes in place (no seam exchange).  See DESIGN.md §7.
// ---------------------------------------------------------------------------
struct Mail {                 // one rank's published partial sums
    double v[4];
    unsigned long long seq;   // (epoch << 32) | (k + 1) once v is valid
    unsigned long long pad[3];
};
// mailbox slots: A(k) -> B(k) (sigma); B(k)/init -> A(k+1); the field-aligned
// term's k_aniso(k) -> B(k) (its sigma part)
enum { MB_A = 0, MB_B = 1, MB_C = 2, MB_SLOTS = 3 };
struct P2P {
    Mail* own;                // this rank's mailbox [MB_SLOTS][nranks]
    Mail* const* peers;       // [nranks] every rank's mailbox (device-visible pointers)
    int nranks;               // 0: transport off
    int rank;
};

// Device-resident PCG state (one per op).  "pend_*" are the current
// rank-local -> (allreduced) sums; the *_hist arrays are archived values.
struct PcgState {
    double pend_sigma;  // <p_k, q_k>_V           written by A(k), read by B(k)
    double pend_rho;    // <r_k, z_k>_V           written by B(k), read by A(k+1)
    double pend_rr;     // <r_k, r_k>_V
    double pend_ff;     // <f, f>_V               written by init
    double sigma_part;  // <p,q> of the interior launch of a split kernel A (multi-GPU overlap)
    double rho_prev;    // rho of the previous A: at A(k) it is rho_{k-2} (A's last block updates)
    double sigma_prev;  // sigma_{k-1}, saved by B(k-1)'s last block
    double tol;
    double relres;
    int k;              // current iteration (A(k), B(k)); B's last block increments
    int maxit;
    int stopped;        // 1 once a kernel decided the solve is over
    int iters;
    int status;         // mas_status_t
    int pad;
    unsigned long long epoch;  // P2P: solve counter (mailbox sequence numbers)
    // single-reduction PCG (MODE_CG1): decided by kernel k's last block for k+1
    double cg_alpha;    // alpha_k
    double cg_beta;     // beta_k
    double cg_gamma;    // gamma_k = <r_k, D^-1 r_k>_V
    // the two-iteration x update: alpha_{k-1} as A(k) used
    // it, saved by A(k)'s last block for A(k+1) and for B(k)'s breakdown fix-up
    double alpha_save;
};

struct Scratch {
    double* partials;    // [max_blocks * 4]
    unsigned* ticket;    // one counter per kernel kind
};

// MODE_CG1: the single-reduction (Chronopoulos-Gear) iteration kernel of
// NEXT-1: its FIRSTK instantiation is the init w0 = L D^-1 r0
enum { MODE_APPLY = 0, MODE_RESID = 1, MODE_PCGA = 2, MODE_CG1 = 3 };

struct StencilArgs {
    Geo g;
    int chunk;                // r-planes per work item
    int ntj, ntk, nchunk;     // tiles in theta, phi; chunks in r
    Halo u;                   // APPLY/RESID: x;  PCGA: r (p = D^-1 r + beta p_old);  CG1: r_{k-1}
    Halo pold;                // PCGA: p_{k-1};  CG1: s_{k-2}
    Halo w;                   // CG1: w_{k-1} = L u_{k-1}
    double* sout;             // CG1: s_{k-1} = w_{k-1} + beta s_{k-2}
    double* rout;             // CG1: r_k = r_{k-1} - alpha s_{k-1}
    Halo dinv;                // PCGA: 1/D with halo;  RESID: own only
    Halo kappa;
    TRows tu, tpold, tdinv, tkappa;  // theta-ghost rows (2-D decomposition; zero: none)
    const double* c;          // [nl][nt][np] or nullptr
    const double* f;          // RESID: rhs [ncomp][nl][nt][np]
    double* out;              // APPLY: y;  RESID: r;  PCGA: q;  CG1: w_k
    double* pnew;             // PCGA: p_k;  CG1: p (in place: p_{k-2} in, p_{k-1} out)
    double* x;                // PCGA: x (deferred update x += alpha_{k-1} p_{k-1});  CG1: x_k
    PcgState* st;             // RESID / PCGA
    double* rho_hist;         // [maxit+2]
    double* sigma_hist;       // [maxit+2]
    double* rr_hist;          // [maxit+2]
    Scratch scr;
    int* host_flag;           // mapped pinned int: iteration at which the solve stopped
    int part;                 // 0: all work items; 1: interior chunks; 2: the two edge chunks
                              // (interior runs while the seams are in flight)
    unsigned long long cond;  // CUDA graph while-loop handle (0: not in a graph)
    P2P p2p;                  // RESID / PCGA: mailbox transport (nranks == 0: off)
    int nopub;                // RESID under P2P with the field-aligned term: k_aniso publishes
    int curv;                 // NC = 3: + kappa_P (2/r^2, 1/(r sin)^2, 1/(r sin)^2) u_m (NEXT-2, R31)
    // PCGA, scalar: the field-aligned term fused into kernel A when ca != nullptr
    const double* ca;         // corner coefficients [3][nl][nt][np] (a, b, e)
    const double* ca_hi;      // r-slabs: corner plane nl (rank+1's plane 0) [3][plane], or nullptr
    const double* ivr;        // [nl] 1 / (rC^2 dr)
};

struct StreamArgs {  // kernel B
    Geo g;
    int ncomp;
    double* r;
    const double* q;
    const double* dinv;
    PcgState* st;
    double* rho_hist;
    double* sigma_hist;
    double* rr_hist;
    Scratch scr;
    int* host_flag;
    unsigned long long cond;
    P2P p2p;
    int aniso;                // the field-aligned term is on: sigma also from MB_C (P2P)
    // the two-iteration x update: on a breakdown in B(k), k even, the pending
    // x += alpha_{k-1} p_{k-1} (p_j lives in p[j & 1]); x == nullptr: none
    double* x;
    const double* p[2];
    int brk_at;               // test hook (MAS_TEST_TRANSPORTS=1 + MAS_TEST_BREAKDOWN_AT=k): B(k) breaks down
    int tnode;                // theta-node placement: kernel B does the pole pass on q first
};

// ---------------------------------------------------------------------------
// Field-aligned conduction (readings R21-R26, DESIGN.md
// §3.4):  V_P (L_par u)_P = sum_{corners c of P} s_c (sr a_c + st b_c + sp e_c),
//   s_c = a_c Dr_c(u) + b_c Dt_c(u) + e_c Dp_c(u)
// with Dr / Dt / Dp the sums of the 4 cell differences across corner c in r /
// theta / phi, sr, st, sp = +-1 the side of P, and the corner coefficients
//   (a, b, e) = sqrt(W_c kpar_c) (b_r/(4 hr), b_t/(4 rF ht), b_p/(4 rF sF hp))
// precomputed once per mas_op_set_aniso (k_aniso_coef), stored at the cell
// whose lower corner c is: ca[3][nl][nt][np].  Single GPU (one r-slab).
// ---------------------------------------------------------------------------
struct AnisoTab {          // 1-D corner metrics (device), 0 on dead corners (R24)
    const double* rF;      // [nl]  r of the lower r-face of plane I
    const double* hr;      // [nl]  rC_I - rC_{I-1}; 0 at the global inner face
    const double* sF;      // [nt]  sin(tF_J); 0 at J = 0
    const double* ht;      // [nt]  tC_J - tC_{J-1}; 0 at J = 0
    const double* hp;      // [np]  centre distance across phi-face K (periodic)
    const double* ivr;     // [nl]  1 / (rC^2 dr) of plane i (the kernel never divides)
};

struct AnisoArgs {
    Geo g;
    int chunk, ntj, ntk, nchunk;  // set by launch_aniso
    int max_blocks;               // capacity of scr.partials (blocks)
    const double* ca;      // [3][nl][nt][np] corner coefficients a, b, e
    const double* ca_hi;   // r-slabs: corner plane nl = rank+1's plane 0, [3][plane]; or nullptr
    const double* ivr;     // AnisoTab::ivr
    Halo u;                // APPLY / RESID: x;  PCGA: p_k (written by kernel A(k)); r-slab
                           // ghost planes -1 / nl (nullptr at a global boundary)
    double* out;           // APPLY: y += L_par x;  RESID: r -= L_par x;  PCGA: q += L_par p
    const double* f;       // RESID: rhs
    const double* dinv;    // RESID: 1/D (for <r, D^-1 r>)
    PcgState* st;
    Scratch scr;
    unsigned long long cond;
    P2P p2p;               // P2P transport: waits for every rank's A(k), publishes MB_C / MB_B
};

// launchers (kernels.cu)
int stencil_blocks(const Geo& g, int chunk);
// first: kernel A of iteration 1 (its own instantiation)
cudaError_t launch_stencil(int mode, int ncomp, const StencilArgs& a, cudaStream_t s,
                           bool first = false);
cudaError_t launch_pcg_b(const StreamArgs& a, int nblocks, cudaStream_t s);
// stacked PCG over several operators (mas_stack_solve, NEXT-2 R34): the
// PcgState of every block; k_stack_sum replaces the doubles [off, off+cnt) of
// each by their sum over the blocks (block order: deterministic)
constexpr int kMaxStack = 8;
struct StackStates {
    PcgState* st[kMaxStack];
    int n;
};
cudaError_t launch_stack_sum(const StackStates& s, int off, int cnt, cudaStream_t stream);
// theta-node placement (NEXT-2): average the pole rows (local rows 0, g.nt-1)
// of planes [plane_lo, plane_lo + nplanes) of every component over phi with
// dp weights (dinv != nullptr: also dinv = 1 / average, ncomp = 1)
cudaError_t launch_pole_avg(const Geo& g, int ncomp, double* y, double* dinv, int plane_lo, int nplanes,
                            cudaStream_t s);
// finite, positive, non-constant test values (kernel-replay timing)
cudaError_t launch_fill_test(double* a, long long n, cudaStream_t s);
cudaError_t launch_l2_sweep(const double* a, long long n, double* sink, cudaStream_t s);
// the init's <f,f>, <r,r>, <r,D^-1 r> into PcgState (after the pole average of r)
cudaError_t launch_init_dots(const Geo& g, int ncomp, const double* f, const double* r, const double* dinv,
                             Scratch scr, PcgState* st, int nblocks, cudaStream_t s);
cudaError_t launch_diag(const Geo& g, Halo kappa, TRows tkappa, const double* c, double* D,
                        double* dinv, int* bad, cudaStream_t s);
// out[side][c][i][k] = in[c][i][side ? nt-1 : 0][k]: a field's first / last theta rows
cudaError_t launch_pack_rows(const Geo& g, int ncomp, const double* in, double* out, cudaStream_t s);
cudaError_t launch_dirichlet(const Geo& g, int ncomp, const double* kappa, const double* ub,
                             int outer, double* f, cudaStream_t s);
cudaError_t launch_dot(const Geo& g, int ncomp, const double* a, const double* b, Scratch scr,
                       double* out, int nblocks, cudaStream_t s);
// out[t] = sum_r stage[8r + t], t < n, ranks summed in rank order (virtual-rank allreduce)
cudaError_t launch_rank_sum(double* out, const double* stage, int nranks, int n, cudaStream_t s);

// out[m * nl + i] = sum_{j,k} w[j][k] x[m][i][j][k] (the paper's sum0, Listings 3-5)
cudaError_t launch_radial_sums(const Geo& g, int ncomp, const double* x, const double* w, double* out,
                               cudaStream_t s);
// launchers (aniso.cu)
cudaError_t launch_aniso(int mode, const AnisoArgs& a, cudaStream_t s);
// ca from kpar [nl][nt][np] and bhat [3][nl][nt][np]; *bad |= 1 on a negative
// or non-finite kpar / non-finite b
cudaError_t launch_aniso_coef(const Geo& g, AnisoTab t, const double* kpar, const double* bhat,
                              double* ca, int* bad, cudaStream_t s);
// D += (1/V) sum_c (sr a + st b + sp e)^2 (R26); dinv = 1/D; *bad |= 1 if D <= 0
cudaError_t launch_aniso_diag(const Geo& g, const double* ca, const double* ca_hi, double* D,
                              double* dinv, int* bad, cudaStream_t s);

void set_last_error(const std::string& msg);

// Per-device one-time launch setup.  cudaFuncSetAttribute (the dynamic
// shared-memory opt-in) is per device and virtual ranks launch from several
// host threads: each call site keeps one bit per device in an atomic word
// (setting the attribute twice is harmless; 64 devices per process).
struct DeviceOnce {
    std::atomic<unsigned long long> done{0};
    template <class F>
    cudaError_t run(F&& f) {
        int dev = 0;
        cudaError_t e = cudaGetDevice(&dev);
        if (e != cudaSuccess) return e;
        const unsigned long long bit = 1ull << (dev & 63);
        if (done.load(std::memory_order_acquire) & bit) return cudaSuccess;
        e = f();
        if (e == cudaSuccess) done.fetch_or(bit, std::memory_order_acq_rel);
        return e;
    }
};
// SM count of the current device (cached per device, thread-safe)
inline int device_sms() {
    static std::atomic<int> cache[64];
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) return 148;
    int v = cache[dev & 63].load(std::memory_order_relaxed);
    if (v > 0) return v;
    if (cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || v <= 0) v = 148;
    cache[dev & 63].store(v, std::memory_order_relaxed);
    return v;
}

}  // namespace mas
