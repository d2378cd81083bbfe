/*
 * mas_pcg.h — C ABI of the B200-native MAS implicit-parabolic PCG library.
 *
 * What the library computes.  The MAS solar MHD code (Caplan, Stulajter &
 * Linker 2023, PAPER.md) uses "a logically rectangular non-uniform staggered
 * spherical grid and finite-difference discretizations with a combination of
 * explicit and implicit time-stepping methods" and is "highly memory-bound"
 * (§III).  Its hot loop is the "viscosity solver iterations" with
 * GPU peer-to-peer halo exchanges (Fig. 4; §V-C),
 * i.e. a Krylov solve of the implicit parabolic operators (ref. [25],
 * P:1212-1216).  The paper gives no formula; the operator, boundary handling,
 * preconditioner and stopping rule are the readings R1..R16 of DESIGN.md §3
 * (SURVEY.md §8(c)), summarised here:
 *
 *   (L u)_P = c_P u_P + (1/V_P) sum_{faces f of P} G_f (u_P - u_N(f))
 *   G_f = kappa_f g_f,  kappa_f = (kappa_P + kappa_N)/2,  midpoint FD metrics
 *   periodic phi, zero-flux pole / theta-wall faces, r-faces Dirichlet
 *   (homogeneous, half-cell distance) or Neumann;
 *   <a,b> = sum_m sum_P V_P a_mP b_mP;  Jacobi (diagonal) preconditioner;
 *   stop when ||r_k||_V <= tol * ||f||_V.
 *
 * Conventions for every call:
 *   - Per-cell arrays are fp64, C order [comp][i=r][j=theta][k=phi] (phi
 *     fastest), interior cells of the caller's LOCAL r-slab only (no ghosts),
 *     16-byte aligned.  Pointers may be device pointers or host pointers
 *     (pageable or pinned); host pointers are staged through library-owned
 *     device buffers, device pointers are used in place.
 *   - 1-D mesh arrays are host pointers, copied at create.
 *   - Handles are opaque and library-owned.  After a call returns the library
 *     keeps no user pointer.
 *   - Setup/update/apply/rhs calls are asynchronous on the given stream;
 *     mas_pcg_solve returns when the solve is complete (it reports the
 *     iteration count).  Stream 0 means the legacy default stream.
 *   - No exception crosses the ABI.  On failure the status is returned and
 *     mas_last_error() gives a thread-local detail string.
 *   - With a mas_dist_t (multi-GPU, one process per GPU, r-slab
 *     decomposition), every call is collective over the ranks: all ranks call
 *     the same functions in the same order.
 */
#ifndef MAS_PCG_H
#define MAS_PCG_H

#include <cuda_runtime_api.h>

#if defined(__GNUC__)
#define MAS_API __attribute__((visibility("default")))
#else
#define MAS_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

typedef struct mas_grid mas_grid_t;
typedef struct mas_op mas_op_t;
typedef struct mas_stack mas_stack_t;

typedef enum {
    MAS_OK = 0,
    MAS_NOT_CONVERGED = 1, /* warning: x holds the last iterate               */
    MAS_ERR_ARG = 2,       /* invalid argument / mesh / coefficient           */
    MAS_ERR_CUDA = 3,
    MAS_ERR_NCCL = 4,
    MAS_ERR_NOMEM = 5,
    MAS_ERR_BREAKDOWN = 6  /* <p, L p>_V <= 0 or non-finite                    */
} mas_status_t;

typedef enum { MAS_BC_DIRICHLET = 0, MAS_BC_NEUMANN = 1 } mas_bc_t;
enum { MAS_POLE_NORTH = 1, MAS_POLE_SOUTH = 2 };

/* Multi-GPU description.  NULL => single GPU.  nccl_id: 128 bytes from
 * mas_comm_unique_id() on rank 0, broadcast by the caller (e.g. with
 * torch.distributed).  The current CUDA device is used.  nranks == 1 with a
 * real id creates a 1-rank NCCL communicator: the op then runs the
 * multi-GPU (NCCL) iteration loop on one GPU (the NCCL code path's check).
 * NCCL waits inside mas_pcg_solve poll ncclCommGetAsyncError and give up
 * after MAS_COMM_TIMEOUT_S seconds (default 600): the communicators are
 * aborted and MAS_ERR_NCCL returned instead of hanging. */
typedef struct {
    int nranks;
    int rank;
    unsigned char nccl_id[128];
} mas_dist_t;

/* Rank 0 only: a fresh NCCL unique id for mas_dist_t.nccl_id. */
MAS_API mas_status_t mas_comm_unique_id(unsigned char out[128]);

/* Create the grid (reading R1: the node/"main" mesh = cell faces, the
 * half mesh = cell centres; "staggered spherical grid").
 *   r_node[nr+1], r_half[nr], t_node[nt+1], t_half[nt], p_node[np+1],
 *   p_half[np]: strictly increasing, half[i] in (node[i], node[i+1]).
 *   t_node within [0, pi]; MAS_POLE_NORTH requires t_node[0] == 0,
 *   MAS_POLE_SOUTH requires |t_node[nt] - pi| <= 4 eps.  Pole faces and
 *   non-pole theta walls carry no flux (R5).
 *   periodic_phi must be 1 and p_node[np]-p_node[0] must equal 2 pi to
 *   1e-12 relative (R7); np must be even (16-byte phi pairs).
 *   nr >= nranks.  On a mas_dist_t each rank owns the r-slab given by
 *   mas_grid_local_extent (rank p: nr/P + (p < nr%P) planes).
 * Errors: MAS_ERR_ARG (validation; checked before any device work),
 *         MAS_ERR_CUDA, MAS_ERR_NCCL, MAS_ERR_NOMEM. */
MAS_API mas_status_t mas_grid_create(int nr, int nt, int np,
                             const double* r_node, const double* r_half,
                             const double* t_node, const double* t_half,
                             const double* p_node, const double* p_half,
                             int pole_flags, int periodic_phi,
                             const mas_dist_t* dist, mas_grid_t** out);

/* (r, theta) decomposition (the north_star's "slabs in
 * r (and in theta where needed)"; the paper's domain decomposition with
 * halo exchanges).  Same mesh arguments and checks as
 * mas_grid_create; dist->nranks = pr * ptheta with ptheta >= 1 dividing it.
 * Rank = rr * ptheta + rt (theta fastest): rank rt of r-slab rr owns r-planes
 * [i0, i0 + nr_local) (the partition of nr over pr) and theta rows
 * [j0, j0 + nt_local) (the partition of nt over ptheta), every phi.  Every
 * per-cell array of every later call on this grid is then the local block
 * [comp][nr_local][nt_local][np].  Needs nr >= pr and nt >= ptheta.
 * ptheta == 1 is mas_grid_create.  The theta-ghost rows are exchanged by the
 * library: packed copies over the grid's communicator at setup / apply / init
 * and in the NCCL loop; read in place from the theta neighbours' arrays by
 * kernel A under the P2P transport (mas_op_enable_p2p).
 * Errors: as mas_grid_create; MAS_ERR_ARG if ptheta does not divide nranks. */
MAS_API mas_status_t mas_grid_create_2d(int nr, int nt, int np,
                             const double* r_node, const double* r_half,
                             const double* t_node, const double* t_half,
                             const double* p_node, const double* p_half,
                             int pole_flags, int periodic_phi,
                             const mas_dist_t* dist, int ptheta, mas_grid_t** out);

/* This rank's block of a 2-D decomposition: r-planes [i0, i0 + nr_local),
 * theta rows [j0, j0 + nt_local). */
MAS_API mas_status_t mas_grid_local_extent_2d(const mas_grid_t* g, int* i0, int* nr_local,
                                              int* j0, int* nt_local);

/* The r-slab partition without a grid (host only, no device work): rank
 * owns nr/nranks + (rank < nr % nranks) planes starting at *i0 (SURVEY.md
 * §8(e)).  Lets a caller size its slab buffers before mas_grid_create.
 * Errors: MAS_ERR_ARG unless 1 <= nranks <= nr and 0 <= rank < nranks. */
MAS_API mas_status_t mas_partition(int nr, int nranks, int rank, int* i0, int* nr_local);

/* First global r-plane and number of planes owned by this rank. */
MAS_API mas_status_t mas_grid_local_extent(const mas_grid_t* g, int* i0, int* nr_local);

MAS_API mas_status_t mas_grid_destroy(mas_grid_t* g);

/* Set up the operator of ncomp (1: conduction, 3: viscosity, R13)
 * uncoupled components sharing kappa (>= 0) and mass c (>= 0; NULL => 0),
 * both [nr_local][nt][np].  Copies kappa and c, computes the Jacobi
 * diagonal D = c + (1/V) sum_f G_f (R8) and exchanges the static kappa / D
 * seams once.  bc_r_inner / bc_r_outer: r-boundary conditions (R3).
 * Errors: MAS_ERR_ARG if ncomp not 1 or 3, a coefficient is negative or
 * non-finite, or some D_P <= 0 (checked on the device; this call then
 * synchronises the stream). */
MAS_API mas_status_t mas_op_setup(mas_grid_t* g, int ncomp, const double* kappa,
                          const double* mass, mas_bc_t bc_r_inner,
                          mas_bc_t bc_r_outer, cudaStream_t stream,
                          mas_op_t** out);

/* Variable placement on MAS's staggered mesh (the
 * paper's "staggered spherical grid").  MAS_PLACE_CELL: unknowns
 * at cell centres (rC, tC, pC) -- mas_op_setup.  MAS_PLACE_THETA_NODE:
 * unknowns at (rC_i, tF_j, pC_k), j = 0..nt, on the theta main mesh, whose
 * rows 0 and nt lie ON the poles (readings R29-R30): every
 * per-cell array of the op is then [comp][nr_local][nt+1][np]; a pole row
 * holds ONE value per radius, stored replicated over phi.  The operator is
 * the same L = c + (1/V) div(kappa grad) on the dual theta cells
 * [tC_{j-1}, tC_j]; a pole's equation is the balance of its polar cap
 * (theta in [0, tC_0]), the phi sum of its slices' fluxes to row 1 -- the
 * paper's per-radius sum0 array reduction (Listings 3-5, P:428-445,
 * P:592-645), done on the GPU after every stencil pass (k_pole_avg; inside a
 * solve's iterations kernel B forms the caps of q itself).
 * kappa and c may vary over a pole row's slots (each slot is a cap slice);
 * rhs and x0 pole rows are taken as one value (x0's are replaced by their
 * dp-weighted phi average; rhs must be phi-constant there).  Needs both pole
 * flags, nt >= 2 and ptheta == 1; r-slabs run the NCCL loop (no P2P, no
 * field-aligned term, no single-reduction loop).  Outputs of apply / diag /
 * dirichlet_rhs / solve have phi-constant pole rows.
 * Errors: as mas_op_setup; MAS_ERR_ARG for an unknown placement or a grid
 * without both poles. */
/* MAS_PLACE_R_NODE / MAS_PLACE_PHI_NODE (readings R32-R33):
 * the face-centred locations of MAS's staggered velocity components, as a
 * scalar unknown of the same operator.  r nodes: unknowns at (rF_i, tC, pC),
 * i = 1..nr-1, control volume the dual r cell [rC_{i-1}, rC_i], the boundary
 * nodes rF_0 / rF_nr carrying the Dirichlet values (ub of the Dirichlet
 * helper) or no flux; arrays [comp][nr-1][nt][np]; one rank only.  phi nodes:
 * unknowns at (rC, tC, pF_k), k = 0..np-1, control volume the dual phi cell
 * [pC_{k-1}, pC_k] (periodic); arrays [comp][nl][ntl][np]; any r-slab / (r,
 * theta) decomposition on the NCCL loop.  Both: no P2P, L_par, single-
 * reduction loop or curvature terms. */
enum { MAS_PLACE_CELL = 0, MAS_PLACE_THETA_NODE = 1, MAS_PLACE_R_NODE = 2, MAS_PLACE_PHI_NODE = 3 };
MAS_API mas_status_t mas_op_setup_placed(mas_grid_t* g, int ncomp, int placement, const double* kappa,
                                         const double* mass, mas_bc_t bc_r_inner,
                                         mas_bc_t bc_r_outer, cudaStream_t stream, mas_op_t** out);

/* Replace kappa and c (e.g. kappa = T^{5/2} each implicit step); same checks. */
MAS_API mas_status_t mas_op_update(mas_op_t* op, const double* kappa, const double* mass,
                           cudaStream_t stream);

/* y = L x with homogeneous boundary conditions.  x, y: [ncomp][nr_local][nt][np]. */
MAS_API mas_status_t mas_op_apply(const mas_op_t* op, const double* x, double* y,
                          cudaStream_t stream);

/* Jacobi diagonal D (before inversion), [nr_local][nt][np]. */
MAS_API mas_status_t mas_op_diag(const mas_op_t* op, double* D, cudaStream_t stream);

/* f += (1/V_P) G_b u_b on Dirichlet r-faces.  ub_inner / ub_outer:
 * [ncomp][nt][np] boundary values or NULL (homogeneous); ignored on a
 * Neumann boundary and on ranks that do not own that boundary. */
MAS_API mas_status_t mas_op_dirichlet_rhs(const mas_op_t* op, const double* ub_inner,
                                  const double* ub_outer, double* f_inout,
                                  cudaStream_t stream);

/* <a,b>_V over all ranks (R9).  Synchronises the stream. */
MAS_API mas_status_t mas_op_dot(const mas_op_t* op, const double* a, const double* b,
                        double* out, cudaStream_t stream);

/* Jacobi-PCG solve of L x = rhs (R10-R12): x in = x0, out = solution.
 *   tol >= 0: stop when ||r_k||_V <= tol ||rhs||_V (k = 0 included);
 *   maxit >= 0: at most maxit L*p products.
 *   iters: products used; relres: ||r||_V/||rhs||_V (recursive residual);
 *   res_hist: NULL or host array of maxit+1 doubles, ||r_k||_V, k=0..iters.
 * Returns MAS_OK, MAS_NOT_CONVERGED (x = last iterate) or MAS_ERR_BREAKDOWN
 * (x = iterate before the breaking step), or an error.  rhs == 0 gives
 * x = 0, iters = 0.  Blocks until done. */
MAS_API mas_status_t mas_pcg_solve(const mas_op_t* op, const double* rhs, double* x,
                           double tol, int maxit, int* iters, double* relres,
                           double* res_hist, cudaStream_t stream);

/* Collective (all ranks, after mas_op_setup): switch this op's PCG iteration
 * loop from NCCL to the P2P transport over NVLink / NVSwitch peer memory.
 * Multi-GPU PCG needs two exchange steps per iteration (
 * the paper's halo exchanges use GPU peer-to-peer transfers, P:1005-1007,
 * Fig. 4):
 *   - seams: kernel A reads the r-neighbours' edge planes of r_{k-1} and
 *     p_{k-1} in place from their device memory (no send/recv, no ghost copy);
 *   - the two scalar allreduces: the reducing kernel's last block writes its
 *     rank-local partials into every rank's mailbox (one-shot NVLink stores
 *     + a sequence number); the consuming kernel sums all ranks' entries in
 *     rank order, so every rank gets identical bits and the same stop
 *     decision.  The loop then runs as one CUDA graph per rank with no host
 *     round trip.
 * Setup uses CUDA IPC (cudaIpcGetMemHandle / cudaIpcOpenMemHandle) on the
 * library-owned r, p and mailbox buffers, with the handles all-gathered over
 * the grid's NCCL communicator; the init residual, op setup/update seams and
 * mas_op_dot keep NCCL.  With one rank the mailbox path runs against itself.
 * With the single-reduction loop switched on BEFORE this call, its ping-pong
 * buffers are mapped too: each of its kernels publishes its 3 partial sums
 * to every rank's mailbox (two slots alternating by parity) and the next
 * kernel sums them there -- NEXT-1's allreduce fused into the kernels.
 * Errors: MAS_ERR_CUDA on every rank if any rank cannot map its peers (the op
 * then keeps the NCCL loop); MAS_ERR_NCCL.  A mailbox wait longer than 60 s
 * traps the kernel (fails loudly rather than hanging). */
MAS_API mas_status_t mas_op_enable_p2p(mas_op_t* op, cudaStream_t stream);

/* Single-reduction PCG (the paper's lesson that
 * fused, asynchronous kernels win).  on != 0: later
 * mas_pcg_solve calls on this op run the Chronopoulos-Gear form of the same
 * Jacobi-PCG (reading R28): ONE fused kernel and ONE
 * reduction (<r,D^-1 r>, <L D^-1 r, D^-1 r>, <r,r>) per iteration instead of
 * two of each:
 *   s = w + beta s;  r -= alpha s;  p = D^-1 r_old + beta p;  x += alpha p;
 *   w = L D^-1 r  (r, s recomputed on the halo cells, so no extra pass).
 * Same arguments, stopping rule (R10) and counting (R11) as the standard
 * loop; iterates equal it in exact arithmetic (rounding differs: parity band
 * +-2 iterations, x <= 1e-9).  HBM traffic per iteration: 13 passes scalar
 * (as the two-kernel loop), 33 passes for 3 components (31).  Allocates 3
 * more vectors.  On r-slabs the NCCL loop runs ONE 3-double allreduce per
 * iteration (two in the two-kernel loop) plus the seams of r, w and s; kernel
 * k+1 takes the stop / alpha / beta decision from the allreduced sums, so
 * every rank decides alike.  Over the P2P transport (mas_op_enable_p2p
 * called after this) the reduction happens in the kernels through the
 * mailbox, and the r, w, s halos are read in place.  on == 0 restores the
 * two-kernel loop.
 * Errors: MAS_ERR_ARG after mas_op_enable_p2p of an op without the loop on,
 * ptheta > 1, the field-aligned term, the theta-node placement or the
 * curvature terms; MAS_ERR_NOMEM. */
MAS_API mas_status_t mas_op_set_single_reduction(mas_op_t* op, int on);

/* Vector-Laplacian curvature terms (reading R31,
 * DESIGN.md §3.7).  For the 3-component viscosity operator, whose components
 * are the spherical (v_r, v_theta, v_phi) (R13), on != 0 adds the terms of the
 * vector Laplacian in the SAME component:
 *   (L v)_r += kappa_P 2/rC^2 v_r,  (L v)_theta += kappa_P v_theta/(rC sin tC)^2,
 *   (L v)_phi += kappa_P v_phi/(rC sin tC)^2        (cell centres, all >= 0)
 * in apply, the residual and every iteration (the terms coupling different
 * components are not included).  The Jacobi preconditioner stays the shared
 * 7-point diagonal.  Errors: MAS_ERR_ARG unless ncomp == 3 and the placement
 * is cell-centred. */
MAS_API mas_status_t mas_op_set_curvature(mas_op_t* op, int on);

/* 1 if the op's solve uses the single-reduction loop, 0 if not, -1 if NULL. */
MAS_API int mas_op_single_reduction(const mas_op_t* op);

/* Transport of the op's PCG loop: 0 NCCL (or one GPU), 1 P2P; -1 if op is NULL. */
MAS_API int mas_op_transport(const mas_op_t* op);

/* Collective measurement of the NCCL loop's exchange steps on this op
 * (SURVEY.md §8(d) "seam bytes / seam time vs 900 GB/s; allreduce latency"):
 * reps rounds of the per-iteration seams (the r and p edge planes to the
 * r-neighbours, grouped ncclSend/ncclRecv) and reps 2-double ncclAllReduce,
 * timed with CUDA events on the stream.  seam_us / allreduce_us: average per
 * round; seam_bytes: bytes this rank sends + receives per round.  Without a
 * communicator all three are 0.  The op's r / p contents are clobbered
 * (call it outside a solve).  Errors: MAS_ERR_ARG (reps < 1, null pointers),
 * MAS_ERR_NCCL, MAS_ERR_CUDA. */
MAS_API mas_status_t mas_op_comm_bench(mas_op_t* op, int reps, double* seam_us,
                                       double* allreduce_us, double* seam_bytes,
                                       cudaStream_t stream);

/* Kernel launches issued by the last mas_pcg_solve on this op (its CUDA path
 * evidence; includes early-exit launches after convergence). */
MAS_API long long mas_op_launch_count(const mas_op_t* op);

/* Per-kernel timing of mas_pcg_solve: when on, every kernel A / kernel B
 * launch of a solve is bracketed by CUDA events on the solve stream. */
MAS_API mas_status_t mas_op_set_profiling(mas_op_t* op, int on);

/* Average device time (ms) of kernel A (fused p-update + stencil + <p,q>)
 * and kernel B (r-update + Jacobi + two dots) over the iterations 1..iters
 * of the last profiled solve; n = number of iterations averaged. */
MAS_API mas_status_t mas_op_kernel_times(const mas_op_t* op, double* a_ms, double* b_ms, int* n);

/* Device time of the iteration kernels, one GPU (measurement helper for
 * bench.py; SURVEY.md §8(d) "ncu per kernel ... time"): reps launches of
 * kernel A (or the single-reduction kernel), kernel B and the L_par kernel,
 * each captured in a CUDA graph, each launch preceded by an L2 flush and a
 * reset of the PCG state; the same graph without the kernels is timed too
 * and subtracted (CUDA events on the stream);
 * a_ms / b_ms / c_ms: average per launch (0 for a kernel the op does not
 * run).  The op's work vectors and PCG state are overwritten with test values
 * (call between solves); the caller's arrays are not touched.
 * Errors: MAS_ERR_ARG (reps < 1, null pointers, a grid with a mas_dist_t),
 * MAS_ERR_CUDA. */
MAS_API mas_status_t mas_op_kernel_bench(mas_op_t* op, int reps, double* a_ms, double* b_ms,
                                         double* c_ms, cudaStream_t stream);

/* Field-aligned (anisotropic) thermal conduction.
 * MAS conducts heat along the magnetic field; the paper names the
 * thermodynamic model of its test problem and the implicit
 * parabolic Krylov schemes of ref. [25] but prints no formula,
 * so the term is the reading R21-R26 of DESIGN.md §3.4:
 *   L = L_iso + L_par,  L_par u = -div(kpar b (b . grad u)) in the symmetric
 *   corner form  V_P (L_par u)_P = sum_{corners c of P} W_c kpar_c (b_c.g_c(u))
 *   (b_c . dg_c/du_P), g_c the 8-cell corner gradient, W_c the corner dual
 *   volume; corners on the r boundaries, poles and theta walls carry no
 *   weight (no field-aligned flux leaves the domain).
 * kpar: [nr][nt][np] >= 0 and bhat: [3][nr][nt][np] (b_r, b_theta, b_phi,
 * used as given) at the LOWER corner (rF_i, tF_j, pF_k) of each cell; the
 * entries of boundary corners (i = 0 or j = 0) are ignored.  Device or host
 * pointers; the library keeps only the derived corner coefficients
 * (3 fields).  The Jacobi diagonal gains the term's diagonal (R26); apply,
 * the residual and every PCG iteration add it (one extra kernel per
 * iteration).  kpar == NULL switches the term off.  Synchronises the stream.
 * On an r-slab grid (mas_grid_create with a mas_dist_t) the call is
 * collective: each rank passes its local slab of kpar / bhat; the corner
 * plane above the slab comes from rank+1.  The p_k planes of the neighbours
 * are exchanged after every kernel A (NCCL loop) or read in place once every
 * rank's kernel A has published (P2P transport; the term's sigma part goes
 * through its own mailbox slot).
 * Errors: MAS_ERR_ARG if ncomp != 1, the grid has ptheta > 1, kpar < 0 or
 * non-finite, b non-finite, or some D_P <= 0 (the term is then off). */
MAS_API mas_status_t mas_op_set_aniso(mas_op_t* op, const double* kpar, const double* bhat,
                                      cudaStream_t stream);

/* 1 if the iteration's L_par runs inside kernel A (opt-in: MAS_LPAR_FUSED=1
 * in the environment at mas_op_setup; kernel A then stages the corner
 * coefficients of each r-plane, computes the tile's corner products once and
 * adds L_par p to q and <p, L_par p> to sigma, so p_k and q skip the extra
 * round trip to HBM -- but the two extra barriers per plane make it slower
 * than the separate kernel), 0 if the separate k_aniso kernel
 * runs (the default, or the term is off), -1 if op is NULL.  The init
 * residual and mas_op_apply use the separate kernel either way. */
MAS_API int mas_op_aniso_fused(const mas_op_t* op);

/* Average device time (ms) of the L_par kernel over the last profiled solve
 * (mas_op_set_profiling); 0 when the term is off or fused into kernel A. */
MAS_API mas_status_t mas_op_aniso_time(const mas_op_t* op, double* ms);

/* Per-radius array reduction, the paper's Listings 3-5 ("sum0(i) =
 * sum0(i) + array(i,j)*...", §IV; MAS uses such sums
 * e.g. for phi-averaged pole values).  Reading R27:
 * the elided factor is an angular weight, so
 *   out[m][i] = sum_{j,k} w[j][k] x[m][i][j][k]
 * for every component m and LOCAL r-plane i of this rank.  x [ncomp][nl][nt][np],
 * w [nt][np] (16-byte aligned), out [ncomp][nl]; each may be a host or a
 * device pointer (a host out makes the call synchronous).  Deterministic:
 * one fixed-order block reduction per plane, no atomics (the paper's DC
 * rewrite replaced the OpenACC atomics by a reduce).  Local to each rank (no
 * communication: r-slab ranks own whole planes).
 * Errors: MAS_ERR_ARG on a null pointer or a grid with ptheta > 1. */
MAS_API mas_status_t mas_op_radial_sums(const mas_op_t* op, const double* x, const double* w,
                                        double* out, cudaStream_t stream);

/* Stacked solve (reading R34 in DESIGN.md §3.9):
 * ONE Jacobi-PCG on the stacked vector of several operators, the block-
 * diagonal operator diag(L_1, .., L_n) with the summed inner product
 * <a,b> = sum_b <a_b, b_b>_V of the blocks.  MAS solves its viscous step for
 * the velocity vector with each component at its own staggered location
 * (P:208-209): v_r at r nodes (MAS_PLACE_R_NODE), v_theta at theta nodes
 * (MAS_PLACE_THETA_NODE), v_phi at phi nodes (MAS_PLACE_PHI_NODE), each its
 * own mas_op_t (own kappa, c, boundary conditions and array shape); the
 * curvature terms of R31 go into each block's c.  alpha, beta and the stop
 * test ||r||_V <= tol ||rhs||_V are those of the stacked vector.
 *   mas_stack_create: ops[0..nops-1], 1 <= nops <= 8, distinct, each on one
 *     GPU without a mas_dist_t, no P2P, no single-reduction loop, no
 *     field-aligned term (MAS_ERR_ARG otherwise).  The stack keeps the op
 *     pointers (not the ops): destroy the stack before its ops.
 *   mas_stack_solve: rhs[b], x[b] arrays of op b's shape ([comp][nl][nt][np]
 *     of its placement), device or host (staged like mas_pcg_solve); x in =
 *     x0, out = solution;
 *     tol, maxit, iters, relres, res_hist as mas_pcg_solve (the stacked
 *     residual).  Runs on `stream` (every op's work goes there; the single-GPU
 *     CUDA-graph loop with one k_stack_sum node after each kernel round).
 *     Blocks until done.  The ops' own solve state is overwritten. */
MAS_API mas_status_t mas_stack_create(mas_op_t* const* ops, int nops, mas_stack_t** out);
MAS_API mas_status_t mas_stack_solve(mas_stack_t* stack, const double* const* rhs, double* const* x,
                                     double tol, int maxit, int* iters, double* relres,
                                     double* res_hist, cudaStream_t stream);
MAS_API mas_status_t mas_stack_destroy(mas_stack_t* stack);

MAS_API mas_status_t mas_op_destroy(mas_op_t* op);

MAS_API const char* mas_status_string(mas_status_t s);
MAS_API const char* mas_last_error(void);

/* Library/build identification: "maspcg <version> sm_100a". */
MAS_API const char* mas_version(void);

#ifdef __cplusplus
}
#endif
#endif /* MAS_PCG_H */
