/*
 * mas_ref.h — ORACLE for the MAS implicit-parabolic PCG path.
 *
 * TEST INFRASTRUCTURE ONLY.  Nothing in the product path
 * (paper_conf_ipps_caplansl23_b200/, include/) may include, link or call this.
 * Only tests/, __graft_entry__.smoke() and bench.py (cpu_baseline leg and
 * --impl reference) may load it.  It shares no source with the CUDA path.
 *
 * What it computes (the paper, Caplan, Stulajter & Linker 2023, prints no
 * formula; every definition below is a reading frozen in SURVEY.md §8(c) and
 * DESIGN.md §3, R1..R16):
 *   P:208-213 (§III)  "logically rectangular non-uniform staggered spherical
 *                      grid", "finite-difference discretizations", implicit
 *                      time stepping, "highly memory-bound".
 *   P:1027-1030 (Fig.4) "viscosity solver iterations" with halo exchanges.
 *   P:1212-1216 ([25])  implicit parabolic schemes "with krylov solvers".
 *
 * Arithmetic: IEEE fp64, compiled -O2 -ffp-contract=off (no FMA contraction,
 * no fast-math).  Reductions are summed per r-plane in (j,k) order, planes in
 * increasing i, then components, so results are independent of the OpenMP
 * thread count.
 *
 * Layout: C order [comp][i=r][j=theta][k=phi], phi fastest (reading R15).
 * All pointers are HOST pointers.  Return value 0 = OK; see codes below.
 */
#ifndef MAS_REF_H
#define MAS_REF_H

#ifdef __cplusplus
extern "C" {
#endif

enum { MAS_REF_OK = 0, MAS_REF_NOT_CONVERGED = 1, MAS_REF_ERR_ARG = 2,
       MAS_REF_ERR_BREAKDOWN = 6 };
enum { MAS_REF_DIRICHLET = 0, MAS_REF_NEUMANN = 1 };

/* Grid description (R1): faces ("node"/main mesh) and centres ("half" mesh).
 * rF[nr+1], rC[nr], tF[nt+1], tC[nt], pF[np+1], pC[np].
 * bc_inner / bc_outer: r-boundary conditions (R3).  Theta faces 0 and nt never
 * carry flux: pole faces have zero area, non-pole walls are Neumann (R5). */
typedef struct {
    int nr, nt, np;
    const double *rF, *rC, *tF, *tC, *pF, *pC;
    int bc_inner, bc_outer;
} mas_ref_grid;

void mas_ref_set_threads(int nthreads);

/* Cell volumes V[i][j][k] = rC^2 dr * sin(tC) dt * dp   (R4). */
int mas_ref_volumes(const mas_ref_grid* g, double* V);

/* y = L x for ncomp components sharing kappa, c   (R2, R4-R7, R13).
 * (L u)_P = c_P u_P + (1/V_P) sum_f G_f (u_P - u_N(f)), homogeneous BCs. */
int mas_ref_op_apply(const mas_ref_grid* g, int ncomp, const double* kappa,
                     const double* c, const double* x, double* y);

/* Jacobi diagonal D_P = c_P + (1/V_P) sum_f G_f (Dirichlet faces included) (R8). */
int mas_ref_op_diag(const mas_ref_grid* g, const double* kappa, const double* c,
                    double* D);

/* f += (1/V_P) G_b u_b on Dirichlet r-faces.  ub_inner/ub_outer: [ncomp][nt][np]
 * or NULL (homogeneous).  A boundary whose bc is Neumann ignores its ub. */
int mas_ref_dirichlet_rhs(const mas_ref_grid* g, int ncomp, const double* kappa,
                          const double* ub_inner, const double* ub_outer,
                          double* f);

/* <a,b>_V = sum_m sum_P V_P a_mP b_mP   (R9). */
int mas_ref_dot(const mas_ref_grid* g, int ncomp, const double* a,
                const double* b, double* out);

/* Jacobi-PCG, textbook order (R10-R12).  x: in x0, out solution.
 * iters = number of L*p products in the loop; relres = ||r||_V/||f||_V.
 * res_hist (NULL or maxit+1): ||r_k||_V for k = 0..iters. */
int mas_ref_pcg_solve(const mas_ref_grid* g, int ncomp, const double* kappa,
                      const double* c, const double* f, double* x, double tol,
                      int maxit, int* iters, double* relres, double* res_hist);

/* Single-reduction PCG (NEXT-1, reading R28): the Chronopoulos-Gear form of
 * the same Jacobi-PCG (one inner-product reduction per iteration); same
 * arguments, stopping rule and counting as mas_ref_pcg_solve (iters = index
 * of the residual that met tol = number of L products). */
int mas_ref_pcg_solve_cg1(const mas_ref_grid* g, int ncomp, const double* kappa,
                          const double* c, const double* f, double* x, double tol,
                          int maxit, int* iters, double* relres, double* res_hist);

/* Slab-local operator for a rank owning r-planes [i0, i0+nl) of the global
 * grid g.  kappa_ext and x_ext hold nl+2 planes per component: plane 0 is the
 * ghost copy of global plane i0-1, plane nl+1 of i0+nl (ignored at a global
 * boundary).  c and y hold nl interior planes. */
int mas_ref_op_apply_slab(const mas_ref_grid* g, int i0, int nl, int ncomp,
                          const double* kappa_ext, const double* c,
                          const double* x_ext, double* y);

/* (r, theta) block [i0,i0+nl) x [j0,j0+ntl): kappa_ext [nl+2][ntl+2][np] and
 * x_ext [ncomp][nl+2][ntl+2][np] carry one ghost plane / theta row on each side
 * (ignored where the face is a global boundary, pole or wall); c [nl][ntl][np],
 * y [ncomp][nl][ntl][np].  mas_ref_dot_block: the block's partial <a,b>_V. */
int mas_ref_op_apply_block(const mas_ref_grid* g, int i0, int nl, int j0, int ntl, int ncomp,
                           const double* kappa_ext, const double* c,
                           const double* x_ext, double* y);
int mas_ref_dot_block(const mas_ref_grid* g, int i0, int nl, int j0, int ntl, int ncomp,
                      const double* a, const double* b, double* out);

/* Per-slab partial of <a,b>_V over planes [i0,i0+nl) (a,b interior, nl planes). */
int mas_ref_dot_slab(const mas_ref_grid* g, int i0, int nl, int ncomp,
                     const double* a, const double* b, double* out);

/* The same PCG run on `nranks` virtual r-slabs inside one process: explicit
 * ghost-plane copies between slab buffers, slab-local partial dots summed in
 * rank order.  Models the multi-GPU decomposition. */
int mas_ref_pcg_solve_vranks(const mas_ref_grid* g, int nranks, int ncomp,
                             const double* kappa, const double* c,
                             const double* f, double* x, double tol, int maxit,
                             int* iters, double* relres, double* res_hist);

/* (L x) evaluated only at the listed flat indices idx[s] = m*N + P (component
 * major), for sampled checks at sizes where a full oracle pass is too slow. */
int mas_ref_op_apply_cells(const mas_ref_grid* g, int ncomp, const double* kappa,
                           const double* c, const double* x, long long ncells,
                           const long long* idx, double* out);

/* The r-slab partition: rank p owns n_p = nr/P + (p < nr%P)
 * planes starting at i0_p. */
void mas_ref_partition(int nr, int nranks, int rank, int* i0, int* nl);

/* Field-aligned (anisotropic) conduction, readings
 * R21-R26 (mas_ref.c): y = L_par x with
 *   V_P (L_par u)_P = sum_{corners c of P} W_c kpar_c (b_c.g_c(u)) (b_c.dg_c/du_P),
 * kpar [nr][nt][np] and bhat [3][nr][nt][np] given at the LOWER corner
 * (rF_i, tF_j, pF_k) of cell (i,j,k); boundary corners carry no weight. */
int mas_ref_aniso_apply(const mas_ref_grid* g, int ncomp, const double* kpar,
                        const double* bhat, const double* x, double* y);
/* Diagonal of L_par (R26). */
int mas_ref_aniso_diag(const mas_ref_grid* g, const double* kpar, const double* bhat,
                       double* D);
/* Slab-local L_par (r-slab protocol): x_ext [ncomp][nl+2][nt][np] with ghost
 * planes i0-1 / i0+nl; kpar_ext [nl+1][nt][np], bhat_ext [3][nl+1][nt][np]
 * hold corner planes i0 .. i0+nl; y [ncomp][nl][nt][np]. */
int mas_ref_aniso_apply_slab(const mas_ref_grid* g, int i0, int nl, int ncomp,
                             const double* kpar_ext, const double* bhat_ext,
                             const double* x_ext, double* y);
/* The Jacobi-PCG of mas_ref_pcg_solve on L = L_iso + L_par, D = D_iso + D_par. */
int mas_ref_pcg_solve_aniso(const mas_ref_grid* g, int ncomp, const double* kappa,
                            const double* c, const double* kpar, const double* bhat,
                            const double* f, double* x, double tol, int maxit, int* iters,
                            double* relres, double* res_hist);

/* Per-radius array reduction (the paper's Listings 3-5, "sum0"; reading R27):
 * out[m][i] = sum_{j,k} w[j][k] x[m][i][j][k], w [nt][np], out [ncomp][nr]. */
int mas_ref_radial_sums(const mas_ref_grid* g, int ncomp, const double* x, const double* w,
                        double* out);

#ifdef __cplusplus
}
#endif
/* theta-node placement with pole unknowns (NEXT-2, readings R29-R30,
 * mas_ref.c): arrays [comp][nr][nt+1][np]; rows 0 and nt are the poles (one
 * value per radius, stored replicated over phi); the grid must have tF[0] = 0
 * and tF[nt] = pi.  volumes [nr][nt+1][np]: V of each slot (pole slots: the
 * cap slices rC^2 dr A dp_k). */
int mas_ref_tn_volumes(const mas_ref_grid* g, double* V);
int mas_ref_tn_apply(const mas_ref_grid* g, int ncomp, const double* kappa, const double* c,
                     const double* x, double* y);
int mas_ref_tn_diag(const mas_ref_grid* g, const double* kappa, const double* c, double* D);
int mas_ref_tn_dirichlet_rhs(const mas_ref_grid* g, int ncomp, const double* kappa,
                             const double* ub_inner, const double* ub_outer, double* f);
int mas_ref_tn_dot(const mas_ref_grid* g, int ncomp, const double* a, const double* b, double* out);
int mas_ref_tn_pcg_solve(const mas_ref_grid* g, int ncomp, const double* kappa, const double* c,
                         const double* f, double* x, double tol, int maxit, int* iters,
                         double* relres, double* res_hist);

/* 3-component viscosity with the vector-Laplacian curvature terms (NEXT-2,
 * reading R31): y = L x + kappa_P (2/rC^2 x_r, x_theta/(rC^2 sin^2 tC),
 * x_phi/(rC^2 sin^2 tC)); PCG with the shared 7-point Jacobi diagonal. */
int mas_ref_op_apply_curv(const mas_ref_grid* g, const double* kappa, const double* c,
                          const double* x, double* y);
int mas_ref_pcg_solve_curv(const mas_ref_grid* g, const double* kappa, const double* c,
                           const double* f, double* x, double tol, int maxit, int* iters,
                           double* relres, double* res_hist);

/* Face-centred placements (NEXT-2, readings R32-R33, mas_ref.c):
 * phi nodes: unknowns at (rC, tC, pF_k), k = 0..np-1: the cell-centred
 * operator on the dual phi mesh (faces pC_{k-1}, centres pF_k);
 * r nodes: unknowns at (rF_i, tC, pC), i = 1..nr-1, arrays [comp][nr-1][nt][np];
 * the boundary nodes rF_0 / rF_nr carry the Dirichlet values (or no flux). */
int mas_ref_pn_apply(const mas_ref_grid* g, int ncomp, const double* kappa, const double* c,
                     const double* x, double* y);
int mas_ref_pn_volumes(const mas_ref_grid* g, double* V);
int mas_ref_pn_diag(const mas_ref_grid* g, const double* kappa, const double* c, double* D);
int mas_ref_pn_dirichlet_rhs(const mas_ref_grid* g, int ncomp, const double* kappa,
                             const double* ub_inner, const double* ub_outer, double* f);
int mas_ref_pn_pcg_solve(const mas_ref_grid* g, int ncomp, const double* kappa, const double* c,
                         const double* f, double* x, double tol, int maxit, int* iters,
                         double* relres, double* res_hist);
int mas_ref_rn_volumes(const mas_ref_grid* g, double* V);
int mas_ref_rn_apply(const mas_ref_grid* g, int ncomp, const double* kappa, const double* c,
                     const double* x, double* y);
int mas_ref_rn_diag(const mas_ref_grid* g, const double* kappa, const double* c, double* D);
int mas_ref_rn_dirichlet_rhs(const mas_ref_grid* g, int ncomp, const double* kappa,
                             const double* ub_inner, const double* ub_outer, double* f);
int mas_ref_rn_pcg_solve(const mas_ref_grid* g, int ncomp, const double* kappa, const double* c,
                         const double* f, double* x, double tol, int maxit, int* iters,
                         double* relres, double* res_hist);

/* Stacked PCG over several placed operators (NEXT-2, reading R34,
 * mas_ref.c): MAS's viscosity solve on the staggered mesh -- v_r at r nodes,
 * v_theta at theta nodes, v_phi at phi nodes -- as ONE Jacobi-PCG on the
 * stacked vector (block-diagonal operator, the sum of the blocks' V-weighted
 * inner products).  Block b: grid g[b] (its mesh and r-boundary conditions),
 * placement[b] (MAS_REF_PLACE_*), ncomp[b], kappa[b], c[b] (may be NULL),
 * f[b], x[b] (in: x0, out: the solution). */
#define MAS_REF_PLACE_CELL 0
#define MAS_REF_PLACE_THETA_NODE 1
#define MAS_REF_PLACE_R_NODE 2
#define MAS_REF_PLACE_PHI_NODE 3
#define MAS_REF_MAX_STACK 8
int mas_ref_stacked_pcg_solve(int nblk, const mas_ref_grid* const* g, const int* placement,
                              const int* ncomp, const double* const* kappa, const double* const* c,
                              const double* const* f, double* const* x, double tol, int maxit,
                              int* iters, double* relres, double* res_hist);

#endif
