/*
 * mas_ref.c — ORACLE (test infrastructure only; see mas_ref.h header).
 *
 * Plain, slow, obviously-correct CPU implementation of the discretised MAS
 * implicit parabolic operator and its Jacobi-PCG solve.  Every formula is the
 * reading frozen in SURVEY.md §8(c) / DESIGN.md §3; the paper itself
 * (Caplan et al. 2023) states no formula.
 *
 * Structure: the 1-D metric tables are the plain definitions of §8(c)
 * "1-D metrics"; cell_L() is the per-cell operator written face by face
 * exactly as "(L u)_P = c_P u_P + (1/V_P) sum_f G_f (u_P - u_N(f))";
 * the PCG loop is the textbook order of §8(c) "PCG, exact order".
 * No blocking, fusion or reordering beyond that.
 *
 * Build: gcc -O2 -ffp-contract=off -fopenmp -shared -fPIC (oracle/build.py).
 */
#include "mas_ref.h"

#include <math.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#define TWO_PI (2.0 * 3.14159265358979323846)

void mas_ref_set_threads(int n) {
#ifdef _OPENMP
    if (n > 0) omp_set_num_threads(n);
#else
    (void)n;
#endif
}

/* ---------------------------------------------------------------------------
 * 1-D metric tables (SURVEY §8(c) "1-D metrics"; readings R1, R3, R7).
 * ------------------------------------------------------------------------- */
typedef struct {
    int nr, nt, np;
    double *dr, *dt, *dp;   /* cell widths                                    */
    double *hr;             /* [nr+1] centre distance across r-face i (R3)    */
    double *ht;             /* [nt+1] centre distance across theta-face j     */
    double *hp;             /* [np]   centre distance across phi-face k (wrap)*/
    double *sC, *sF;        /* sin(theta) at centres [nt] and faces [nt+1]    */
} tables;

static void tables_free(tables* T) {
    free(T->dr); free(T->dt); free(T->dp); free(T->hr); free(T->ht);
    free(T->hp); free(T->sC); free(T->sF);
}

static int tables_make(const mas_ref_grid* g, tables* T) {
    int nr = g->nr, nt = g->nt, np = g->np, i, j, k;
    memset(T, 0, sizeof(*T));
    if (nr < 1 || nt < 1 || np < 2) return MAS_REF_ERR_ARG;
    T->nr = nr; T->nt = nt; T->np = np;
    T->dr = malloc(sizeof(double) * nr);
    T->dt = malloc(sizeof(double) * nt);
    T->dp = malloc(sizeof(double) * np);
    T->hr = malloc(sizeof(double) * (nr + 1));
    T->ht = malloc(sizeof(double) * (nt + 1));
    T->hp = malloc(sizeof(double) * np);
    T->sC = malloc(sizeof(double) * nt);
    T->sF = malloc(sizeof(double) * (nt + 1));
    if (!T->dr || !T->dt || !T->dp || !T->hr || !T->ht || !T->hp || !T->sC || !T->sF) {
        tables_free(T);
        return MAS_REF_ERR_ARG;
    }
    for (i = 0; i < nr; i++) T->dr[i] = g->rF[i + 1] - g->rF[i];
    for (j = 0; j < nt; j++) T->dt[j] = g->tF[j + 1] - g->tF[j];
    for (k = 0; k < np; k++) T->dp[k] = g->pF[k + 1] - g->pF[k];
    /* hr: interior faces centre-to-centre; boundary faces half-cell (R3). */
    T->hr[0] = g->rC[0] - g->rF[0];
    for (i = 1; i < nr; i++) T->hr[i] = g->rC[i] - g->rC[i - 1];
    T->hr[nr] = g->rF[nr] - g->rC[nr - 1];
    /* ht only for interior theta faces; faces 0 and nt carry no flux (R5). */
    T->ht[0] = 0.0; T->ht[nt] = 0.0;
    for (j = 1; j < nt; j++) T->ht[j] = g->tC[j] - g->tC[j - 1];
    /* hp: periodic, face 0 lies between cell np-1 and cell 0 (R7). */
    T->hp[0] = g->pC[0] + TWO_PI - g->pC[np - 1];
    for (k = 1; k < np; k++) T->hp[k] = g->pC[k] - g->pC[k - 1];
    for (j = 0; j < nt; j++) T->sC[j] = sin(g->tC[j]);
    T->sF[0] = 0.0; T->sF[nt] = 0.0;       /* never used: pole / wall faces */
    for (j = 1; j < nt; j++) T->sF[j] = sin(g->tF[j]);
    return MAS_REF_OK;
}

/* Cell volume (R4): V = rC^2 dr * sC dt * dp. */
static double cell_V(const mas_ref_grid* g, const tables* T, int i, int j, int k) {
    return g->rC[i] * g->rC[i] * T->dr[i] * T->sC[j] * T->dt[j] * T->dp[k];
}

/* Face geometric conductances (R4), faces numbered:
 *   0: r-face i (toward i-1)   1: r-face i+1 (toward i+1)
 *   2: t-face j (toward j-1)   3: t-face j+1 (toward j+1)
 *   4: p-face k (toward k-1)   5: p-face k+1 (toward k+1), periodic
 *   gR(i;j,k) = rF[i]^2 * sC[j]*dt[j]*dp[k] / hr[i]
 *   gT(j;i,k) = dr[i] * sF[j]*dp[k] / ht[j]
 *   gP(k;i,j) = dr[i] * dt[j] / (sC[j]*hp[k])                                */
static double gR(const mas_ref_grid* g, const tables* T, int iface, int j, int k) {
    return g->rF[iface] * g->rF[iface] * T->sC[j] * T->dt[j] * T->dp[k] / T->hr[iface];
}
static double gT(const tables* T, int i, int jface, int k) {
    return T->dr[i] * T->sF[jface] * T->dp[k] / T->ht[jface];
}
static double gP(const tables* T, int i, int j, int kface) {
    return T->dr[i] * T->dt[j] / (T->sC[j] * T->hp[kface]);
}

enum { FACE_NONE = 0, FACE_INTERIOR = 1, FACE_DIRICHLET = 2 };

/* Face kinds of cell (i,j,k) in the GLOBAL grid (R3, R5, R7). */
static void face_kinds(const mas_ref_grid* g, int i, int j, int kind[6]) {
    kind[0] = (i > 0) ? FACE_INTERIOR
              : (g->bc_inner == MAS_REF_DIRICHLET ? FACE_DIRICHLET : FACE_NONE);
    kind[1] = (i < g->nr - 1) ? FACE_INTERIOR
              : (g->bc_outer == MAS_REF_DIRICHLET ? FACE_DIRICHLET : FACE_NONE);
    kind[2] = (j > 0) ? FACE_INTERIOR : FACE_NONE;          /* pole / wall (R5) */
    kind[3] = (j < g->nt - 1) ? FACE_INTERIOR : FACE_NONE;
    kind[4] = FACE_INTERIOR;                                /* periodic phi (R7) */
    kind[5] = FACE_INTERIOR;
}

static void face_geoms(const mas_ref_grid* g, const tables* T, int i, int j, int k,
                       const int kind[6], double gf[6]) {
    int np = g->np;
    gf[0] = kind[0] ? gR(g, T, i, j, k) : 0.0;
    gf[1] = kind[1] ? gR(g, T, i + 1, j, k) : 0.0;
    gf[2] = kind[2] ? gT(T, i, j, k) : 0.0;
    gf[3] = kind[3] ? gT(T, i, j + 1, k) : 0.0;
    gf[4] = gP(T, i, j, k);
    gf[5] = gP(T, i, j, (k + 1) % np);
}

/* (L u)_P = c_P u_P + (1/V_P) * sum_f G_f (u_P - u_N(f)),
 * G_f = kappa_f g_f, kappa_f = (kappa_P + kappa_N)/2 on interior faces (R6),
 * kappa_f = kappa_P and u_N = 0 on a Dirichlet face (homogeneous).          */
static double cell_L(double V, double cP, double kP, double uP, const int kind[6],
                     const double gf[6], const double kN[6], const double uN[6]) {
    double acc = 0.0;
    int f;
    for (f = 0; f < 6; f++) {
        if (kind[f] == FACE_INTERIOR) {
            double G = 0.5 * (kP + kN[f]) * gf[f];
            acc += G * (uP - uN[f]);
        } else if (kind[f] == FACE_DIRICHLET) {
            double G = kP * gf[f];
            acc += G * uP;
        }
    }
    return cP * uP + acc / V;
}

/* Jacobi diagonal D_P = c_P + (1/V_P) sum_f G_f (R8). */
static double cell_D(double V, double cP, double kP, const int kind[6],
                     const double gf[6], const double kN[6]) {
    double acc = 0.0;
    int f;
    for (f = 0; f < 6; f++) {
        if (kind[f] == FACE_INTERIOR) acc += 0.5 * (kP + kN[f]) * gf[f];
        else if (kind[f] == FACE_DIRICHLET) acc += kP * gf[f];
    }
    return cP + acc / V;
}

#define IDX(g, i, j, k) (((size_t)(i) * (g)->nt + (size_t)(j)) * (g)->np + (size_t)(k))

/* Gather the 6 neighbour values of a monolithic field a at (i,j,k). */
static void gather(const mas_ref_grid* g, const double* a, int i, int j, int k,
                   const int kind[6], double out[6]) {
    int np = g->np;
    out[0] = (kind[0] == FACE_INTERIOR) ? a[IDX(g, i - 1, j, k)] : 0.0;
    out[1] = (kind[1] == FACE_INTERIOR) ? a[IDX(g, i + 1, j, k)] : 0.0;
    out[2] = (kind[2] == FACE_INTERIOR) ? a[IDX(g, i, j - 1, k)] : 0.0;
    out[3] = (kind[3] == FACE_INTERIOR) ? a[IDX(g, i, j + 1, k)] : 0.0;
    out[4] = a[IDX(g, i, j, (k + np - 1) % np)];
    out[5] = a[IDX(g, i, j, (k + 1) % np)];
}

int mas_ref_volumes(const mas_ref_grid* g, double* V) {
    tables T;
    int i;
    if (!g || !V || tables_make(g, &T)) return MAS_REF_ERR_ARG;
#pragma omp parallel for schedule(static)
    for (i = 0; i < g->nr; i++) {
        int j, k;
        for (j = 0; j < g->nt; j++)
            for (k = 0; k < g->np; k++) V[IDX(g, i, j, k)] = cell_V(g, &T, i, j, k);
    }
    tables_free(&T);
    return MAS_REF_OK;
}

int mas_ref_op_apply(const mas_ref_grid* g, int ncomp, const double* kappa,
                     const double* c, const double* x, double* y) {
    tables T;
    size_t N;
    int i;
    if (!g || !kappa || !x || !y || ncomp < 1 || tables_make(g, &T)) return MAS_REF_ERR_ARG;
    N = (size_t)g->nr * g->nt * g->np;
#pragma omp parallel for schedule(static)
    for (i = 0; i < g->nr; i++) {
        int j, k, m, kind[6];
        double gf[6], kN[6], uN[6];
        for (j = 0; j < g->nt; j++) {
            face_kinds(g, i, j, kind);
            for (k = 0; k < g->np; k++) {
                size_t P = IDX(g, i, j, k);
                double V = cell_V(g, &T, i, j, k);
                double cP = c ? c[P] : 0.0;
                face_geoms(g, &T, i, j, k, kind, gf);
                gather(g, kappa, i, j, k, kind, kN);
                for (m = 0; m < ncomp; m++) {
                    const double* u = x + (size_t)m * N;
                    gather(g, u, i, j, k, kind, uN);
                    y[(size_t)m * N + P] = cell_L(V, cP, kappa[P], u[P], kind, gf, kN, uN);
                }
            }
        }
    }
    tables_free(&T);
    return MAS_REF_OK;
}

int mas_ref_op_diag(const mas_ref_grid* g, const double* kappa, const double* c,
                    double* D) {
    tables T;
    int i;
    if (!g || !kappa || !D || tables_make(g, &T)) return MAS_REF_ERR_ARG;
#pragma omp parallel for schedule(static)
    for (i = 0; i < g->nr; i++) {
        int j, k, kind[6];
        double gf[6], kN[6];
        for (j = 0; j < g->nt; j++) {
            face_kinds(g, i, j, kind);
            for (k = 0; k < g->np; k++) {
                size_t P = IDX(g, i, j, k);
                face_geoms(g, &T, i, j, k, kind, gf);
                gather(g, kappa, i, j, k, kind, kN);
                D[P] = cell_D(cell_V(g, &T, i, j, k), c ? c[P] : 0.0, kappa[P], kind, gf, kN);
            }
        }
    }
    tables_free(&T);
    return MAS_REF_OK;
}

int mas_ref_dirichlet_rhs(const mas_ref_grid* g, int ncomp, const double* kappa,
                          const double* ub_inner, const double* ub_outer, double* f) {
    tables T;
    size_t N, plane;
    int j, k, m;
    if (!g || !kappa || !f || ncomp < 1 || tables_make(g, &T)) return MAS_REF_ERR_ARG;
    N = (size_t)g->nr * g->nt * g->np;
    plane = (size_t)g->nt * g->np;
    for (m = 0; m < ncomp; m++)
        for (j = 0; j < g->nt; j++)
            for (k = 0; k < g->np; k++) {
                if (ub_inner && g->bc_inner == MAS_REF_DIRICHLET) {
                    size_t P = IDX(g, 0, j, k);
                    double G = kappa[P] * gR(g, &T, 0, j, k);
                    f[(size_t)m * N + P] += G * ub_inner[(size_t)m * plane + (size_t)j * g->np + k]
                                            / cell_V(g, &T, 0, j, k);
                }
                if (ub_outer && g->bc_outer == MAS_REF_DIRICHLET) {
                    int i = g->nr - 1;
                    size_t P = IDX(g, i, j, k);
                    double G = kappa[P] * gR(g, &T, g->nr, j, k);
                    f[(size_t)m * N + P] += G * ub_outer[(size_t)m * plane + (size_t)j * g->np + k]
                                            / cell_V(g, &T, i, j, k);
                }
            }
    tables_free(&T);
    return MAS_REF_OK;
}

/* V-weighted dot over planes [i0, i0+nl) of arrays holding exactly those
 * planes; per-plane partials in (j,k) order, then planes in order, then
 * components (R9). */
static double dot_planes(const mas_ref_grid* g, const tables* T, int i0, int nl,
                         int ncomp, const double* a, const double* b) {
    size_t plane = (size_t)g->nt * g->np, Nl = plane * nl;
    double* part = malloc(sizeof(double) * (size_t)nl * ncomp);
    double s = 0.0;
    int il, m;
    if (!part) return NAN;
    for (m = 0; m < ncomp; m++) {
#pragma omp parallel for schedule(static)
        for (il = 0; il < nl; il++) {
            int j, k, i = i0 + il;
            double ps = 0.0;
            for (j = 0; j < g->nt; j++)
                for (k = 0; k < g->np; k++) {
                    size_t P = (size_t)m * Nl + (size_t)il * plane + (size_t)j * g->np + k;
                    ps += cell_V(g, T, i, j, k) * a[P] * b[P];
                }
            part[(size_t)m * nl + il] = ps;
        }
    }
    for (m = 0; m < ncomp; m++)
        for (il = 0; il < nl; il++) s += part[(size_t)m * nl + il];
    free(part);
    return s;
}

int mas_ref_dot(const mas_ref_grid* g, int ncomp, const double* a, const double* b,
                double* out) {
    tables T;
    if (!g || !a || !b || !out || ncomp < 1 || tables_make(g, &T)) return MAS_REF_ERR_ARG;
    *out = dot_planes(g, &T, 0, g->nr, ncomp, a, b);
    tables_free(&T);
    return MAS_REF_OK;
}

/* ---------------------------------------------------------------------------
 * Jacobi-PCG (SURVEY §8(c) "PCG, exact order"; R10 stopping, R11 counting).
 * ------------------------------------------------------------------------- */
static int aniso_add(const mas_ref_grid* g, int ncomp, const double* kpar,
                     const double* bhat, const double* x, double* y);
static int aniso_diag_add(const mas_ref_grid* g, const double* kpar, const double* bhat,
                          double* D);
static void curv_add(const mas_ref_grid* g, const double* kappa, const double* x, double* y);

/* The PCG loop for L = L_iso (+ L_par when kpar != NULL, NEXT-4; + the
 * vector-Laplacian curvature terms when curv, NEXT-2, R31: the Jacobi
 * diagonal stays the 7-point one). */
static int pcg_core(const mas_ref_grid* g, int ncomp, const double* kappa,
                    const double* c, const double* kpar, const double* bhat, int curv,
                    const double* f, double* x, double tol,
                    int maxit, int* iters, double* relres, double* res_hist) {
    tables T;
    size_t N, n, e;
    double *D, *r, *z, *p, *q;
    double bn, rn, rho, sigma, alpha, rho_new, beta;
    int k, status = MAS_REF_NOT_CONVERGED, m;
    if (!g || !kappa || !f || !x || !iters || !relres || ncomp < 1 || maxit < 0 ||
        !(tol >= 0.0) || tables_make(g, &T))
        return MAS_REF_ERR_ARG;
    N = (size_t)g->nr * g->nt * g->np;
    n = N * ncomp;
    D = malloc(sizeof(double) * N);
    r = malloc(sizeof(double) * n);
    z = malloc(sizeof(double) * n);
    p = malloc(sizeof(double) * n);
    q = malloc(sizeof(double) * n);
    if (!D || !r || !z || !p || !q) { status = MAS_REF_ERR_ARG; goto done; }
    mas_ref_op_diag(g, kappa, c, D);
    if (kpar) aniso_diag_add(g, kpar, bhat, D);                  /* D += D_par  */

    bn = sqrt(dot_planes(g, &T, 0, g->nr, ncomp, f, f));
    if (bn == 0.0) {
        for (e = 0; e < n; e++) x[e] = 0.0;
        *iters = 0; *relres = 0.0;
        if (res_hist) res_hist[0] = 0.0;
        status = MAS_REF_OK; goto done;
    }
    mas_ref_op_apply(g, ncomp, kappa, c, x, r);                  /* r = L x     */
    if (kpar) aniso_add(g, ncomp, kpar, bhat, x, r);
    if (curv) curv_add(g, kappa, x, r);
#pragma omp parallel for schedule(static)
    for (e = 0; e < n; e++) r[e] = f[e] - r[e];                  /* r = f - L x */
    rn = sqrt(dot_planes(g, &T, 0, g->nr, ncomp, r, r));
    if (res_hist) res_hist[0] = rn;
    if (rn <= tol * bn) { *iters = 0; *relres = rn / bn; status = MAS_REF_OK; goto done; }
    for (m = 0; m < ncomp; m++)
#pragma omp parallel for schedule(static)
        for (e = 0; e < N; e++) z[m * N + e] = r[m * N + e] / D[e];   /* z = D^-1 r  */
    memcpy(p, z, sizeof(double) * n);                            /* p = z       */
    rho = dot_planes(g, &T, 0, g->nr, ncomp, r, z);

    for (k = 1; k <= maxit; k++) {
        mas_ref_op_apply(g, ncomp, kappa, c, p, q);              /* q = L p     */
        if (kpar) aniso_add(g, ncomp, kpar, bhat, p, q);
        if (curv) curv_add(g, kappa, p, q);
        sigma = dot_planes(g, &T, 0, g->nr, ncomp, p, q);
        if (!(sigma > 0.0) || !isfinite(sigma)) {
            *iters = k; *relres = rn / bn; status = MAS_REF_ERR_BREAKDOWN; goto done;
        }
        alpha = rho / sigma;
#pragma omp parallel for schedule(static)
        for (e = 0; e < n; e++) { x[e] += alpha * p[e]; r[e] -= alpha * q[e]; }
        rn = sqrt(dot_planes(g, &T, 0, g->nr, ncomp, r, r));
        if (res_hist) res_hist[k] = rn;
        if (rn <= tol * bn) { *iters = k; *relres = rn / bn; status = MAS_REF_OK; goto done; }
        for (m = 0; m < ncomp; m++)
#pragma omp parallel for schedule(static)
            for (e = 0; e < N; e++) z[m * N + e] = r[m * N + e] / D[e];
        rho_new = dot_planes(g, &T, 0, g->nr, ncomp, r, z);
        beta = rho_new / rho;
        rho = rho_new;
#pragma omp parallel for schedule(static)
        for (e = 0; e < n; e++) p[e] = z[e] + beta * p[e];
    }
    *iters = maxit; *relres = rn / bn; status = MAS_REF_NOT_CONVERGED;
done:
    free(D); free(r); free(z); free(p); free(q);
    tables_free(&T);
    return status;
}

int mas_ref_pcg_solve(const mas_ref_grid* g, int ncomp, const double* kappa,
                      const double* c, const double* f, double* x, double tol,
                      int maxit, int* iters, double* relres, double* res_hist) {
    return pcg_core(g, ncomp, kappa, c, NULL, NULL, 0, f, x, tol, maxit, iters, relres, res_hist);
}

/* ---------------------------------------------------------------------------
 * r-slab decomposition; "virtual ranks" in one process.
 * ------------------------------------------------------------------------- */
void mas_ref_partition(int nr, int nranks, int rank, int* i0, int* nl) {
    int base = nr / nranks, rem = nr % nranks;
    *nl = base + (rank < rem ? 1 : 0);
    *i0 = rank * base + (rank < rem ? rank : rem);
}

int mas_ref_op_apply_slab(const mas_ref_grid* g, int i0, int nl, int ncomp,
                          const double* kappa_ext, const double* c,
                          const double* x_ext, double* y) {
    tables T;
    size_t plane, Ne, Nl;
    int il;
    if (!g || !kappa_ext || !x_ext || !y || ncomp < 1 || nl < 1 || i0 < 0 ||
        i0 + nl > g->nr || tables_make(g, &T))
        return MAS_REF_ERR_ARG;
    plane = (size_t)g->nt * g->np;
    Ne = plane * (nl + 2);
    Nl = plane * nl;
#pragma omp parallel for schedule(static)
    for (il = 0; il < nl; il++) {
        int i = i0 + il, j, k, m, kind[6], np = g->np;
        double gf[6], kN[6], uN[6];
        for (j = 0; j < g->nt; j++) {
            face_kinds(g, i, j, kind);
            for (k = 0; k < np; k++) {
                /* extended index: local plane il sits at ext plane il+1 */
                size_t Pe = (size_t)(il + 1) * plane + (size_t)j * np + k;
                size_t Pl = (size_t)il * plane + (size_t)j * np + k;
                size_t km = (size_t)j * np + (k + np - 1) % np, kp = (size_t)j * np + (k + 1) % np;
                double V = cell_V(g, &T, i, j, k);
                face_geoms(g, &T, i, j, k, kind, gf);
                kN[0] = kappa_ext[Pe - plane];
                kN[1] = kappa_ext[Pe + plane];
                kN[2] = (j > 0) ? kappa_ext[Pe - np] : 0.0;
                kN[3] = (j < g->nt - 1) ? kappa_ext[Pe + np] : 0.0;
                kN[4] = kappa_ext[(size_t)(il + 1) * plane + km];
                kN[5] = kappa_ext[(size_t)(il + 1) * plane + kp];
                for (m = 0; m < ncomp; m++) {
                    const double* u = x_ext + (size_t)m * Ne;
                    uN[0] = u[Pe - plane];
                    uN[1] = u[Pe + plane];
                    uN[2] = (j > 0) ? u[Pe - np] : 0.0;
                    uN[3] = (j < g->nt - 1) ? u[Pe + np] : 0.0;
                    uN[4] = u[(size_t)(il + 1) * plane + km];
                    uN[5] = u[(size_t)(il + 1) * plane + kp];
                    y[(size_t)m * Nl + Pl] =
                        cell_L(V, c ? c[Pl] : 0.0, kappa_ext[Pe], u[Pe], kind, gf, kN, uN);
                }
            }
        }
    }
    tables_free(&T);
    return MAS_REF_OK;
}

/* (r, theta) block [i0,i0+nl) x [j0,j0+ntl) of the global grid (SURVEY §8(f)
 * NEXT-3, the north_star's "slabs in r (and in theta where needed)"): the same
 * cell_L as mas_ref_op_apply, with the neighbour values read from the
 * block's extended arrays (one ghost plane / row on each side).  Face kinds,
 * metrics and volumes use the GLOBAL indices (i, j), so a face on a block
 * edge is an interior face and only the global r-boundaries, poles and theta
 * walls are boundary faces (readings R3, R5). */
int mas_ref_op_apply_block(const mas_ref_grid* g, int i0, int nl, int j0, int ntl, int ncomp,
                           const double* kappa_ext, const double* c,
                           const double* x_ext, double* y) {
    tables T;
    size_t te, pe, Ne, pl, Nl;
    int il;
    if (!g || !kappa_ext || !x_ext || !y || ncomp < 1 || nl < 1 || ntl < 1 || i0 < 0 || j0 < 0 ||
        i0 + nl > g->nr || j0 + ntl > g->nt || tables_make(g, &T))
        return MAS_REF_ERR_ARG;
    te = (size_t)g->np;                 /* ext row stride   */
    pe = (size_t)(ntl + 2) * g->np;     /* ext plane stride */
    Ne = pe * (nl + 2);
    pl = (size_t)ntl * g->np;
    Nl = pl * nl;
#pragma omp parallel for schedule(static)
    for (il = 0; il < nl; il++) {
        int i = i0 + il, jl, k, m, kind[6], np = g->np;
        double gf[6], kN[6], uN[6];
        for (jl = 0; jl < ntl; jl++) {
            int j = j0 + jl;
            face_kinds(g, i, j, kind);
            for (k = 0; k < np; k++) {
                size_t Pe = (size_t)(il + 1) * pe + (size_t)(jl + 1) * te + k;
                size_t Pl = (size_t)il * pl + (size_t)jl * np + k;
                size_t row = (size_t)(il + 1) * pe + (size_t)(jl + 1) * te;
                size_t km = row + (k + np - 1) % np, kp = row + (k + 1) % np;
                double V = cell_V(g, &T, i, j, k);
                face_geoms(g, &T, i, j, k, kind, gf);
                kN[0] = kappa_ext[Pe - pe];
                kN[1] = kappa_ext[Pe + pe];
                kN[2] = (kind[2] == FACE_INTERIOR) ? kappa_ext[Pe - te] : 0.0;
                kN[3] = (kind[3] == FACE_INTERIOR) ? kappa_ext[Pe + te] : 0.0;
                kN[4] = kappa_ext[km];
                kN[5] = kappa_ext[kp];
                for (m = 0; m < ncomp; m++) {
                    const double* u = x_ext + (size_t)m * Ne;
                    uN[0] = u[Pe - pe];
                    uN[1] = u[Pe + pe];
                    uN[2] = (kind[2] == FACE_INTERIOR) ? u[Pe - te] : 0.0;
                    uN[3] = (kind[3] == FACE_INTERIOR) ? u[Pe + te] : 0.0;
                    uN[4] = u[km];
                    uN[5] = u[kp];
                    y[(size_t)m * Nl + Pl] =
                        cell_L(V, c ? c[Pl] : 0.0, kappa_ext[Pe], u[Pe], kind, gf, kN, uN);
                }
            }
        }
    }
    tables_free(&T);
    return MAS_REF_OK;
}

/* Per-block partial of <a,b>_V (a, b: [ncomp][nl][ntl][np]), summed per
 * r-plane in (j,k) order, then planes, then components. */
int mas_ref_dot_block(const mas_ref_grid* g, int i0, int nl, int j0, int ntl, int ncomp,
                      const double* a, const double* b, double* out) {
    tables T;
    size_t pl, Nl;
    int il, jl, k, m;
    double s = 0.0;
    if (!g || !a || !b || !out || nl < 1 || ntl < 1 || tables_make(g, &T)) return MAS_REF_ERR_ARG;
    pl = (size_t)ntl * g->np;
    Nl = pl * nl;
    for (m = 0; m < ncomp; m++)
        for (il = 0; il < nl; il++) {
            double ps = 0.0;
            for (jl = 0; jl < ntl; jl++)
                for (k = 0; k < g->np; k++) {
                    size_t P = (size_t)m * Nl + (size_t)il * pl + (size_t)jl * g->np + k;
                    ps += cell_V(g, &T, i0 + il, j0 + jl, k) * a[P] * b[P];
                }
            s += ps;
        }
    tables_free(&T);
    *out = s;
    return MAS_REF_OK;
}

int mas_ref_dot_slab(const mas_ref_grid* g, int i0, int nl, int ncomp,
                     const double* a, const double* b, double* out) {
    tables T;
    if (!g || !a || !b || !out || nl < 1 || tables_make(g, &T)) return MAS_REF_ERR_ARG;
    *out = dot_planes(g, &T, i0, nl, ncomp, a, b);
    tables_free(&T);
    return MAS_REF_OK;
}

typedef struct {
    int i0, nl;
    double *k_ext, *c, *D, *f, *x_ext, *r, *z, *p_ext, *q;
} vslab;

/* Seam exchange: copy the edge planes of every slab's extended field into the
 * ghost planes of its r-neighbours (what ncclSend/ncclRecv do per rank). */
static void vseam(const mas_ref_grid* g, vslab* S, int P, int ncomp, int which) {
    size_t plane = (size_t)g->nt * g->np, bytes = sizeof(double) * plane;
    int s, m;
    for (s = 0; s < P; s++)
        for (m = 0; m < ncomp; m++) {
            size_t Ne = plane * (S[s].nl + 2);
            double* a = (which == 0 ? S[s].x_ext : which == 1 ? S[s].p_ext : S[s].k_ext) + m * Ne;
            if (s > 0) {
                vslab* L = &S[s - 1];
                size_t NeL = plane * (L->nl + 2);
                double* b = (which == 0 ? L->x_ext : which == 1 ? L->p_ext : L->k_ext) + m * NeL;
                memcpy(a, b + (size_t)L->nl * plane, bytes);           /* ghost lo <- L's last  */
                memcpy(b + (size_t)(L->nl + 1) * plane, a + plane, bytes); /* L's ghost hi <- my first */
            }
        }
}

int mas_ref_pcg_solve_vranks(const mas_ref_grid* g, int P, int ncomp,
                             const double* kappa, const double* c, const double* f,
                             double* x, double tol, int maxit, int* iters,
                             double* relres, double* res_hist) {
    size_t plane, N;
    vslab* S;
    int s, m, k, status = MAS_REF_NOT_CONVERGED;
    double bn, rn, rho, sigma, alpha, rho_new, beta, part;
    if (!g || P < 1 || P > g->nr || !kappa || !f || !x || !iters || !relres || ncomp < 1)
        return MAS_REF_ERR_ARG;
    plane = (size_t)g->nt * g->np;
    N = plane * g->nr;
    S = calloc(P, sizeof(vslab));
    for (s = 0; s < P; s++) {
        size_t Nl, Ne;
        mas_ref_partition(g->nr, P, s, &S[s].i0, &S[s].nl);
        Nl = plane * S[s].nl; Ne = plane * (S[s].nl + 2);
        S[s].k_ext = calloc(Ne, sizeof(double));
        S[s].c = calloc(Nl, sizeof(double));
        S[s].D = calloc(Nl, sizeof(double));
        S[s].f = calloc(Nl * ncomp, sizeof(double));
        S[s].x_ext = calloc(Ne * ncomp, sizeof(double));
        S[s].r = calloc(Nl * ncomp, sizeof(double));
        S[s].z = calloc(Nl * ncomp, sizeof(double));
        S[s].p_ext = calloc(Ne * ncomp, sizeof(double));
        S[s].q = calloc(Nl * ncomp, sizeof(double));
        memcpy(S[s].k_ext + plane, kappa + S[s].i0 * plane, sizeof(double) * Nl);
        if (c) memcpy(S[s].c, c + S[s].i0 * plane, sizeof(double) * Nl);
        for (m = 0; m < ncomp; m++) {
            memcpy(S[s].f + m * Nl, f + m * N + S[s].i0 * plane, sizeof(double) * Nl);
            memcpy(S[s].x_ext + m * Ne + plane, x + m * N + S[s].i0 * plane, sizeof(double) * Nl);
        }
    }
    vseam(g, S, P, 1, 2);                                   /* static kappa seams */
    /* Jacobi diagonal: setup-time quantity, taken from the monolithic routine
     * restricted to each slab's planes. */
    {
        double* Dg = malloc(sizeof(double) * N);
        mas_ref_op_diag(g, kappa, c, Dg);
        for (s = 0; s < P; s++)
            memcpy(S[s].D, Dg + S[s].i0 * plane, sizeof(double) * plane * S[s].nl);
        free(Dg);
    }
    bn = 0.0;
    for (s = 0; s < P; s++) { mas_ref_dot_slab(g, S[s].i0, S[s].nl, ncomp, S[s].f, S[s].f, &part); bn += part; }
    bn = sqrt(bn);
    if (bn == 0.0) {
        memset(x, 0, sizeof(double) * N * ncomp);
        *iters = 0; *relres = 0.0; if (res_hist) res_hist[0] = 0.0;
        status = MAS_REF_OK; goto done;
    }
    vseam(g, S, P, ncomp, 0);
    rn = 0.0;
    for (s = 0; s < P; s++) {
        size_t Nl = plane * S[s].nl, e;
        mas_ref_op_apply_slab(g, S[s].i0, S[s].nl, ncomp, S[s].k_ext, c ? S[s].c : NULL, S[s].x_ext, S[s].r);
        for (e = 0; e < Nl * ncomp; e++) S[s].r[e] = S[s].f[e] - S[s].r[e];
        mas_ref_dot_slab(g, S[s].i0, S[s].nl, ncomp, S[s].r, S[s].r, &part); rn += part;
    }
    rn = sqrt(rn);
    if (res_hist) res_hist[0] = rn;
    if (rn <= tol * bn) { *iters = 0; *relres = rn / bn; status = MAS_REF_OK; goto copyout; }
    rho = 0.0;
    for (s = 0; s < P; s++) {
        size_t Nl = plane * S[s].nl, Ne = plane * (S[s].nl + 2), e;
        for (m = 0; m < ncomp; m++)
            for (e = 0; e < Nl; e++) {
                S[s].z[m * Nl + e] = S[s].r[m * Nl + e] / S[s].D[e];
                S[s].p_ext[m * Ne + plane + e] = S[s].z[m * Nl + e];
            }
        mas_ref_dot_slab(g, S[s].i0, S[s].nl, ncomp, S[s].r, S[s].z, &part); rho += part;
    }
    for (k = 1; k <= maxit; k++) {
        vseam(g, S, P, ncomp, 1);                           /* p seams        */
        sigma = 0.0;
        for (s = 0; s < P; s++) {
            size_t Nl = plane * S[s].nl, Ne = plane * (S[s].nl + 2), e;
            double* pl = malloc(sizeof(double) * Nl * ncomp);
            mas_ref_op_apply_slab(g, S[s].i0, S[s].nl, ncomp, S[s].k_ext, c ? S[s].c : NULL, S[s].p_ext, S[s].q);
            for (m = 0; m < ncomp; m++)
                for (e = 0; e < Nl; e++) pl[m * Nl + e] = S[s].p_ext[m * Ne + plane + e];
            mas_ref_dot_slab(g, S[s].i0, S[s].nl, ncomp, pl, S[s].q, &part); sigma += part;
            free(pl);
        }
        if (!(sigma > 0.0) || !isfinite(sigma)) {
            *iters = k; *relres = rn / bn; status = MAS_REF_ERR_BREAKDOWN; goto copyout;
        }
        alpha = rho / sigma;
        rn = 0.0;
        for (s = 0; s < P; s++) {
            size_t Nl = plane * S[s].nl, Ne = plane * (S[s].nl + 2), e;
            for (m = 0; m < ncomp; m++)
                for (e = 0; e < Nl; e++) {
                    S[s].x_ext[m * Ne + plane + e] += alpha * S[s].p_ext[m * Ne + plane + e];
                    S[s].r[m * Nl + e] -= alpha * S[s].q[m * Nl + e];
                }
            mas_ref_dot_slab(g, S[s].i0, S[s].nl, ncomp, S[s].r, S[s].r, &part); rn += part;
        }
        rn = sqrt(rn);
        if (res_hist) res_hist[k] = rn;
        if (rn <= tol * bn) { *iters = k; *relres = rn / bn; status = MAS_REF_OK; goto copyout; }
        rho_new = 0.0;
        for (s = 0; s < P; s++) {
            size_t Nl = plane * S[s].nl, e;
            for (m = 0; m < ncomp; m++)
                for (e = 0; e < Nl; e++) S[s].z[m * Nl + e] = S[s].r[m * Nl + e] / S[s].D[e];
            mas_ref_dot_slab(g, S[s].i0, S[s].nl, ncomp, S[s].r, S[s].z, &part); rho_new += part;
        }
        beta = rho_new / rho;
        rho = rho_new;
        for (s = 0; s < P; s++) {
            size_t Nl = plane * S[s].nl, Ne = plane * (S[s].nl + 2), e;
            for (m = 0; m < ncomp; m++)
                for (e = 0; e < Nl; e++)
                    S[s].p_ext[m * Ne + plane + e] = S[s].z[m * Nl + e] + beta * S[s].p_ext[m * Ne + plane + e];
        }
    }
    *iters = maxit; *relres = rn / bn; status = MAS_REF_NOT_CONVERGED;
copyout:
    for (s = 0; s < P; s++) {
        size_t Nl = plane * S[s].nl, Ne = plane * (S[s].nl + 2);
        for (m = 0; m < ncomp; m++)
            memcpy(x + m * N + S[s].i0 * plane, S[s].x_ext + m * Ne + plane, sizeof(double) * Nl);
    }
done:
    for (s = 0; s < P; s++) {
        free(S[s].k_ext); free(S[s].c); free(S[s].D); free(S[s].f); free(S[s].x_ext);
        free(S[s].r); free(S[s].z); free(S[s].p_ext); free(S[s].q);
    }
    free(S);
    return status;
}

/* Per-cell evaluation of (L x) at a list of flat cell indices (comp-major
 * flat index m*N + P): used to check GPU results sampled at full size. */
int mas_ref_op_apply_cells(const mas_ref_grid* g, int ncomp, const double* kappa,
                           const double* c, const double* x, long long ncells,
                           const long long* idx, double* out) {
    tables T;
    size_t N;
    long long s;
    if (!g || !kappa || !x || !idx || !out || ncomp < 1 || tables_make(g, &T)) return MAS_REF_ERR_ARG;
    N = (size_t)g->nr * g->nt * g->np;
#pragma omp parallel for schedule(static)
    for (s = 0; s < ncells; s++) {
        size_t flat = (size_t)idx[s], P = flat % N;
        int m = (int)(flat / N);
        int i = (int)(P / ((size_t)g->nt * g->np));
        int j = (int)((P / g->np) % g->nt);
        int k = (int)(P % g->np), kind[6];
        double gf[6], kN[6], uN[6];
        const double* u = x + (size_t)m * N;
        face_kinds(g, i, j, kind);
        face_geoms(g, &T, i, j, k, kind, gf);
        gather(g, kappa, i, j, k, kind, kN);
        gather(g, u, i, j, k, kind, uN);
        out[s] = cell_L(cell_V(g, &T, i, j, k), c ? c[P] : 0.0, kappa[P], u[P], kind, gf, kN, uN);
    }
    tables_free(&T);
    return MAS_REF_OK;
}

/* ---------------------------------------------------------------------------
 * Field-aligned (anisotropic) thermal conduction — SURVEY §8(f) NEXT-4.
 * The paper names MAS's thermal conduction only through its test problem
 * ("thermodynamic MHD") and the implicit parabolic Krylov solvers
 * of ref. [25]; it prints no formula.  Readings (DESIGN.md
 * §3.4, R21-R26):
 *
 *   R21  L = L_iso + L_par with L_par u = -div(kpar b (b . grad u)), written in
 *        the symmetric corner ("dual-cell") form
 *          V_P (L_par u)_P = sum_{corners c of P} W_c kpar_c (b_c . g_c(u))
 *                                                      (b_c . d g_c / d u_P)
 *        (so V L_par = G^T W K G is symmetric positive semi-definite).
 *   R22  g_c = (d_r u, (1/r) d_theta u, (1/(r sin theta)) d_phi u) at the
 *        corner c = (rF_I, tF_J, pF_K) from its 8 cells (I-1+a, J-1+b,
 *        K-1+e mod np), a,b,e in {0,1}: each component is the mean of the 4
 *        cell-centre differences across the corner in that direction,
 *          g_r   = sum_{b,e} (u[I][..] - u[I-1][..]) / (4 hr_I)
 *          g_t   = sum_{a,e} (u[..][J][..] - u[..][J-1][..]) / (4 rF_I ht_J)
 *          g_p   = sum_{a,b} (u[..][..][K] - u[..][..][K-1]) / (4 rF_I sF_J hp_K)
 *   R23  dual volume W_c = rF_I^2 sin(tF_J) hr_I ht_J hp_K (midpoint FD, R4).
 *   R24  corners on the domain boundary (r faces 0 and nr, theta faces 0 and
 *        nt: poles and walls) carry no weight: no field-aligned flux leaves
 *        the domain; the boundary conditions stay with L_iso.
 *   R25  kpar and b are given AT CORNERS, stored at the cell whose lower
 *        corner it is: kpar[i][j][k] belongs to (rF_i, tF_j, pF_k); entries
 *        with i = 0 or j = 0 are ignored.  b = (b_r, b_theta, b_phi) is used as
 *        given (not renormalised), layout bhat[3][nr][nt][np].
 *   R26  the Jacobi diagonal adds (1/V_P) sum_c W_c kpar_c (b_c . dg_c/du_P)^2.
 * ------------------------------------------------------------------------- */
static int corner_live(const mas_ref_grid* g, int I, int J) {          /* R24 */
    return I >= 1 && I <= g->nr - 1 && J >= 1 && J <= g->nt - 1;
}

static double corner_W(const mas_ref_grid* g, const tables* T, int I, int J, int K) { /* R23 */
    return g->rF[I] * g->rF[I] * T->sF[J] * T->hr[I] * T->ht[J] * T->hp[K];
}

/* R22: the corner gradient of u (one component).  u holds global r-planes
 * uo .. (array plane 0 = global plane uo): uo = 0 for a monolithic field,
 * i0 - 1 for a slab with its ghost planes. */
#define UIDX(g, uo, i, j, k) IDX(g, (i) - (uo), j, k)
static void corner_grad(const mas_ref_grid* g, const tables* T, const double* u, int uo, int I,
                        int J, int K, double gr[3]) {
    int np = g->np, Km = (K + np - 1) % np, a, b, e;
    int ii[2] = {I - 1, I}, jj[2] = {J - 1, J}, kk[2] = {Km, K};
    double sr = 0.0, st = 0.0, sp = 0.0;
    for (b = 0; b < 2; b++)
        for (e = 0; e < 2; e++)
            sr += u[UIDX(g, uo, I, jj[b], kk[e])] - u[UIDX(g, uo, I - 1, jj[b], kk[e])];
    for (a = 0; a < 2; a++)
        for (e = 0; e < 2; e++)
            st += u[UIDX(g, uo, ii[a], J, kk[e])] - u[UIDX(g, uo, ii[a], J - 1, kk[e])];
    for (a = 0; a < 2; a++)
        for (b = 0; b < 2; b++)
            sp += u[UIDX(g, uo, ii[a], jj[b], K)] - u[UIDX(g, uo, ii[a], jj[b], Km)];
    gr[0] = sr / (4.0 * T->hr[I]);
    gr[1] = st / (4.0 * g->rF[I] * T->ht[J]);
    gr[2] = sp / (4.0 * g->rF[I] * T->sF[J] * T->hp[K]);
}

/* d g_c / d u_Q for the cell Q = (I-1+a, J-1+b, K-1+e) of corner c. */
static void corner_dgrad(const mas_ref_grid* g, const tables* T, int I, int J, int K, int a,
                         int b, int e, double d[3]) {
    d[0] = (a ? 1.0 : -1.0) / (4.0 * T->hr[I]);
    d[1] = (b ? 1.0 : -1.0) / (4.0 * g->rF[I] * T->ht[J]);
    d[2] = (e ? 1.0 : -1.0) / (4.0 * g->rF[I] * T->sF[J] * T->hp[K]);
}

/* R21 / R26 for cell (i,j,k): sum over its 8 corners of W kpar (b.g)(b.dg)
 * (want_diag: W kpar (b.dg)^2), divided by V_P.  u may be NULL for the diagonal.
 * The corner fields hold global corner planes co .. (bhat components Nc apart),
 * u holds global planes uo .. (UIDX); monolithic: co = uo = 0, Nc = N. */
static double aniso_cell_at(const mas_ref_grid* g, const tables* T, const double* kpar,
                            const double* bhat, size_t Nc, int co, const double* u, int uo,
                            int i, int j, int k, int want_diag) {
    size_t N = Nc;
    double acc = 0.0;
    int a, b, e;
    for (a = 0; a < 2; a++)           /* a = 1: the corner plane I = i (cell above it) */
        for (b = 0; b < 2; b++)
            for (e = 0; e < 2; e++) {
                int I = a ? i : i + 1, J = b ? j : j + 1, K = e ? k : (k + 1) % g->np;
                size_t C;
                double W, kc, bv[3], d[3], bd, gr[3];
                if (!corner_live(g, I, J)) continue;
                C = IDX(g, I - co, J, K);
                W = corner_W(g, T, I, J, K);
                kc = kpar[C];
                bv[0] = bhat[C]; bv[1] = bhat[N + C]; bv[2] = bhat[2 * N + C];
                corner_dgrad(g, T, I, J, K, a, b, e, d);
                bd = bv[0] * d[0] + bv[1] * d[1] + bv[2] * d[2];
                if (want_diag) {
                    acc += W * kc * bd * bd;
                } else {
                    corner_grad(g, T, u, uo, I, J, K, gr);
                    acc += W * kc * (bv[0] * gr[0] + bv[1] * gr[1] + bv[2] * gr[2]) * bd;
                }
            }
    return acc / cell_V(g, T, i, j, k);
}

static double aniso_cell(const mas_ref_grid* g, const tables* T, const double* kpar,
                         const double* bhat, const double* u, int i, int j, int k, int want_diag) {
    return aniso_cell_at(g, T, kpar, bhat, (size_t)g->nr * g->nt * g->np, 0, u, 0, i, j, k,
                         want_diag);
}

static int aniso_check(const mas_ref_grid* g, const double* kpar, const double* bhat) {
    return g && kpar && bhat && g->nr >= 1 && g->nt >= 1 && g->np >= 2;
}

int mas_ref_aniso_apply(const mas_ref_grid* g, int ncomp, const double* kpar,
                        const double* bhat, const double* x, double* y) {
    tables T;
    size_t N;
    int i;
    if (!aniso_check(g, kpar, bhat) || !x || !y || ncomp < 1 || tables_make(g, &T))
        return MAS_REF_ERR_ARG;
    N = (size_t)g->nr * g->nt * g->np;
#pragma omp parallel for schedule(static)
    for (i = 0; i < g->nr; i++) {
        int j, k, m;
        for (m = 0; m < ncomp; m++)
            for (j = 0; j < g->nt; j++)
                for (k = 0; k < g->np; k++)
                    y[(size_t)m * N + IDX(g, i, j, k)] =
                        aniso_cell(g, &T, kpar, bhat, x + (size_t)m * N, i, j, k, 0);
    }
    tables_free(&T);
    return MAS_REF_OK;
}

int mas_ref_aniso_diag(const mas_ref_grid* g, const double* kpar, const double* bhat,
                       double* D) {
    tables T;
    int i;
    if (!aniso_check(g, kpar, bhat) || !D || tables_make(g, &T)) return MAS_REF_ERR_ARG;
#pragma omp parallel for schedule(static)
    for (i = 0; i < g->nr; i++) {
        int j, k;
        for (j = 0; j < g->nt; j++)
            for (k = 0; k < g->np; k++)
                D[IDX(g, i, j, k)] = aniso_cell(g, &T, kpar, bhat, NULL, i, j, k, 1);
    }
    tables_free(&T);
    return MAS_REF_OK;
}

/* y += L_par x (the PCG's full operator is L_iso + L_par, summed per cell). */
static int aniso_add(const mas_ref_grid* g, int ncomp, const double* kpar,
                     const double* bhat, const double* x, double* y) {
    size_t n = (size_t)g->nr * g->nt * g->np * ncomp, e;
    double* t = malloc(sizeof(double) * n);
    int rc;
    if (!t) return MAS_REF_ERR_ARG;
    rc = mas_ref_aniso_apply(g, ncomp, kpar, bhat, x, t);
    for (e = 0; e < n; e++) y[e] += t[e];
    free(t);
    return rc;
}

static int aniso_diag_add(const mas_ref_grid* g, const double* kpar, const double* bhat,
                          double* D) {
    size_t n = (size_t)g->nr * g->nt * g->np, e;
    double* t = malloc(sizeof(double) * n);
    int rc;
    if (!t) return MAS_REF_ERR_ARG;
    rc = mas_ref_aniso_diag(g, kpar, bhat, t);
    for (e = 0; e < n; e++) D[e] += t[e];
    free(t);
    return rc;
}

int mas_ref_pcg_solve_aniso(const mas_ref_grid* g, int ncomp, const double* kappa,
                            const double* c, const double* kpar, const double* bhat,
                            const double* f, double* x, double tol, int maxit, int* iters,
                            double* relres, double* res_hist) {
    if (!aniso_check(g, kpar, bhat)) return MAS_REF_ERR_ARG;
    return pcg_core(g, ncomp, kappa, c, kpar, bhat, 0, f, x, tol, maxit, iters, relres, res_hist);
}

/* Slab-local L_par for a rank owning r-planes [i0, i0+nl) (the r-slab
 * protocol of the library): x_ext [ncomp][nl+2][nt][np] with
 * the ghost planes i0-1 / i0+nl at ext planes 0 / nl+1; the corner fields
 * kpar_ext [nl+1][nt][np], bhat_ext [3][nl+1][nt][np] hold corner planes
 * i0 .. i0+nl (the last one is rank+1's first; ignored at the global outer
 * face).  y [ncomp][nl][nt][np]. */
int mas_ref_aniso_apply_slab(const mas_ref_grid* g, int i0, int nl, int ncomp,
                             const double* kpar_ext, const double* bhat_ext,
                             const double* x_ext, double* y) {
    tables T;
    size_t plane, Nc, Ne, Nl;
    int il;
    if (!aniso_check(g, kpar_ext, bhat_ext) || !x_ext || !y || ncomp < 1 || nl < 1 || i0 < 0 ||
        i0 + nl > g->nr || tables_make(g, &T))
        return MAS_REF_ERR_ARG;
    plane = (size_t)g->nt * g->np;
    Nc = plane * (nl + 1);
    Ne = plane * (nl + 2);
    Nl = plane * nl;
#pragma omp parallel for schedule(static)
    for (il = 0; il < nl; il++) {
        int j, k, m, i = i0 + il;
        for (m = 0; m < ncomp; m++)
            for (j = 0; j < g->nt; j++)
                for (k = 0; k < g->np; k++)
                    y[(size_t)m * Nl + IDX(g, il, j, k)] =
                        aniso_cell_at(g, &T, kpar_ext, bhat_ext, Nc, i0, x_ext + (size_t)m * Ne,
                                      i0 - 1, i, j, k, 0);
    }
    tables_free(&T);
    return MAS_REF_OK;
}

/* ---------------------------------------------------------------------------
 * Per-radius array reductions, the paper's Listings 3-5 (P:428-445,
 * P:592-645, §IV): "sum0(i)=sum0(i)+array(i,j)*..." over the angular index,
 * one sum per radius i.  MAS uses them e.g. for the phi-averaged values of
 * node-in-theta variables at the poles.  Reading R27:
 * the elided factor "..." is a caller-supplied angular weight w[j][k], so
 *   sum0[m][i] = sum_{j,k} w[j][k] x[m][i][j][k]     (summed in (j,k) order).
 * ------------------------------------------------------------------------- */
int mas_ref_radial_sums(const mas_ref_grid* g, int ncomp, const double* x, const double* w,
                        double* out) {
    size_t plane, N;
    int m, i;
    if (!g || !x || !w || !out || ncomp < 1 || g->nr < 1 || g->nt < 1 || g->np < 1)
        return MAS_REF_ERR_ARG;
    plane = (size_t)g->nt * g->np;
    N = plane * g->nr;
    for (m = 0; m < ncomp; m++)
        for (i = 0; i < g->nr; i++) {
            const double* xp = x + (size_t)m * N + (size_t)i * plane;
            double s = 0.0;
            size_t e;
            for (e = 0; e < plane; e++) s += w[e] * xp[e];
            out[(size_t)m * g->nr + i] = s;
        }
    return MAS_REF_OK;
}

/* ---------------------------------------------------------------------------
 * Single-reduction PCG: the Chronopoulos-Gear
 * rearrangement of the same Jacobi-PCG, in which the two inner products of
 * an iteration (<r,z> and the curvature <Lz,z>) come from ONE reduction, so a
 * distributed solve needs one allreduce per iteration instead of two (the
 * paper's async / fusion lesson; its solver is
 * "Krylov", without further detail).  Reading R28:
 * Chronopoulos & Gear (1989), preconditioned form, with u = D^-1 r:
 *
 *   r0 = f - L x0;  u0 = D^-1 r0;  w0 = L u0;  g0 = <r0,u0>;  d0 = <w0,u0>
 *   a0 = g0 / d0;  p0 = u0;  s0 = w0
 *   for k = 1, 2, ...:
 *       x_k = x_{k-1} + a_{k-1} p_{k-1};  r_k = r_{k-1} - a_{k-1} s_{k-1}
 *       stop if ||r_k||_V <= tol ||f||_V   (R10; iters = k, R11: k products)
 *       u_k = D^-1 r_k;  w_k = L u_k
 *       g_k = <r_k,u_k>;  d_k = <w_k,u_k>          (one reduction: + ||r_k||^2)
 *       b_k = g_k / g_{k-1};  a_k = g_k / (d_k - b_k g_k / a_{k-1})
 *       p_k = u_k + b_k p_{k-1};  s_k = w_k + b_k s_{k-1}   (s_k = L p_k)
 *
 * In exact arithmetic x_k, r_k equal the standard PCG iterates (pcg_core).
 * The denominator d_k - b_k g_k / a_{k-1} equals <p_k, L p_k>: !(> 0) is a
 * breakdown (iters = k, x = x_k).  The residual ||r_k|| needed for the stop
 * is the recursive one, as in pcg_core.
 * ------------------------------------------------------------------------- */
int mas_ref_pcg_solve_cg1(const mas_ref_grid* g, int ncomp, const double* kappa,
                          const double* c, const double* f, double* x, double tol,
                          int maxit, int* iters, double* relres, double* res_hist) {
    tables T;
    size_t N, n, e;
    double *D, *r, *u, *w, *p, *s;
    double bn, rn, gam, del, alpha, beta, gam_new, den;
    int k, status = MAS_REF_NOT_CONVERGED, m;
    if (!g || !kappa || !f || !x || !iters || !relres || ncomp < 1 || maxit < 0 ||
        !(tol >= 0.0) || tables_make(g, &T))
        return MAS_REF_ERR_ARG;
    N = (size_t)g->nr * g->nt * g->np;
    n = N * ncomp;
    D = malloc(sizeof(double) * N);
    r = malloc(sizeof(double) * n);
    u = malloc(sizeof(double) * n);
    w = malloc(sizeof(double) * n);
    p = malloc(sizeof(double) * n);
    s = malloc(sizeof(double) * n);
    if (!D || !r || !u || !w || !p || !s) { status = MAS_REF_ERR_ARG; goto done; }
    mas_ref_op_diag(g, kappa, c, D);

    bn = sqrt(dot_planes(g, &T, 0, g->nr, ncomp, f, f));
    if (bn == 0.0) {
        for (e = 0; e < n; e++) x[e] = 0.0;
        *iters = 0; *relres = 0.0;
        if (res_hist) res_hist[0] = 0.0;
        status = MAS_REF_OK; goto done;
    }
    mas_ref_op_apply(g, ncomp, kappa, c, x, r);                  /* r = L x       */
#pragma omp parallel for schedule(static)
    for (e = 0; e < n; e++) r[e] = f[e] - r[e];                  /* r0 = f - L x0 */
    rn = sqrt(dot_planes(g, &T, 0, g->nr, ncomp, r, r));
    if (res_hist) res_hist[0] = rn;
    if (rn <= tol * bn) { *iters = 0; *relres = rn / bn; status = MAS_REF_OK; goto done; }
    if (maxit == 0) { *iters = 0; *relres = rn / bn; status = MAS_REF_NOT_CONVERGED; goto done; }
    for (m = 0; m < ncomp; m++)
#pragma omp parallel for schedule(static)
        for (e = 0; e < N; e++) u[m * N + e] = r[m * N + e] / D[e];   /* u0 = D^-1 r0 */
    mas_ref_op_apply(g, ncomp, kappa, c, u, w);                  /* w0 = L u0     */
    gam = dot_planes(g, &T, 0, g->nr, ncomp, r, u);
    del = dot_planes(g, &T, 0, g->nr, ncomp, w, u);
    if (!(del > 0.0) || !isfinite(del)) {
        *iters = 1; *relres = rn / bn; status = MAS_REF_ERR_BREAKDOWN; goto done;
    }
    alpha = gam / del;
    memcpy(p, u, sizeof(double) * n);                            /* p0 = u0       */
    memcpy(s, w, sizeof(double) * n);                            /* s0 = w0       */

    for (k = 1; k <= maxit; k++) {
#pragma omp parallel for schedule(static)
        for (e = 0; e < n; e++) { x[e] += alpha * p[e]; r[e] -= alpha * s[e]; }
        rn = sqrt(dot_planes(g, &T, 0, g->nr, ncomp, r, r));
        if (res_hist) res_hist[k] = rn;
        if (rn <= tol * bn) { *iters = k; *relres = rn / bn; status = MAS_REF_OK; goto done; }
        if (k == maxit) break;
        for (m = 0; m < ncomp; m++)
#pragma omp parallel for schedule(static)
            for (e = 0; e < N; e++) u[m * N + e] = r[m * N + e] / D[e];
        mas_ref_op_apply(g, ncomp, kappa, c, u, w);              /* w = L u       */
        gam_new = dot_planes(g, &T, 0, g->nr, ncomp, r, u);
        del = dot_planes(g, &T, 0, g->nr, ncomp, w, u);
        beta = gam_new / gam;
        gam = gam_new;
        den = del - beta * gam / alpha;                          /* = <p, L p>    */
        if (!(den > 0.0) || !isfinite(den)) {
            *iters = k; *relres = rn / bn; status = MAS_REF_ERR_BREAKDOWN; goto done;
        }
        alpha = gam / den;
#pragma omp parallel for schedule(static)
        for (e = 0; e < n; e++) { p[e] = u[e] + beta * p[e]; s[e] = w[e] + beta * s[e]; }
    }
    *iters = maxit; *relres = rn / bn; status = MAS_REF_NOT_CONVERGED;
done:
    free(D); free(r); free(u); free(w); free(p); free(s);
    tables_free(&T);
    return status;
}

/* ---------------------------------------------------------------------------
 * theta-node placement with pole unknowns (readings
 * R29-R30 in DESIGN.md §3.5).  MAS's grid is staggered: some
 * variables live on the theta "main" mesh tF_j, j = 0..nt, whose end rows sit
 * ON the poles.  A pole is one point per radius, so a pole row holds a single
 * value (stored replicated over phi).  The operator is the finite-volume
 * balance of the same L = c + (1/V) div(kappa grad):
 *   - interior rows 1..nt-1: theta extent [tC_{j-1}, tC_j] around tF_j,
 *       V = rC^2 dr * sin(tF_j) (tC_j - tC_{j-1}) * dp,
 *       theta face at tC_{j-1}: g = dr sin(tC_{j-1}) dp / (tF_j - tF_{j-1}),
 *       phi face: g = dr (tC_j - tC_{j-1}) / (sin(tF_j) hp),
 *       r face: g = rF^2 sin(tF_j) (tC_j - tC_{j-1}) dp / hr   (R4 midpoint form);
 *   - pole rows: the polar cap theta in [0, tC_0] (north; [tC_{nt-1}, pi]
 *     south) of exact measure A = 1 - cos(tC_0) (1 + cos(tC_{nt-1})), split
 *     into the np phi slices k of volume V_k = rC^2 dr A dp_k; the cap balance
 *       V_cap (L u)_pole = sum_k [ V_k c_k u_pole + sum_{r faces} G_{R,k}(u_pole - u_N)
 *                                  + G_{T,k} (u_pole - u_{row 1 or nt-1, k}) ]
 *     with V_cap = sum_k V_k, G_{T,k} the theta face at tC_0 of slice k and
 *     G_{R,k} = kappa_f rF^2 A dp_k / hr: a per-radius sum over phi -- the
 *     paper's sum0 array reduction (Listings 3-5).
 * kappa, c per slot as stored (kappa_f the face mean, R6); x's pole rows must
 * be phi-constant (every slot holds the pole value); y's pole rows are
 * written replicated.  Arrays [comp][nr][nt+1][np].  The inner product
 * weights a pole slot with V_k (so a replicated pole row weighs V_cap).
 * ------------------------------------------------------------------------- */
typedef struct {
    double* m;    /* [nt+1] theta measure of row j: sin(tF_j) dtau_j; A_N, A_S at the poles */
    double* dtau; /* [nt+1] tC_j - tC_{j-1} (interior rows)                                  */
    double* sT;   /* [nt+1] sin(tC_{j-1}): theta face between rows j-1 and j (j = 1..nt)      */
    double* hT;   /* [nt+1] tF_j - tF_{j-1}                                                   */
} tn_tables;

static void tn_free(tn_tables* Q) { free(Q->m); free(Q->dtau); free(Q->sT); free(Q->hT); }

static int tn_make(const mas_ref_grid* g, tn_tables* Q) {
    int nt = g->nt, j;
    memset(Q, 0, sizeof(*Q));
    if (nt < 2) return MAS_REF_ERR_ARG;
    if (g->tF[0] != 0.0 || fabs(g->tF[nt] - 3.14159265358979323846) > 1e-14) return MAS_REF_ERR_ARG;
    Q->m = calloc(nt + 1, sizeof(double));
    Q->dtau = calloc(nt + 1, sizeof(double));
    Q->sT = calloc(nt + 1, sizeof(double));
    Q->hT = calloc(nt + 1, sizeof(double));
    if (!Q->m || !Q->dtau || !Q->sT || !Q->hT) { tn_free(Q); return MAS_REF_ERR_ARG; }
    for (j = 1; j < nt; j++) {
        Q->dtau[j] = g->tC[j] - g->tC[j - 1];
        Q->m[j] = sin(g->tF[j]) * Q->dtau[j];
    }
    Q->m[0] = 1.0 - cos(g->tC[0]);        /* north cap measure */
    Q->m[nt] = 1.0 + cos(g->tC[nt - 1]);  /* south cap measure */
    for (j = 1; j <= nt; j++) {
        Q->sT[j] = sin(g->tC[j - 1]);
        Q->hT[j] = g->tF[j] - g->tF[j - 1];
    }
    return MAS_REF_OK;
}

#define TIDX(g, i, j, k) (((size_t)(i) * ((g)->nt + 1) + (size_t)(j)) * (g)->np + (size_t)(k))

/* one slot (row j, slice k) of radius i: V, the face conductances and the
 * neighbour slots (r-faces: 0 toward i-1, 1 toward i+1; theta: 2 toward j-1,
 * 3 toward j+1; phi: 4, 5 -- none on a pole row) */
static void tn_slot(const mas_ref_grid* g, const tables* T, const tn_tables* Q, int i, int j, int k,
                    double* V, int kind[6], double gf[6], size_t nb[6]) {
    int nt = g->nt, np = g->np, f;
    const int pole = (j == 0 || j == nt);
    for (f = 0; f < 6; f++) { kind[f] = FACE_NONE; gf[f] = 0.0; nb[f] = 0; }
    *V = g->rC[i] * g->rC[i] * T->dr[i] * Q->m[j] * T->dp[k];
    kind[0] = (i > 0) ? FACE_INTERIOR : (g->bc_inner == MAS_REF_DIRICHLET ? FACE_DIRICHLET : FACE_NONE);
    kind[1] = (i < g->nr - 1) ? FACE_INTERIOR : (g->bc_outer == MAS_REF_DIRICHLET ? FACE_DIRICHLET : FACE_NONE);
    if (kind[0]) gf[0] = g->rF[i] * g->rF[i] * Q->m[j] * T->dp[k] / T->hr[i];
    if (kind[1]) gf[1] = g->rF[i + 1] * g->rF[i + 1] * Q->m[j] * T->dp[k] / T->hr[i + 1];
    if (kind[0] == FACE_INTERIOR) nb[0] = TIDX(g, i - 1, j, k);
    if (kind[1] == FACE_INTERIOR) nb[1] = TIDX(g, i + 1, j, k);
    if (j > 0) {  /* theta face at tC_{j-1} */
        kind[2] = FACE_INTERIOR;
        gf[2] = T->dr[i] * Q->sT[j] * T->dp[k] / Q->hT[j];
        nb[2] = TIDX(g, i, j - 1, k);
    }
    if (j < nt) { /* theta face at tC_j */
        kind[3] = FACE_INTERIOR;
        gf[3] = T->dr[i] * Q->sT[j + 1] * T->dp[k] / Q->hT[j + 1];
        nb[3] = TIDX(g, i, j + 1, k);
    }
    if (!pole) {
        kind[4] = kind[5] = FACE_INTERIOR;
        gf[4] = T->dr[i] * Q->dtau[j] / (sin(g->tF[j]) * T->hp[k]);
        gf[5] = T->dr[i] * Q->dtau[j] / (sin(g->tF[j]) * T->hp[(k + 1) % np]);
        nb[4] = TIDX(g, i, j, (k + np - 1) % np);
        nb[5] = TIDX(g, i, j, (k + 1) % np);
    }
}

/* the face sum of one slot: sum_f G_f (u - u_N), G_f = kappa_f g_f (as
 * cell_L's sum, before the division by the volume; the mass term apart) */
static double tn_slot_flux(const int kind[6], const double gf[6], const size_t nb[6],
                           double kP, double uP, const double* kappa, const double* u) {
    double acc = 0.0;
    int f;
    for (f = 0; f < 6; f++) {
        if (kind[f] == FACE_INTERIOR) acc += 0.5 * (kP + kappa[nb[f]]) * gf[f] * (uP - u[nb[f]]);
        else if (kind[f] == FACE_DIRICHLET) acc += kP * gf[f] * uP;
    }
    return acc;
}
static double tn_slot_diag(const int kind[6], const double gf[6], const size_t nb[6],
                           double kP, const double* kappa) {
    double acc = 0.0;
    int f;
    for (f = 0; f < 6; f++) {
        if (kind[f] == FACE_INTERIOR) acc += 0.5 * (kP + kappa[nb[f]]) * gf[f];
        else if (kind[f] == FACE_DIRICHLET) acc += kP * gf[f];
    }
    return acc;
}

int mas_ref_tn_volumes(const mas_ref_grid* g, double* V) {
    tables T;
    tn_tables Q;
    int i, j, k, kind[6];
    double gf[6];
    size_t nb[6];
    if (!g || !V || tables_make(g, &T)) return MAS_REF_ERR_ARG;
    if (tn_make(g, &Q)) { tables_free(&T); return MAS_REF_ERR_ARG; }
    for (i = 0; i < g->nr; i++)
        for (j = 0; j <= g->nt; j++)
            for (k = 0; k < g->np; k++) tn_slot(g, &T, &Q, i, j, k, &V[TIDX(g, i, j, k)], kind, gf, nb);
    tn_free(&Q);
    tables_free(&T);
    return MAS_REF_OK;
}

int mas_ref_tn_apply(const mas_ref_grid* g, int ncomp, const double* kappa, const double* c,
                     const double* x, double* y) {
    tables T;
    tn_tables Q;
    size_t N;
    int i;
    if (!g || !kappa || !x || !y || ncomp < 1 || tables_make(g, &T)) return MAS_REF_ERR_ARG;
    if (tn_make(g, &Q)) { tables_free(&T); return MAS_REF_ERR_ARG; }
    N = (size_t)g->nr * (g->nt + 1) * g->np;
#pragma omp parallel for schedule(static)
    for (i = 0; i < g->nr; i++) {
        int j, k, m, kind[6];
        double gf[6], V;
        size_t nb[6];
        for (m = 0; m < ncomp; m++) {
            const double* u = x + (size_t)m * N;
            double* out = y + (size_t)m * N;
            for (j = 0; j <= g->nt; j++) {
                if (j == 0 || j == g->nt) {
                    /* the polar cap: sum the slices' balances over phi (sum0) */
                    double num = 0.0, vcap = 0.0;
                    for (k = 0; k < g->np; k++) {
                        size_t P = TIDX(g, i, j, k);
                        tn_slot(g, &T, &Q, i, j, k, &V, kind, gf, nb);
                        num += V * (c ? c[P] : 0.0) * u[P] + tn_slot_flux(kind, gf, nb, kappa[P], u[P], kappa, u);
                        vcap += V;
                    }
                    for (k = 0; k < g->np; k++) out[TIDX(g, i, j, k)] = num / vcap;
                } else {
                    for (k = 0; k < g->np; k++) {
                        size_t P = TIDX(g, i, j, k);
                        tn_slot(g, &T, &Q, i, j, k, &V, kind, gf, nb);
                        out[P] = (c ? c[P] : 0.0) * u[P] + tn_slot_flux(kind, gf, nb, kappa[P], u[P], kappa, u) / V;
                    }
                }
            }
        }
    }
    tn_free(&Q);
    tables_free(&T);
    return MAS_REF_OK;
}

int mas_ref_tn_diag(const mas_ref_grid* g, const double* kappa, const double* c, double* D) {
    tables T;
    tn_tables Q;
    int i;
    if (!g || !kappa || !D || tables_make(g, &T)) return MAS_REF_ERR_ARG;
    if (tn_make(g, &Q)) { tables_free(&T); return MAS_REF_ERR_ARG; }
#pragma omp parallel for schedule(static)
    for (i = 0; i < g->nr; i++) {
        int j, k, kind[6];
        double gf[6], V;
        size_t nb[6];
        for (j = 0; j <= g->nt; j++) {
            if (j == 0 || j == g->nt) {
                double num = 0.0, vcap = 0.0;
                for (k = 0; k < g->np; k++) {
                    size_t P = TIDX(g, i, j, k);
                    tn_slot(g, &T, &Q, i, j, k, &V, kind, gf, nb);
                    num += V * (c ? c[P] : 0.0) + tn_slot_diag(kind, gf, nb, kappa[P], kappa);
                    vcap += V;
                }
                for (k = 0; k < g->np; k++) D[TIDX(g, i, j, k)] = num / vcap;
            } else {
                for (k = 0; k < g->np; k++) {
                    size_t P = TIDX(g, i, j, k);
                    tn_slot(g, &T, &Q, i, j, k, &V, kind, gf, nb);
                    D[P] = (c ? c[P] : 0.0) + tn_slot_diag(kind, gf, nb, kappa[P], kappa) / V;
                }
            }
        }
    }
    tn_free(&Q);
    tables_free(&T);
    return MAS_REF_OK;
}

/* f += (1/V) G_b u_b on the Dirichlet r-faces (pole rows: the cap sum). */
int mas_ref_tn_dirichlet_rhs(const mas_ref_grid* g, int ncomp, const double* kappa,
                             const double* ub_inner, const double* ub_outer, double* f) {
    tables T;
    tn_tables Q;
    size_t N, plane;
    int m, side, j, k, kind[6];
    double gf[6], V;
    size_t nb[6];
    if (!g || !kappa || !f || ncomp < 1 || tables_make(g, &T)) return MAS_REF_ERR_ARG;
    if (tn_make(g, &Q)) { tables_free(&T); return MAS_REF_ERR_ARG; }
    N = (size_t)g->nr * (g->nt + 1) * g->np;
    plane = (size_t)(g->nt + 1) * g->np;
    for (m = 0; m < ncomp; m++)
        for (side = 0; side < 2; side++) {
            const double* ub = side ? ub_outer : ub_inner;
            const int i = side ? g->nr - 1 : 0, face = side ? 1 : 0;
            if (!ub || (side ? g->bc_outer : g->bc_inner) != MAS_REF_DIRICHLET) continue;
            for (j = 0; j <= g->nt; j++) {
                double num = 0.0, vcap = 0.0;
                for (k = 0; k < g->np; k++) {
                    size_t P = TIDX(g, i, j, k);
                    tn_slot(g, &T, &Q, i, j, k, &V, kind, gf, nb);
                    const double t = kappa[P] * gf[face] * ub[(size_t)m * plane + (size_t)j * g->np + k];
                    if (j == 0 || j == g->nt) { num += t; vcap += V; }
                    else f[(size_t)m * N + P] += t / V;
                }
                if (j == 0 || j == g->nt)
                    for (k = 0; k < g->np; k++) f[(size_t)m * N + TIDX(g, i, j, k)] += num / vcap;
            }
        }
    tn_free(&Q);
    tables_free(&T);
    return MAS_REF_OK;
}

/* <a,b>_V over the theta-node slots, per r-plane in (j,k) order, then planes,
 * then components (as dot_planes). */
static double tn_dot_raw(const mas_ref_grid* g, const double* V, int ncomp, const double* a,
                         const double* b) {
    size_t plane = (size_t)(g->nt + 1) * g->np, N = plane * g->nr;
    double s = 0.0;
    int m, i;
    for (m = 0; m < ncomp; m++)
        for (i = 0; i < g->nr; i++) {
            double ps = 0.0;
            size_t e;
            for (e = 0; e < plane; e++) {
                size_t P = (size_t)i * plane + e;
                ps += V[P] * a[(size_t)m * N + P] * b[(size_t)m * N + P];
            }
            s += ps;
        }
    return s;
}

int mas_ref_tn_dot(const mas_ref_grid* g, int ncomp, const double* a, const double* b, double* out) {
    double* V;
    if (!g || !a || !b || !out || ncomp < 1) return MAS_REF_ERR_ARG;
    V = malloc(sizeof(double) * (size_t)g->nr * (g->nt + 1) * g->np);
    if (!V || mas_ref_tn_volumes(g, V)) { free(V); return MAS_REF_ERR_ARG; }
    *out = tn_dot_raw(g, V, ncomp, a, b);
    free(V);
    return MAS_REF_OK;
}

/* Jacobi-PCG on the theta-node operator: the textbook loop of pcg_core
 * (R10-R12) with mas_ref_tn_apply / _diag / the theta-node inner product. */
int mas_ref_tn_pcg_solve(const mas_ref_grid* g, int ncomp, const double* kappa, const double* c,
                         const double* f, double* x, double tol, int maxit, int* iters,
                         double* relres, double* res_hist) {
    size_t N, n, e;
    double *V, *D, *r, *z, *p, *q;
    double bn, rn, rho, sigma, alpha, rho_new, beta;
    int k, m, status = MAS_REF_NOT_CONVERGED;
    if (!g || !kappa || !f || !x || !iters || !relres || ncomp < 1 || maxit < 0 || !(tol >= 0.0))
        return MAS_REF_ERR_ARG;
    N = (size_t)g->nr * (g->nt + 1) * g->np;
    n = N * ncomp;
    V = malloc(sizeof(double) * N);
    D = malloc(sizeof(double) * N);
    r = malloc(sizeof(double) * n);
    z = malloc(sizeof(double) * n);
    p = malloc(sizeof(double) * n);
    q = malloc(sizeof(double) * n);
    if (!V || !D || !r || !z || !p || !q || mas_ref_tn_volumes(g, V) || mas_ref_tn_diag(g, kappa, c, D)) {
        status = MAS_REF_ERR_ARG; goto done;
    }
    bn = sqrt(tn_dot_raw(g, V, ncomp, f, f));
    if (bn == 0.0) {
        for (e = 0; e < n; e++) x[e] = 0.0;
        *iters = 0; *relres = 0.0;
        if (res_hist) res_hist[0] = 0.0;
        status = MAS_REF_OK; goto done;
    }
    mas_ref_tn_apply(g, ncomp, kappa, c, x, r);
    for (e = 0; e < n; e++) r[e] = f[e] - r[e];
    rn = sqrt(tn_dot_raw(g, V, ncomp, r, r));
    if (res_hist) res_hist[0] = rn;
    if (rn <= tol * bn) { *iters = 0; *relres = rn / bn; status = MAS_REF_OK; goto done; }
    for (m = 0; m < ncomp; m++)
        for (e = 0; e < N; e++) z[m * N + e] = r[m * N + e] / D[e];
    memcpy(p, z, sizeof(double) * n);
    rho = tn_dot_raw(g, V, ncomp, r, z);
    for (k = 1; k <= maxit; k++) {
        mas_ref_tn_apply(g, ncomp, kappa, c, p, q);
        sigma = tn_dot_raw(g, V, ncomp, p, q);
        if (!(sigma > 0.0) || !isfinite(sigma)) {
            *iters = k; *relres = rn / bn; status = MAS_REF_ERR_BREAKDOWN; goto done;
        }
        alpha = rho / sigma;
        for (e = 0; e < n; e++) { x[e] += alpha * p[e]; r[e] -= alpha * q[e]; }
        rn = sqrt(tn_dot_raw(g, V, ncomp, r, r));
        if (res_hist) res_hist[k] = rn;
        if (rn <= tol * bn) { *iters = k; *relres = rn / bn; status = MAS_REF_OK; goto done; }
        for (m = 0; m < ncomp; m++)
            for (e = 0; e < N; e++) z[m * N + e] = r[m * N + e] / D[e];
        rho_new = tn_dot_raw(g, V, ncomp, r, z);
        beta = rho_new / rho;
        rho = rho_new;
        for (e = 0; e < n; e++) p[e] = z[e] + beta * p[e];
    }
    *iters = maxit; *relres = rn / bn; status = MAS_REF_NOT_CONVERGED;
done:
    free(V); free(D); free(r); free(z); free(p); free(q);
    return status;
}

/* ---------------------------------------------------------------------------
 * Vector-Laplacian curvature terms of the 3-component viscosity operator
 * (reading R31).  The components of the
 * viscosity unknown are the spherical components (v_r, v_theta, v_phi) (R13);
 * the vector Laplacian in spherical coordinates adds to each component's
 * scalar Laplacian a term in the SAME component,
 *   (lap v)_r     = lap v_r     - 2 v_r / r^2                 - (coupling)
 *   (lap v)_theta = lap v_theta - v_theta / (r^2 sin^2 theta) + (coupling)
 *   (lap v)_phi   = lap v_phi   - v_phi   / (r^2 sin^2 theta) + (coupling)
 * ("coupling": derivatives of the OTHER components, not included).  For
 * L v = c v - div(kappa grad v) the curvature terms are
 *   + kappa_P (2 / rC^2) v_r,  + kappa_P / (rC^2 sin^2 tC) v_theta,  + the same for v_phi,
 * evaluated at the cell centre (all >= 0: L stays SPD).  The Jacobi
 * preconditioner stays the shared 7-point diagonal D (R31).
 * ------------------------------------------------------------------------- */
static void curv_add(const mas_ref_grid* g, const double* kappa, const double* x, double* y) {
    size_t N = (size_t)g->nr * g->nt * g->np;
    int i;
#pragma omp parallel for schedule(static)
    for (i = 0; i < g->nr; i++) {
        int j, k, m;
        for (j = 0; j < g->nt; j++) {
            const double s = sin(g->tC[j]);
            const double w[3] = {2.0 / (g->rC[i] * g->rC[i]), 1.0 / (g->rC[i] * g->rC[i] * s * s),
                                 1.0 / (g->rC[i] * g->rC[i] * s * s)};
            for (k = 0; k < g->np; k++) {
                size_t P = IDX(g, i, j, k);
                for (m = 0; m < 3; m++) y[(size_t)m * N + P] += kappa[P] * w[m] * x[(size_t)m * N + P];
            }
        }
    }
}

int mas_ref_op_apply_curv(const mas_ref_grid* g, const double* kappa, const double* c,
                          const double* x, double* y) {
    int rc = mas_ref_op_apply(g, 3, kappa, c, x, y);
    if (rc == MAS_REF_OK) curv_add(g, kappa, x, y);
    return rc;
}

int mas_ref_pcg_solve_curv(const mas_ref_grid* g, const double* kappa, const double* c,
                           const double* f, double* x, double tol, int maxit, int* iters,
                           double* relres, double* res_hist) {
    return pcg_core(g, 3, kappa, c, NULL, NULL, 1, f, x, tol, maxit, iters, relres, res_hist);
}

/* ---------------------------------------------------------------------------
 * Face-centred placements of the staggered mesh (readings
 * R32-R33): MAS stores a velocity component on the faces
 * normal to it ("staggered"): v_r at the r faces, v_phi at the phi
 * faces (v_theta at the theta faces is the theta-node placement above).  As a
 * scalar unknown of the same operator L = c + (1/V) div(kappa grad):
 *
 * phi nodes (R33): unknowns at (rC_i, tC_j, pF_k), k = 0..np-1 (pF_np = pF_0 +
 *   2 pi).  The control volume of node k is the dual phi cell [pC_{k-1}, pC_k]
 *   (pC_{-1} = pC_{np-1} - 2 pi): it IS the cell-centred operator of R1-R16 on
 *   the dual phi mesh (faces pC_{k-1}, centres pF_k), which is how it is
 *   written here.
 * r nodes (R32): unknowns at (rF_i, tC_j, pC_k), i = 1..nr-1 (the boundary
 *   nodes rF_0, rF_nr carry the boundary values).  Node i's control volume is
 *   the dual r cell [rC_{i-1}, rC_i]:
 *     V = rF_i^2 (rC_i - rC_{i-1}) sin(tC) dt dp,
 *     r face at rC_{i-1}: g = rC_{i-1}^2 sin(tC) dt dp / (rF_i - rF_{i-1})
 *       (node i-1; for i = 1 the boundary node rF_0: Dirichlet with kappa_P
 *        and u_b, or Neumann: no flux), likewise at rC_i (node i+1 / rF_nr),
 *     theta / phi faces as R4 with the dual cell's r extent rC_i - rC_{i-1}.
 *   Arrays [comp][nr-1][nt][np].
 * ------------------------------------------------------------------------- */
static int pn_dual_grid(const mas_ref_grid* g, mas_ref_grid* d, double** pF, double** pC) {
    int np = g->np, k;
    *pF = malloc(sizeof(double) * (np + 1));
    *pC = malloc(sizeof(double) * np);
    if (!*pF || !*pC) { free(*pF); free(*pC); return MAS_REF_ERR_ARG; }
    (*pF)[0] = g->pC[np - 1] - TWO_PI;
    for (k = 1; k <= np; k++) (*pF)[k] = g->pC[k - 1];
    for (k = 0; k < np; k++) (*pC)[k] = g->pF[k];
    *d = *g;
    d->pF = *pF;
    d->pC = *pC;
    return MAS_REF_OK;
}

int mas_ref_pn_apply(const mas_ref_grid* g, int ncomp, const double* kappa, const double* c,
                     const double* x, double* y) {
    mas_ref_grid d;
    double *pF, *pC;
    int rc;
    if (!g || pn_dual_grid(g, &d, &pF, &pC)) return MAS_REF_ERR_ARG;
    rc = mas_ref_op_apply(&d, ncomp, kappa, c, x, y);
    free(pF); free(pC);
    return rc;
}

int mas_ref_pn_volumes(const mas_ref_grid* g, double* V) {
    mas_ref_grid d;
    double *pF, *pC;
    int rc;
    if (!g || pn_dual_grid(g, &d, &pF, &pC)) return MAS_REF_ERR_ARG;
    rc = mas_ref_volumes(&d, V);
    free(pF); free(pC);
    return rc;
}

int mas_ref_pn_pcg_solve(const mas_ref_grid* g, int ncomp, const double* kappa, const double* c,
                         const double* f, double* x, double tol, int maxit, int* iters,
                         double* relres, double* res_hist) {
    mas_ref_grid d;
    double *pF, *pC;
    int rc;
    if (!g || pn_dual_grid(g, &d, &pF, &pC)) return MAS_REF_ERR_ARG;
    rc = mas_ref_pcg_solve(&d, ncomp, kappa, c, f, x, tol, maxit, iters, relres, res_hist);
    free(pF); free(pC);
    return rc;
}

/* r nodes: the slot of node i (1..nr-1) at (j, k): volume, face kinds /
 * conductances, neighbours (flat indices of [nr-1][nt][np]) */
#define RIDX(g, i, j, k) ((((size_t)(i) - 1) * (g)->nt + (size_t)(j)) * (g)->np + (size_t)(k))
static void rn_slot(const mas_ref_grid* g, const tables* T, int i, int j, int k, double* V, int kind[6],
                    double gf[6], size_t nb[6]) {
    const int nr = g->nr, np = g->np;
    const double drd = g->rC[i] - g->rC[i - 1];   /* the dual cell's r extent */
    int f;
    for (f = 0; f < 6; f++) { kind[f] = FACE_NONE; gf[f] = 0.0; nb[f] = 0; }
    *V = g->rF[i] * g->rF[i] * drd * T->sC[j] * T->dt[j] * T->dp[k];
    kind[0] = (i > 1) ? FACE_INTERIOR : (g->bc_inner == MAS_REF_DIRICHLET ? FACE_DIRICHLET : FACE_NONE);
    kind[1] = (i < nr - 1) ? FACE_INTERIOR : (g->bc_outer == MAS_REF_DIRICHLET ? FACE_DIRICHLET : FACE_NONE);
    if (kind[0]) gf[0] = g->rC[i - 1] * g->rC[i - 1] * T->sC[j] * T->dt[j] * T->dp[k] / (g->rF[i] - g->rF[i - 1]);
    if (kind[1]) gf[1] = g->rC[i] * g->rC[i] * T->sC[j] * T->dt[j] * T->dp[k] / (g->rF[i + 1] - g->rF[i]);
    if (kind[0] == FACE_INTERIOR) nb[0] = RIDX(g, i - 1, j, k);
    if (kind[1] == FACE_INTERIOR) nb[1] = RIDX(g, i + 1, j, k);
    if (j > 0) {
        kind[2] = FACE_INTERIOR;
        gf[2] = drd * T->sF[j] * T->dp[k] / T->ht[j];
        nb[2] = RIDX(g, i, j - 1, k);
    }
    if (j < g->nt - 1) {
        kind[3] = FACE_INTERIOR;
        gf[3] = drd * T->sF[j + 1] * T->dp[k] / T->ht[j + 1];
        nb[3] = RIDX(g, i, j + 1, k);
    }
    kind[4] = kind[5] = FACE_INTERIOR;
    gf[4] = drd * T->dt[j] / (T->sC[j] * T->hp[k]);
    gf[5] = drd * T->dt[j] / (T->sC[j] * T->hp[(k + 1) % np]);
    nb[4] = RIDX(g, i, j, (k + np - 1) % np);
    nb[5] = RIDX(g, i, j, (k + 1) % np);
}

int mas_ref_rn_volumes(const mas_ref_grid* g, double* V) {
    tables T;
    int i, j, k, kind[6];
    double gf[6];
    size_t nb[6];
    if (!g || !V || g->nr < 2 || tables_make(g, &T)) return MAS_REF_ERR_ARG;
    for (i = 1; i < g->nr; i++)
        for (j = 0; j < g->nt; j++)
            for (k = 0; k < g->np; k++) rn_slot(g, &T, i, j, k, &V[RIDX(g, i, j, k)], kind, gf, nb);
    tables_free(&T);
    return MAS_REF_OK;
}

int mas_ref_rn_apply(const mas_ref_grid* g, int ncomp, const double* kappa, const double* c,
                     const double* x, double* y) {
    tables T;
    size_t N;
    int i;
    if (!g || !kappa || !x || !y || ncomp < 1 || g->nr < 2 || tables_make(g, &T)) return MAS_REF_ERR_ARG;
    N = (size_t)(g->nr - 1) * g->nt * g->np;
#pragma omp parallel for schedule(static)
    for (i = 1; i < g->nr; i++) {
        int j, k, m, kind[6];
        double gf[6], V;
        size_t nb[6];
        for (j = 0; j < g->nt; j++)
            for (k = 0; k < g->np; k++) {
                const size_t P = RIDX(g, i, j, k);
                rn_slot(g, &T, i, j, k, &V, kind, gf, nb);
                for (m = 0; m < ncomp; m++) {
                    const double* u = x + (size_t)m * N;
                    y[(size_t)m * N + P] = (c ? c[P] : 0.0) * u[P] +
                                           tn_slot_flux(kind, gf, nb, kappa[P], u[P], kappa, u) / V;
                }
            }
    }
    tables_free(&T);
    return MAS_REF_OK;
}

int mas_ref_rn_diag(const mas_ref_grid* g, const double* kappa, const double* c, double* D) {
    tables T;
    int i;
    if (!g || !kappa || !D || g->nr < 2 || tables_make(g, &T)) return MAS_REF_ERR_ARG;
#pragma omp parallel for schedule(static)
    for (i = 1; i < g->nr; i++) {
        int j, k, kind[6];
        double gf[6], V;
        size_t nb[6];
        for (j = 0; j < g->nt; j++)
            for (k = 0; k < g->np; k++) {
                const size_t P = RIDX(g, i, j, k);
                rn_slot(g, &T, i, j, k, &V, kind, gf, nb);
                D[P] = (c ? c[P] : 0.0) + tn_slot_diag(kind, gf, nb, kappa[P], kappa) / V;
            }
    }
    tables_free(&T);
    return MAS_REF_OK;
}

/* f += (1/V) G_b u_b at the boundary nodes' faces; ub [ncomp][nt][np] */
int mas_ref_rn_dirichlet_rhs(const mas_ref_grid* g, int ncomp, const double* kappa,
                             const double* ub_inner, const double* ub_outer, double* f) {
    tables T;
    size_t N, plane;
    int m, side, j, k, kind[6];
    double gf[6], V;
    size_t nb[6];
    if (!g || !kappa || !f || ncomp < 1 || g->nr < 2 || tables_make(g, &T)) return MAS_REF_ERR_ARG;
    N = (size_t)(g->nr - 1) * g->nt * g->np;
    plane = (size_t)g->nt * g->np;
    for (m = 0; m < ncomp; m++)
        for (side = 0; side < 2; side++) {
            const double* ub = side ? ub_outer : ub_inner;
            const int i = side ? g->nr - 1 : 1, face = side ? 1 : 0;
            if (!ub || (side ? g->bc_outer : g->bc_inner) != MAS_REF_DIRICHLET) continue;
            for (j = 0; j < g->nt; j++)
                for (k = 0; k < g->np; k++) {
                    const size_t P = RIDX(g, i, j, k);
                    rn_slot(g, &T, i, j, k, &V, kind, gf, nb);
                    f[(size_t)m * N + P] += kappa[P] * gf[face] * ub[(size_t)m * plane + (size_t)j * g->np + k] / V;
                }
        }
    tables_free(&T);
    return MAS_REF_OK;
}

/* Jacobi-PCG on the r-node operator (the textbook loop of pcg_core). */
int mas_ref_rn_pcg_solve(const mas_ref_grid* g, int ncomp, const double* kappa, const double* c,
                         const double* f, double* x, double tol, int maxit, int* iters,
                         double* relres, double* res_hist) {
    size_t N, n, e;
    double *V, *D, *r, *z, *p, *q;
    double bn, rn, rho, sigma, alpha, rho_new, beta;
    int k, m, status = MAS_REF_NOT_CONVERGED;
    if (!g || !kappa || !f || !x || !iters || !relres || ncomp < 1 || maxit < 0 || !(tol >= 0.0) || g->nr < 2)
        return MAS_REF_ERR_ARG;
    N = (size_t)(g->nr - 1) * g->nt * g->np;
    n = N * ncomp;
    V = malloc(sizeof(double) * N);
    D = malloc(sizeof(double) * N);
    r = malloc(sizeof(double) * n);
    z = malloc(sizeof(double) * n);
    p = malloc(sizeof(double) * n);
    q = malloc(sizeof(double) * n);
    if (!V || !D || !r || !z || !p || !q || mas_ref_rn_volumes(g, V) || mas_ref_rn_diag(g, kappa, c, D)) {
        status = MAS_REF_ERR_ARG; goto done;
    }
    /* the V-weighted dot, per node plane in (j,k) order, then planes, then components */
#define RDOT(a, b, out) do { size_t pl = (size_t)g->nt * g->np; int mm, ii; double s_ = 0.0; \
        for (mm = 0; mm < ncomp; mm++) for (ii = 0; ii < g->nr - 1; ii++) { double ps = 0.0; size_t ee; \
            for (ee = 0; ee < pl; ee++) { size_t P_ = (size_t)ii * pl + ee; \
                ps += V[P_] * (a)[(size_t)mm * N + P_] * (b)[(size_t)mm * N + P_]; } s_ += ps; } \
        (out) = s_; } while (0)
    RDOT(f, f, bn);
    bn = sqrt(bn);
    if (bn == 0.0) {
        for (e = 0; e < n; e++) x[e] = 0.0;
        *iters = 0; *relres = 0.0;
        if (res_hist) res_hist[0] = 0.0;
        status = MAS_REF_OK; goto done;
    }
    mas_ref_rn_apply(g, ncomp, kappa, c, x, r);
    for (e = 0; e < n; e++) r[e] = f[e] - r[e];
    RDOT(r, r, rn);
    rn = sqrt(rn);
    if (res_hist) res_hist[0] = rn;
    if (rn <= tol * bn) { *iters = 0; *relres = rn / bn; status = MAS_REF_OK; goto done; }
    for (m = 0; m < ncomp; m++)
        for (e = 0; e < N; e++) z[m * N + e] = r[m * N + e] / D[e];
    memcpy(p, z, sizeof(double) * n);
    RDOT(r, z, rho);
    for (k = 1; k <= maxit; k++) {
        mas_ref_rn_apply(g, ncomp, kappa, c, p, q);
        RDOT(p, q, sigma);
        if (!(sigma > 0.0) || !isfinite(sigma)) {
            *iters = k; *relres = rn / bn; status = MAS_REF_ERR_BREAKDOWN; goto done;
        }
        alpha = rho / sigma;
        for (e = 0; e < n; e++) { x[e] += alpha * p[e]; r[e] -= alpha * q[e]; }
        RDOT(r, r, rn);
        rn = sqrt(rn);
        if (res_hist) res_hist[k] = rn;
        if (rn <= tol * bn) { *iters = k; *relres = rn / bn; status = MAS_REF_OK; goto done; }
        for (m = 0; m < ncomp; m++)
            for (e = 0; e < N; e++) z[m * N + e] = r[m * N + e] / D[e];
        RDOT(r, z, rho_new);
        beta = rho_new / rho;
        rho = rho_new;
        for (e = 0; e < n; e++) p[e] = z[e] + beta * p[e];
    }
#undef RDOT
    *iters = maxit; *relres = rn / bn; status = MAS_REF_NOT_CONVERGED;
done:
    free(V); free(D); free(r); free(z); free(p); free(q);
    return status;
}

int mas_ref_pn_diag(const mas_ref_grid* g, const double* kappa, const double* c, double* D) {
    mas_ref_grid d;
    double *pF, *pC;
    int rc;
    if (!g || pn_dual_grid(g, &d, &pF, &pC)) return MAS_REF_ERR_ARG;
    rc = mas_ref_op_diag(&d, kappa, c, D);
    free(pF); free(pC);
    return rc;
}

int mas_ref_pn_dirichlet_rhs(const mas_ref_grid* g, int ncomp, const double* kappa,
                             const double* ub_inner, const double* ub_outer, double* f) {
    mas_ref_grid d;
    double *pF, *pC;
    int rc;
    if (!g || pn_dual_grid(g, &d, &pF, &pC)) return MAS_REF_ERR_ARG;
    rc = mas_ref_dirichlet_rhs(&d, ncomp, kappa, ub_inner, ub_outer, f);
    free(pF); free(pC);
    return rc;
}

/* ---------------------------------------------------------------------------
 * Stacked PCG over several placed operators (NEXT-2, reading R34).
 * MAS solves the viscous step for the velocity VECTOR, each component at its
 * staggered location ("staggered spherical grid"; the survey's R13
 * takes one PCG on the stacked vector with the summed inner product).  With
 * the components at different locations the operator is block-diagonal: block
 * b is the placed operator of its location (R1-R16 on the cell centres, R29
 * theta nodes, R32 r nodes, R33 phi nodes) with its own D, V and arrays.  The
 * loop is pcg_core's, line for line; every inner product is the sum over the
 * blocks (in block order) of the block's V-weighted one.
 * ------------------------------------------------------------------------- */
static size_t stk_cells(const mas_ref_grid* g, int pl) {
    switch (pl) {
    case MAS_REF_PLACE_THETA_NODE: return (size_t)g->nr * (g->nt + 1) * g->np;
    case MAS_REF_PLACE_R_NODE: return (size_t)(g->nr - 1) * g->nt * g->np;
    default: return (size_t)g->nr * g->nt * g->np;
    }
}
static int stk_apply(const mas_ref_grid* g, int pl, int ncomp, const double* kappa, const double* c,
                     const double* x, double* y) {
    switch (pl) {
    case MAS_REF_PLACE_CELL: return mas_ref_op_apply(g, ncomp, kappa, c, x, y);
    case MAS_REF_PLACE_THETA_NODE: return mas_ref_tn_apply(g, ncomp, kappa, c, x, y);
    case MAS_REF_PLACE_R_NODE: return mas_ref_rn_apply(g, ncomp, kappa, c, x, y);
    case MAS_REF_PLACE_PHI_NODE: return mas_ref_pn_apply(g, ncomp, kappa, c, x, y);
    default: return MAS_REF_ERR_ARG;
    }
}
static int stk_diag(const mas_ref_grid* g, int pl, const double* kappa, const double* c, double* D) {
    switch (pl) {
    case MAS_REF_PLACE_CELL: return mas_ref_op_diag(g, kappa, c, D);
    case MAS_REF_PLACE_THETA_NODE: return mas_ref_tn_diag(g, kappa, c, D);
    case MAS_REF_PLACE_R_NODE: return mas_ref_rn_diag(g, kappa, c, D);
    case MAS_REF_PLACE_PHI_NODE: return mas_ref_pn_diag(g, kappa, c, D);
    default: return MAS_REF_ERR_ARG;
    }
}
static int stk_volumes(const mas_ref_grid* g, int pl, double* V) {
    switch (pl) {
    case MAS_REF_PLACE_CELL: return mas_ref_volumes(g, V);
    case MAS_REF_PLACE_THETA_NODE: return mas_ref_tn_volumes(g, V);
    case MAS_REF_PLACE_R_NODE: return mas_ref_rn_volumes(g, V);
    case MAS_REF_PLACE_PHI_NODE: return mas_ref_pn_volumes(g, V);
    default: return MAS_REF_ERR_ARG;
    }
}
/* sum over the blocks of sum_m sum_P V_P a_m,P b_m,P (per block: per
 * component, per r-plane partial sums, as dot_planes) */
static double stk_dot(int nblk, const mas_ref_grid* const* g, const int* pl, const int* ncomp,
                      double* const* V, double* const* a, double* const* b) {
    double s = 0.0;
    int q, m, i;
    for (q = 0; q < nblk; q++) {
        const size_t N = stk_cells(g[q], pl[q]);
        const int nplanes = pl[q] == MAS_REF_PLACE_R_NODE ? g[q]->nr - 1 : g[q]->nr;
        const size_t plane = N / (size_t)nplanes;
        double sb = 0.0;
        for (m = 0; m < ncomp[q]; m++)
            for (i = 0; i < nplanes; i++) {
                double ps = 0.0;
                size_t e;
                for (e = 0; e < plane; e++) {
                    const size_t P = (size_t)i * plane + e;
                    ps += V[q][P] * a[q][(size_t)m * N + P] * b[q][(size_t)m * N + P];
                }
                sb += ps;
            }
        s += sb;
    }
    return s;
}

int mas_ref_stacked_pcg_solve(int nblk, const mas_ref_grid* const* g, const int* pl,
                              const int* ncomp, const double* const* kappa, const double* const* c,
                              const double* const* f, double* const* x, double tol, int maxit,
                              int* iters, double* relres, double* res_hist) {
    double *V[MAS_REF_MAX_STACK] = {0}, *D[MAS_REF_MAX_STACK] = {0}, *r[MAS_REF_MAX_STACK] = {0},
           *z[MAS_REF_MAX_STACK] = {0}, *p[MAS_REF_MAX_STACK] = {0}, *q[MAS_REF_MAX_STACK] = {0};
    double* fc[MAS_REF_MAX_STACK];
    size_t N[MAS_REF_MAX_STACK];
    double bn, rn, rho, sigma, alpha, rho_new, beta;
    int k, b, m, status = MAS_REF_NOT_CONVERGED;
    size_t e;
    if (nblk < 1 || nblk > MAS_REF_MAX_STACK || !g || !pl || !ncomp || !kappa || !c || !f || !x ||
        !iters || !relres || maxit < 0 || !(tol >= 0.0))
        return MAS_REF_ERR_ARG;
    for (b = 0; b < nblk; b++) {
        if (!g[b] || !kappa[b] || !f[b] || !x[b] || ncomp[b] < 1 || pl[b] < MAS_REF_PLACE_CELL ||
            pl[b] > MAS_REF_PLACE_PHI_NODE || (pl[b] == MAS_REF_PLACE_R_NODE && g[b]->nr < 2))
            return MAS_REF_ERR_ARG;
        N[b] = stk_cells(g[b], pl[b]);
        fc[b] = (double*)f[b];
    }
    for (b = 0; b < nblk; b++) {
        const size_t n = N[b] * ncomp[b];
        V[b] = malloc(sizeof(double) * N[b]);
        D[b] = malloc(sizeof(double) * N[b]);
        r[b] = malloc(sizeof(double) * n);
        z[b] = malloc(sizeof(double) * n);
        p[b] = malloc(sizeof(double) * n);
        q[b] = malloc(sizeof(double) * n);
        if (!V[b] || !D[b] || !r[b] || !z[b] || !p[b] || !q[b] || stk_volumes(g[b], pl[b], V[b]) ||
            stk_diag(g[b], pl[b], kappa[b], c[b], D[b])) {
            status = MAS_REF_ERR_ARG; goto done;
        }
    }
    bn = sqrt(stk_dot(nblk, g, pl, ncomp, V, fc, fc));
    if (bn == 0.0) {
        for (b = 0; b < nblk; b++)
            for (e = 0; e < N[b] * ncomp[b]; e++) x[b][e] = 0.0;
        *iters = 0; *relres = 0.0;
        if (res_hist) res_hist[0] = 0.0;
        status = MAS_REF_OK; goto done;
    }
    for (b = 0; b < nblk; b++) {                                 /* r = f - L x */
        stk_apply(g[b], pl[b], ncomp[b], kappa[b], c[b], x[b], r[b]);
        for (e = 0; e < N[b] * ncomp[b]; e++) r[b][e] = f[b][e] - r[b][e];
    }
    rn = sqrt(stk_dot(nblk, g, pl, ncomp, V, r, r));
    if (res_hist) res_hist[0] = rn;
    if (rn <= tol * bn) { *iters = 0; *relres = rn / bn; status = MAS_REF_OK; goto done; }
    for (b = 0; b < nblk; b++) {                                 /* z = D^-1 r, p = z */
        for (m = 0; m < ncomp[b]; m++)
            for (e = 0; e < N[b]; e++) z[b][m * N[b] + e] = r[b][m * N[b] + e] / D[b][e];
        memcpy(p[b], z[b], sizeof(double) * N[b] * ncomp[b]);
    }
    rho = stk_dot(nblk, g, pl, ncomp, V, r, z);
    for (k = 1; k <= maxit; k++) {
        for (b = 0; b < nblk; b++) stk_apply(g[b], pl[b], ncomp[b], kappa[b], c[b], p[b], q[b]);
        sigma = stk_dot(nblk, g, pl, ncomp, V, p, q);
        if (!(sigma > 0.0) || !isfinite(sigma)) {
            *iters = k; *relres = rn / bn; status = MAS_REF_ERR_BREAKDOWN; goto done;
        }
        alpha = rho / sigma;
        for (b = 0; b < nblk; b++)
            for (e = 0; e < N[b] * ncomp[b]; e++) { x[b][e] += alpha * p[b][e]; r[b][e] -= alpha * q[b][e]; }
        rn = sqrt(stk_dot(nblk, g, pl, ncomp, V, r, r));
        if (res_hist) res_hist[k] = rn;
        if (rn <= tol * bn) { *iters = k; *relres = rn / bn; status = MAS_REF_OK; goto done; }
        for (b = 0; b < nblk; b++)
            for (m = 0; m < ncomp[b]; m++)
                for (e = 0; e < N[b]; e++) z[b][m * N[b] + e] = r[b][m * N[b] + e] / D[b][e];
        rho_new = stk_dot(nblk, g, pl, ncomp, V, r, z);
        beta = rho_new / rho;
        rho = rho_new;
        for (b = 0; b < nblk; b++)
            for (e = 0; e < N[b] * ncomp[b]; e++) p[b][e] = z[b][e] + beta * p[b][e];
    }
    *iters = maxit; *relres = rn / bn; status = MAS_REF_NOT_CONVERGED;
done:
    for (b = 0; b < nblk; b++) { free(V[b]); free(D[b]); free(r[b]); free(z[b]); free(p[b]); free(q[b]); }
    return status;
}
