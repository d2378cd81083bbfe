// grid.cpp — mas_grid_create: mesh validation, 1-D metric/coefficient tables
// and the r-slab partition (host C++; a1 of SURVEY.md §8(a)).
//
// The mesh is MAS's "logically rectangular non-uniform staggered spherical
// grid" (§III): node (face) and half (centre) meshes in r,
// theta, phi (reading R1).  The tables below are the 1-D factors of the
// finite-difference midpoint metrics (reading R4):
//   V = rC^2 dr * sin(tC) dt * dp
//   G_r(i)/V = rF_i^2 / (hr_i rC^2 dr)                      -> wRm, wRp
//   G_t(j)/V = sin(tF_j) / (ht_j sin(tC) dt) * 1/rC^2        -> wTm, wTp, irc2
//   G_p(k)/V = 1 / (hp_k dp) * 1/(rC^2 sin^2(tC))            -> wPm, wPp, isc2
// with hr at the r-boundaries the half-cell distance (R3), hp periodic (R7)
// and the theta faces 0 and nt carrying no flux (poles / walls, R5).
#include <cmath>
#include <cstring>
#include <new>
#include <string>
#include <vector>

#include "grid.h"

namespace mas {

static const double kTwoPi = 6.283185307179586476925286766559;

static bool strictly_inside(const double* node, const double* half, int n, std::string* why,
                            const char* name) {
    for (int i = 0; i < n; i++) {
        if (!(node[i] < node[i + 1])) {
            *why = std::string(name) + "_node is not strictly increasing at " + std::to_string(i);
            return false;
        }
        if (!(half[i] > node[i] && half[i] < node[i + 1])) {
            *why = std::string(name) + "_half[" + std::to_string(i) + "] is not inside its cell";
            return false;
        }
    }
    return true;
}

int validate_mesh(int nr, int nt, int np, const double* rF, const double* rC, const double* tF,
                  const double* tC, const double* pF, const double* pC, int pole_flags,
                  int periodic_phi, int pr, int ptheta, std::string* why) {
    if (!rF || !rC || !tF || !tC || !pF || !pC) { *why = "null mesh pointer"; return 0; }
    if (nr < 1 || nt < 1 || np < 2) { *why = "need nr >= 1, nt >= 1, np >= 2"; return 0; }
    if (np % 2) { *why = "np must be even (16-byte phi pairs)"; return 0; }
    if (pr < 1 || nr < pr) { *why = "need nr >= nranks / ptheta >= 1"; return 0; }
    if (ptheta < 1 || nt < ptheta) { *why = "need nt >= ptheta >= 1"; return 0; }
    if ((long long)nt * np > (1LL << 30)) { *why = "theta-phi plane too large"; return 0; }
    if (!periodic_phi) { *why = "periodic_phi must be 1 (reading R7)"; return 0; }
    if (pole_flags & ~(MAS_POLE_NORTH | MAS_POLE_SOUTH)) { *why = "unknown pole flag"; return 0; }
    for (int i = 0; i <= nr; i++)
        if (!std::isfinite(rF[i])) { *why = "non-finite r_node"; return 0; }
    for (int i = 0; i <= nt; i++)
        if (!std::isfinite(tF[i])) { *why = "non-finite t_node"; return 0; }
    for (int i = 0; i <= np; i++)
        if (!std::isfinite(pF[i])) { *why = "non-finite p_node"; return 0; }
    if (!strictly_inside(rF, rC, nr, why, "r")) return 0;
    if (!strictly_inside(tF, tC, nt, why, "t")) return 0;
    if (!strictly_inside(pF, pC, np, why, "p")) return 0;
    if (!(rF[0] > 0.0)) { *why = "r_node[0] must be > 0"; return 0; }
    if (tF[0] < 0.0 || tF[nt] > M_PI) { *why = "t_node outside [0, pi]"; return 0; }
    if ((pole_flags & MAS_POLE_NORTH) && tF[0] != 0.0) {
        *why = "north pole flag requires t_node[0] == 0";
        return 0;
    }
    if ((pole_flags & MAS_POLE_SOUTH) && std::fabs(tF[nt] - M_PI) > 4.0 * 2.220446049250313e-16) {
        *why = "south pole flag requires t_node[nt] == pi";
        return 0;
    }
    if (std::fabs((pF[np] - pF[0]) - kTwoPi) > 1e-12 * kTwoPi) {
        *why = "p_node must span exactly 2 pi (periodic phi)";
        return 0;
    }
    for (int j = 0; j < nt; j++)
        if (!(std::sin(tC[j]) > 0.0)) { *why = "sin(t_half) must be > 0"; return 0; }
    return 1;
}

void partition(int nr, int nranks, int rank, int* i0, int* nl) {
    const int base = nr / nranks, rem = nr % nranks;
    *nl = base + (rank < rem ? 1 : 0);
    *i0 = rank * base + (rank < rem ? rank : rem);
}

void build_tables(mas_grid* g) {
    const int nr = g->nr, nt = g->nt, np = g->np, i0 = g->i0, nl = g->nl;
    const int j0 = g->j0, ntl = g->ntl;  // local theta rows (global faces 0 / nt stay flux-free)
    const double *rF = g->rF.data(), *rC = g->rC.data(), *tF = g->tF.data(), *tC = g->tC.data(),
                 *pF = g->pF.data(), *pC = g->pC.data();
    Tables& T = g->tab;
    T.wRm.assign(nl, 0.0); T.wRp.assign(nl, 0.0); T.irc2.assign(nl, 0.0); T.vr.assign(nl, 0.0);
    T.wTm.assign(ntl, 0.0); T.wTp.assign(ntl, 0.0); T.isc2.assign(ntl, 0.0); T.vt.assign(ntl, 0.0);
    T.wPm.assign(np, 0.0); T.wPp.assign(np, 0.0); T.vp.assign(np, 0.0);
    auto hr = [&](int f) {  // centre distance across r-face f (R3 at the boundaries)
        if (f == 0) return rC[0] - rF[0];
        if (f == nr) return rF[nr] - rC[nr - 1];
        return rC[f] - rC[f - 1];
    };
    for (int il = 0; il < nl; il++) {
        const int i = i0 + il;
        const double dr = rF[i + 1] - rF[i], rc2 = rC[i] * rC[i];
        T.wRm[il] = rF[i] * rF[i] / (hr(i) * rc2 * dr);
        T.wRp[il] = rF[i + 1] * rF[i + 1] / (hr(i + 1) * rc2 * dr);
        T.irc2[il] = 1.0 / rc2;
        T.vr[il] = rc2 * dr;
    }
    for (int jl = 0; jl < ntl; jl++) {
        const int j = j0 + jl;
        const double dt = tF[j + 1] - tF[j], sC = std::sin(tC[j]);
        if (j > 0) T.wTm[jl] = std::sin(tF[j]) / ((tC[j] - tC[j - 1]) * sC * dt);
        if (j < nt - 1) T.wTp[jl] = std::sin(tF[j + 1]) / ((tC[j + 1] - tC[j]) * sC * dt);
        T.isc2[jl] = 1.0 / (sC * sC);
        T.vt[jl] = sC * dt;
    }
    std::vector<double> hp(np);
    hp[0] = pC[0] + kTwoPi - pC[np - 1];
    for (int k = 1; k < np; k++) hp[k] = pC[k] - pC[k - 1];
    for (int k = 0; k < np; k++) {
        const double dp = pF[k + 1] - pF[k];
        T.wPm[k] = 1.0 / (hp[k] * dp);
        T.wPp[k] = 1.0 / (hp[(k + 1) % np] * dp);
        T.vp[k] = dp;
    }
}

// theta-node placement (NEXT-2, readings R29-R30):
// rows j = 0..nt at tF_j; interior rows span [tC_{j-1}, tC_j] (theta measure
// m_j = sin(tF_j)(tC_j - tC_{j-1})), the pole rows are polar-cap slices of
// measure A = 1 - cos(tC_0) (north) and 1 + cos(tC_{nt-1}) (south) without
// phi faces.  Same layout as Tables' theta part: [wTm | wTp | isc2 | vt](nt+1).
std::vector<double> tnode_tables(const mas_grid* g) {
    const int nt = g->nt;
    const double *tF = g->tF.data(), *tC = g->tC.data();
    std::vector<double> t(4 * (size_t)(nt + 1), 0.0);
    double *wTm = t.data(), *wTp = wTm + nt + 1, *isc2 = wTp + nt + 1, *vt = isc2 + nt + 1;
    for (int j = 0; j <= nt; j++) {
        double m;
        if (j == 0) m = 1.0 - std::cos(tC[0]);
        else if (j == nt) m = 1.0 + std::cos(tC[nt - 1]);
        else m = std::sin(tF[j]) * (tC[j] - tC[j - 1]);
        vt[j] = m;
        if (j > 0) wTm[j] = std::sin(tC[j - 1]) / ((tF[j] - tF[j - 1]) * m);
        if (j < nt) wTp[j] = std::sin(tC[j]) / ((tF[j + 1] - tF[j]) * m);
        if (j > 0 && j < nt) isc2[j] = 1.0 / (std::sin(tF[j]) * std::sin(tF[j]));  // pole rows: no phi faces
    }
    return t;
}

// phi-node placement (NEXT-2, R33): unknowns at pF_k; the dual phi cells
// [pC_{k-1}, pC_k] (width hp_k) with node distances pF_k - pF_{k-1} (dp_{k-1},
// periodic).  Same layout as Tables' phi part: [wPm | wPp | vp](np).
std::vector<double> pnode_tables(const mas_grid* g) {
    const int np = g->np;
    const double *pF = g->pF.data(), *pC = g->pC.data();
    std::vector<double> t(3 * (size_t)np);
    double *wPm = t.data(), *wPp = wPm + np, *vp = wPp + np;
    auto width = [&](int k) { return k == 0 ? pC[0] + kTwoPi - pC[np - 1] : pC[k] - pC[k - 1]; };
    auto dist = [&](int k) { k = (k + np) % np; return pF[k == 0 ? np : k] - pF[k == 0 ? np - 1 : k - 1]; };
    for (int k = 0; k < np; k++) {
        const double w = width(k);
        wPm[k] = 1.0 / (dist(k) * w);
        wPp[k] = 1.0 / (dist(k + 1) * w);
        vp[k] = w;
    }
    return t;
}

// r-node placement (NEXT-2, R32): unknowns at rF_i, i = 1..nr-1 (one rank);
// the dual r cells [rC_{i-1}, rC_i] with node distances rF_i - rF_{i-1}; the
// boundary nodes rF_0 / rF_nr are the Dirichlet faces' values.
// [wRm | wRp | irc2 | vr](nr-1)
std::vector<double> rnode_tables(const mas_grid* g) {
    const int n = g->nr - 1;
    const double *rF = g->rF.data(), *rC = g->rC.data();
    std::vector<double> t(4 * (size_t)(n > 0 ? n : 0));
    double *wRm = t.data(), *wRp = wRm + n, *irc2 = wRp + n, *vr = irc2 + n;
    for (int l = 0; l < n; l++) {
        const int i = l + 1;
        const double drd = rC[i] - rC[i - 1], rf2 = rF[i] * rF[i];
        wRm[l] = rC[i - 1] * rC[i - 1] / ((rF[i] - rF[i - 1]) * rf2 * drd);
        wRp[l] = rC[i] * rC[i] / ((rF[i + 1] - rF[i]) * rf2 * drd);
        irc2[l] = 1.0 / rf2;
        vr[l] = rf2 * drd;
    }
    return t;
}

}  // namespace mas
