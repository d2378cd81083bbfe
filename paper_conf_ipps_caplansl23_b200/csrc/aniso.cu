// aniso.cu — the field-aligned (anisotropic) thermal-conduction term L_par of
// the implicit conduction operator (readings R21-R26
// in DESIGN.md §3.4).  MAS conducts heat along the magnetic field; the paper
// names the thermodynamic model of its test problem and the
// implicit Krylov schemes of ref. [25] but prints no formula.
//
//   V_P (L_par u)_P = sum_{corners c of P} s_c (sr a_c + st b_c + sp e_c)
//   s_c = a_c Dr_c(u) + b_c Dt_c(u) + e_c Dp_c(u)
//
// (mas_internal.h).  The corner form is symmetric positive semi-definite in
// the V-weighted inner product, so L_iso + L_par keeps PCG applicable.
//
// k_aniso runs right after the fused stencil kernel of the same mode and adds
// its term in place (APPLY: y += L_par x; RESID: r -= L_par x and the three
// initial dots; PCGA: q += L_par p_k and sigma += <p_k, L_par p_k>_V), so
// kernel A and kernel B are unchanged.  Work item: one 8 (theta) x 64 (phi)
// cell tile x one chunk of r-planes; the block marches the corner planes
// I = ia..ib: p plane I (tile + 1-cell halo, periodic in phi) into a 2-slot
// shared ring, the (9 x 65) corner products (s a, s b, s e) of plane I into a
// second 2-slot ring, then the cells of plane I-1 gather their 8 corners.
// Bytes per cell (PCGA): p 8 + (a, b, e) 24 + q read/write 16 = 48 B.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdlib>

#include "mas_internal.h"
#include "reduce.cuh"

namespace mas {

namespace {
constexpr int AJ = 8, AK = 64;           // cell tile: theta rows x phi cells
constexpr int PR = AJ + 2;               // p tile rows with a 1-cell halo
constexpr int CR = AJ + 1;               // corner rows of the tile
constexpr int TKT_ANISO = 3;
}  // namespace

// ---------------------------------------------------------------------------
// setup: corner coefficients (R21-R25)
// ---------------------------------------------------------------------------
__global__ void __launch_bounds__(kThreads) k_aniso_coef(const Geo g, const AnisoTab t,
                                                         const double* kpar, const double* bhat,
                                                         double* ca, int* bad) {
    const long long N = (long long)g.nl * g.plane;
    for (long long P = blockIdx.x * (long long)kThreads + threadIdx.x; P < N;
         P += (long long)gridDim.x * kThreads) {
        const int i = (int)(P / g.plane);
        const long long off = P - (long long)i * g.plane;
        const int j = (int)(off / g.np), k = (int)(off - (long long)j * g.np);
        double a = 0.0, b = 0.0, e = 0.0;
        const double hr = t.hr[i], ht = t.ht[j];
        if (hr > 0.0 && ht > 0.0) {  // a live corner (R24): not on an r boundary, pole or wall
            const double kp = kpar[P], br = bhat[P], bt = bhat[N + P], bp = bhat[2 * N + P];
            const bool ok = kp >= 0.0 && isfinite(kp) && isfinite(br) && isfinite(bt) && isfinite(bp);
            if (!ok) atomicOr(bad, 1);
            const double rF = t.rF[i], sF = t.sF[j], hp = t.hp[k];
            const double beta = sqrt(rF * rF * sF * hr * ht * hp * kp);  // sqrt(W_c kpar_c), R23
            a = beta * br / (4.0 * hr);
            b = beta * bt / (4.0 * rF * ht);
            e = beta * bp / (4.0 * rF * sF * hp);
        }
        ca[P] = a;
        ca[N + P] = b;
        ca[2 * N + P] = e;
    }
}

// corner coefficient f (0 a, 1 b, 2 e) of corner (I, J, K); 0 beyond the array
// (J = nt: the south pole / wall; I = nl: the global outer r-face, or on an
// r-slab rank+1's plane 0, taken from the ghost copy ca_hi)
__device__ __forceinline__ double corner_coef(const Geo& g, const double* ca, const double* ca_hi,
                                              int f, int I, int J, int K) {
    if (J >= g.nt) return 0.0;
    if (K >= g.np) K -= g.np;
    if (I >= g.nl) return ca_hi ? __ldg(ca_hi + f * g.plane + (long long)J * g.np + K) : 0.0;
    const long long N = (long long)g.nl * g.plane;
    return __ldg(ca + f * N + ((long long)I * g.nt + J) * g.np + K);
}

// D += (1/V) sum over the 8 corners of (sr a + st b + sp e)^2  (R26)
__global__ void __launch_bounds__(kThreads) k_aniso_diag(const Geo g, const double* ca,
                                                         const double* ca_hi, double* D, double* dinv,
                                                         int* bad) {
    const long long N = (long long)g.nl * g.plane;
    for (long long P = blockIdx.x * (long long)kThreads + threadIdx.x; P < N;
         P += (long long)gridDim.x * kThreads) {
        const int i = (int)(P / g.plane);
        const long long off = P - (long long)i * g.plane;
        const int j = (int)(off / g.np), k = (int)(off - (long long)j * g.np);
        double s = 0.0;
        for (int di = 0; di < 2; di++)
            for (int dj = 0; dj < 2; dj++)
                for (int dk = 0; dk < 2; dk++) {
                    const int I = i + di, J = j + dj, K = k + dk;
                    const double sr = di ? -1.0 : 1.0, st = dj ? -1.0 : 1.0, sp = dk ? -1.0 : 1.0;
                    const double d = sr * corner_coef(g, ca, ca_hi, 0, I, J, K) +
                                     st * corner_coef(g, ca, ca_hi, 1, I, J, K) +
                                     sp * corner_coef(g, ca, ca_hi, 2, I, J, K);
                    s += d * d;
                }
        const double V = g.vr[i] * g.vt[j] * g.vp[k];
        const double Dn = D[P] + s / V;
        D[P] = Dn;
        dinv[P] = 1.0 / Dn;
        if (!(Dn > 0.0) || !isfinite(Dn)) atomicOr(bad, 1);
    }
}

// ---------------------------------------------------------------------------
// the operator term
// ---------------------------------------------------------------------------
__device__ __forceinline__ double2 lds2(const double* p) { return *reinterpret_cast<const double2*>(p); }
__device__ __forceinline__ void sts2(double* p, double2 v) { *reinterpret_cast<double2*>(p) = v; }
__device__ __forceinline__ void stg2(double* p, double2 v) { *reinterpret_cast<double2*>(p) = v; }
__device__ __forceinline__ double2 ld2(const double* p) { return __ldg(reinterpret_cast<const double2*>(p)); }
// cp.async (LDGSTS) with zero-fill: src_bytes = 0 writes zeros and reads
// nothing (dead corners, rows beyond a pole, planes outside the slab)
__device__ __forceinline__ void cpa16(double* dst, const double* src, bool ok) {
    const unsigned sa = (unsigned)__cvta_generic_to_shared(dst);
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;\n" ::"r"(sa), "l"(src), "r"(ok ? 16 : 0)
                 : "memory");
}
__device__ __forceinline__ void cpa8(double* dst, const double* src, bool ok) {
    const unsigned sa = (unsigned)__cvta_generic_to_shared(dst);
    asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;\n" ::"r"(sa), "l"(src), "r"(ok ? 8 : 0)
                 : "memory");
}
// the same with a precomputed 32-bit shared-window address
__device__ __forceinline__ void cpa16s(unsigned sa, const double* src, bool ok) {
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;\n" ::"r"(sa), "l"(src), "r"(ok ? 16 : 0)
                 : "memory");
}
__device__ __forceinline__ void cpa8s(unsigned sa, const double* src, bool ok) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;\n" ::"r"(sa), "l"(src), "r"(ok ? 8 : 0)
                 : "memory");
}
__device__ __forceinline__ void cpa_commit_group() { asm volatile("cp.async.commit_group;\n" ::: "memory"); }
__device__ __forceinline__ void cpa_wait_1() { asm volatile("cp.async.wait_group 1;\n" ::: "memory"); }

namespace {
// Shared-memory rings.  A "stage" I is {p plane I, corner coefficients of
// corner plane I, out/q plane I-1}; p and the coefficients use 4 slots
// (slot = plane & 3), out uses 3 (slot = (plane + 3) % 3).
constexpr int PW = AK + 4;             // p row: [pad][k0-1][64 cells][k0+width][pad], 16 B aligned
constexpr int CW = AK + 2;             // corner row: corners k0 .. k0+64 (+ pad), 16 B aligned
constexpr int CA = CR * CW;            // one corner array of a slot
constexpr int P_SLOT = PR * PW;        // 680 doubles
constexpr int C_SLOT = 4 * CA;         // raw a, b, e -> the 4 sign combinations (see corners)
constexpr int Q_SLOT = AJ * AK;        // 512 doubles
constexpr int SMEM_DOUBLES = 4 * P_SLOT + 4 * C_SLOT + 3 * Q_SLOT;
// per-thread work lists (plane independent, computed once per block)
constexpr int NP_IT = (PR * (AK / 2 + 2) + kThreads - 1) / kThreads;  // p copies
constexpr int NC_IT = (CR * (AK / 2 + 1) + kThreads - 1) / kThreads;  // coefficient copies per field
constexpr int NQ_IT = (AJ * AK / 2 + kThreads - 1) / kThreads;         // out copies
}  // namespace
constexpr int kAnisoSmem = SMEM_DOUBLES * (int)sizeof(double);  // 110,336 B: 2 blocks per SM

#ifndef MAS_ANISO_MINB
#define MAS_ANISO_MINB 2
#endif
// Per step I (corner plane I, cells of plane I-1):
//   wait for stage I -> barrier A -> issue stage I+2 -> corners(I) ->
//   barrier B -> cells(I-1)
// Stage I+2 is issued after barrier A of step I, when every thread is past
// step I-1, so the slots it overwrites are free.  The corner thread replaces
// the raw (a, b, e) of its corner by the 4 sign combinations
//   c[st,sp] = s a + st s b + sp s e   (st, sp = +-1)
// so that a cell reads one value per corner: corner plane i (sr = +1) gives
// c[st,sp] of its 4 corners, plane i+1 (sr = -1) gives -c[-st,-sp].
// sigma_par = <p, L_par p>_V = sum_c s_c^2 (V L_par = G^T W K G), summed in
// the corner phase.
template <int MODE>
__global__ void __launch_bounds__(kThreads, MAS_ANISO_MINB) k_aniso(const AnisoArgs a) {
    extern __shared__ __align__(16) double sm[];
    double* Ps = sm;
    double* Cs = Ps + 4 * P_SLOT;
    double* Qs = Cs + 4 * C_SLOT;
    if (MODE == MODE_PCGA && __ldcg(&a.st->stopped)) {
        if (a.cond && blockIdx.x == 0 && threadIdx.x == 0)
            cudaGraphSetConditional((cudaGraphConditionalHandle)a.cond, 0);
        return;
    }
    const Geo& g = a.g;
    const int plane = (int)g.plane;
    const long long Nl = (long long)g.nl * plane;
    double acc[3] = {0.0, 0.0, 0.0};
    // Balanced partition: the (tile, r-plane) units, tile-major, are split
    // into gridDim.x equal ranges; a block's range covers one or two
    // segments (a run of planes of one tile), each marched with its own
    // pipeline (one resident wave of blocks, no tail).
    const long long units = (long long)a.ntj * a.ntk * g.nl;
    long long u0 = units * blockIdx.x / gridDim.x;
    const long long u1 = units * (blockIdx.x + 1) / gridDim.x;
    while (u0 < u1) {
        const int tile = (int)(u0 / g.nl);
        const int ia = (int)(u0 - (long long)tile * g.nl);
        const int ib = (int)min((long long)g.nl, ia + (u1 - u0));
        u0 += ib - ia;
        const int tk = tile % a.ntk, tj = tile / a.ntk;
        const int j0 = tj * AJ, k0 = tk * AK;
        const int height = min(AJ, g.nt - j0), width = min(AK, g.np - k0);  // width is even
        const int hw = width >> 1;  // 16-byte pairs per row

        // ---- per-thread work lists ---------------------------------------------
        // copies: byte offset within the slot (-1: none), in-plane source
        // offset (elements), 16 B (1) or 8 B (0), row valid (rows beyond a
        // pole / the tile: zero-fill).  The coefficient items are the same for
        // the 3 fields (a, b, e) up to the field's array offset.
        const unsigned sP = (unsigned)__cvta_generic_to_shared(Ps);
        const unsigned sC = (unsigned)__cvta_generic_to_shared(Cs);
        const unsigned sQ = (unsigned)__cvta_generic_to_shared(Qs);
        int pd[NP_IT], ps[NP_IT];
        unsigned pflag = 0;  // bit 2s: 16 B, bit 2s+1: row valid
        for (int s = 0; s < NP_IT; s++) {
            const int t = threadIdx.x + s * kThreads;
            pd[s] = -1;
            ps[s] = 0;
            if (t < PR * (hw + 2)) {
                const int r = t / (hw + 2), c = t - r * (hw + 2);
                const int j = j0 - 1 + r;
                const bool ok = j >= 0 && j < g.nt && r <= height + 1;
                if (c < hw) {
                    pd[s] = 8 * (r * PW + 2 + 2 * c);
                    ps[s] = (ok ? j : 0) * g.np + k0 + 2 * c;
                    pflag |= 1u << (2 * s);
                } else {
                    const int side = c - hw;  // 0: k0-1, 1: k0+width (periodic)
                    int k = side ? k0 + width : k0 - 1;
                    k = k < 0 ? k + g.np : (k >= g.np ? k - g.np : k);
                    pd[s] = 8 * (r * PW + (side ? 2 + width : 1));
                    ps[s] = (ok ? j : 0) * g.np + k;
                }
                if (ok) pflag |= 2u << (2 * s);
            }
        }
        int cd[NC_IT], cs[NC_IT];
        unsigned cflag = 0;  // bits as pflag
        for (int s = 0; s < NC_IT; s++) {
            const int t = threadIdx.x + s * kThreads;
            cd[s] = -1;
            cs[s] = 0;
            const int crow = hw + 1;
            if (t < CR * crow) {
                const int r = t / crow, c = t - r * crow;
                const int J = j0 + r;
                const bool ok = r <= height && J < g.nt;
                if (c < hw) {
                    cd[s] = 8 * (r * CW + 2 * c);
                    cs[s] = (ok ? J : 0) * g.np + k0 + 2 * c;
                    cflag |= 1u << (2 * s);
                } else {
                    int K = k0 + width;
                    if (K >= g.np) K -= g.np;
                    cd[s] = 8 * (r * CW + width);
                    cs[s] = (ok ? J : 0) * g.np + K;
                }
                if (ok) cflag |= 2u << (2 * s);
            }
        }
        int qd[NQ_IT], qs[NQ_IT];
        for (int s = 0; s < NQ_IT; s++) {
            const int t = threadIdx.x + s * kThreads;
            qd[s] = -1;
            qs[s] = 0;
            if (t < height * hw) {
                const int r = t / hw, c = t - r * hw;
                qd[s] = 8 * (r * AK + 2 * c);
                qs[s] = (j0 + r) * g.np + k0 + 2 * c;
            }
        }
        // compute mapping: warp w = tile row, lane l = the column pair 2l, 2l+1
        // (cells (w, 2l..2l+1) and corners (w, 2l..2l+1)); the corners of row
        // 8 and column 64 (the next tiles' first row / column) are an extra
        // item of threads 0..72
        const int w = threadIdx.x >> 5, c2 = 2 * (threadIdx.x & 31);
        const bool crow_ok = w <= height && c2 <= width;  // corner pair in use
        const bool cell_ok = w < height && c2 < width;    // cell pair in use (width even)
        int xr = -1, xc = 0;  // extra corner of this thread
        {
            const int t = threadIdx.x;
            if (height == AJ && t <= width) {
                xr = AJ, xc = t;
            } else if (width == AK && t >= AK + 1 && t - (AK + 1) < min(height + 1, AJ)) {
                xr = t - (AK + 1), xc = AK;
            }
        }
        double cw0 = 0.0, cw1 = 0.0;  // 1 / (vt_j vp_k) of the two cells
        if (cell_ok) {
            const double vt = __ldg(g.vt + j0 + w);
            cw0 = 1.0 / (vt * __ldg(g.vp + k0 + c2));
            cw1 = 1.0 / (vt * __ldg(g.vp + k0 + c2 + 1));
        }

        // ---- stages ------------------------------------------------------------
        auto issue = [&](int I) {
            if (I <= ib) {
                const unsigned P = sP + (unsigned)((I & 3) * P_SLOT * 8);
                // p plane I: own planes, or the r-slab ghost planes -1 / nl
                const double* pb = I >= 0 && I < g.nl ? a.u.in + (size_t)I * plane
                                   : I < 0            ? a.u.glo
                                                      : a.u.ghi;
                const bool pl = pb != nullptr;
                if (!pl) pb = a.u.in;
    #pragma unroll
                for (int s = 0; s < NP_IT; s++) {
                    if (pd[s] < 0) continue;
                    const bool ok = pl && ((pflag >> (2 * s + 1)) & 1u);
                    if ((pflag >> (2 * s)) & 1u)
                        cpa16s(P + pd[s], pb + ps[s], ok);
                    else
                        cpa8s(P + pd[s], pb + ps[s], ok);
                }
                const unsigned Cf = sC + (unsigned)((I & 3) * C_SLOT * 8);
                // corner plane I (plane ia-1, p only, may be -1); plane nl: the
                // ghost copy of rank+1's plane 0, else the dead outer face
                const bool cin = I >= 0 && I < g.nl;
                const bool cl = cin || (I == g.nl && a.ca_hi != nullptr);
    #pragma unroll
                for (int f = 0; f < 3; f++) {
                    const double* cb = cin ? a.ca + f * Nl + (size_t)I * plane
                                           : (cl ? a.ca_hi + (size_t)f * plane : a.ca);
                    const unsigned Cff = Cf + (unsigned)(f * CA * 8);
    #pragma unroll
                    for (int s = 0; s < NC_IT; s++) {
                        if (cd[s] < 0) continue;
                        const bool ok = cl && ((cflag >> (2 * s + 1)) & 1u);
                        if ((cflag >> (2 * s)) & 1u)
                            cpa16s(Cff + cd[s], cb + cs[s], ok);
                        else
                            cpa8s(Cff + cd[s], cb + cs[s], ok);
                    }
                }
            }
            const int iq = I - 1;  // out plane I-1: its cells are computed at step I
            if (iq >= ia && iq < ib) {
                const unsigned Q = sQ + (unsigned)(((iq + 3) % 3) * Q_SLOT * 8);
                const double* qb = a.out + (size_t)iq * plane;
    #pragma unroll
                for (int s = 0; s < NQ_IT; s++)
                    if (qd[s] >= 0) cpa16s(Q + qd[s], qb + qs[s], true);
            }
            cpa_commit_group();
        };

        // corner products of corner plane I: corner (J, K) = (j0 + r, k0 + c)
        // sits between cell rows J-1, J (p rows r, r+1) and cols K-1, K
        // (p cols c+1, c+2).  Each corner's raw (a, b, e) are replaced by the
        // 4 sign combinations c[st,sp] = s a + st s b + sp s e.
        auto corner_math = [&](double a00, double a01, double a10, double a11, double b00, double b01,
                               double b10, double b11, double A0, double B0, double E0, double& o0,
                               double& o1, double& o2, double& o3) -> double {
            const double Dr = ((b00 - a00) + (b01 - a01)) + ((b10 - a10) + (b11 - a11));
            const double Dt = ((a10 - a00) + (a11 - a01)) + ((b10 - b00) + (b11 - b01));
            const double Dp = ((a01 - a00) + (a11 - a10)) + ((b01 - b00) + (b11 - b10));
            const double sc = A0 * Dr + B0 * Dt + E0 * Dp;
            const double A = sc * A0, B = sc * B0, E = sc * E0;
            o0 = (A + B) + E;  // st +, sp +
            o1 = (A + B) - E;  // st +, sp -
            o2 = (A - B) + E;  // st -, sp +
            o3 = (A - B) - E;  // st -, sp -
            return sc;
        };
        auto corners = [&](int I) {
            const double* p0 = Ps + ((I - 1) & 3) * P_SLOT;
            const double* p1 = Ps + (I & 3) * P_SLOT;
            double* Cf = Cs + (I & 3) * C_SLOT;
            const bool own_plane = MODE == MODE_PCGA && I < ib;  // plane ib: the next segment's
            if (crow_ok) {
                // p cols c2+1 (scalar), c2+2..c2+3 (aligned pair), rows w, w+1
                const double* q0 = p0 + w * PW + c2;
                const double* q1 = p1 + w * PW + c2;
                const double x0 = q0[1], y0 = q0[PW + 1], X0 = q1[1], Y0 = q1[PW + 1];
                const double2 x12 = lds2(q0 + 2), y12 = lds2(q0 + PW + 2);
                const double2 X12 = lds2(q1 + 2), Y12 = lds2(q1 + PW + 2);
                double* c0 = Cf + w * CW + c2;
                const double2 A0 = lds2(c0), B0 = lds2(c0 + CA), E0 = lds2(c0 + 2 * CA);
                double o[2][4];
                const double s0 = corner_math(x0, x12.x, y0, y12.x, X0, X12.x, Y0, Y12.x, A0.x, B0.x, E0.x,
                                              o[0][0], o[0][1], o[0][2], o[0][3]);
                const double s1 = corner_math(x12.x, x12.y, y12.x, y12.y, X12.x, X12.y, Y12.x, Y12.y, A0.y,
                                              B0.y, E0.y, o[1][0], o[1][1], o[1][2], o[1][3]);
#pragma unroll
                for (int q = 0; q < 4; q++) sts2(c0 + q * CA, make_double2(o[0][q], o[1][q]));
                // sigma: corners of this tile (row < height, col < width) only
                if (own_plane && w < height && c2 < width) acc[0] += s0 * s0 + s1 * s1;
            }
            if (xr >= 0) {  // row 8 / column 64: counted by the neighbouring tile
                const double* q0 = p0 + xr * PW + xc + 1;
                const double* q1 = p1 + xr * PW + xc + 1;
                double* c0 = Cf + xr * CW + xc;
                double o0, o1, o2, o3;
                corner_math(q0[0], q0[1], q0[PW], q0[PW + 1], q1[0], q1[1], q1[PW], q1[PW + 1], c0[0],
                            c0[CA], c0[2 * CA], o0, o1, o2, o3);
                c0[0] = o0;
                c0[CA] = o1;
                c0[2 * CA] = o2;
                c0[3 * CA] = o3;
            }
        };

        // cells (w, c2), (w, c2+1) of plane i: corner planes i (sr = +1) and
        // i+1 (sr = -1); corner rows w (st = +1), w+1 (st = -1); corner cols
        // c (sp = +1), c+1 (sp = -1).  Plane i gives c[st,sp] of the 4 corners,
        // plane i+1 gives -c[-st,-sp].
        auto cells = [&](int i) {
            if (!cell_ok) return;
            const double* l = Cs + (i & 3) * C_SLOT + w * CW + c2;
            const double* h = Cs + ((i + 1) & 3) * C_SLOT + w * CW + c2;
            const double2 l0 = lds2(l), l2 = lds2(l + 2 * CA + CW);
            const double2 h3 = lds2(h + 3 * CA), h1 = lds2(h + CA + CW);
            const double l1a = l[CA + 1], l1b = l[CA + 2];
            const double l3a = l[3 * CA + CW + 1], l3b = l[3 * CA + CW + 2];
            const double h2a = h[2 * CA + 1], h2b = h[2 * CA + 2];
            const double h0a = h[CW + 1], h0b = h[CW + 2];
            const double s0 = ((l0.x + l1a) + (l2.x + l3a)) - ((h3.x + h2a) + (h1.x + h0a));
            const double s1 = ((l0.y + l1b) + (l2.y + l3b)) - ((h3.y + h2b) + (h1.y + h0b));
            const double ivr = __ldg(a.ivr + i);
            const double y0 = s0 * (ivr * cw0), y1 = s1 * (ivr * cw1);
            const double2 qv = lds2(Qs + ((i + 3) % 3) * Q_SLOT + w * AK + c2);
            double* o = a.out + (size_t)i * plane + (j0 + w) * g.np + k0 + c2;
            if (MODE == MODE_RESID) {
                const double r0 = qv.x - y0, r1 = qv.y - y1;
                stg2(o, make_double2(r0, r1));
                const double vr = __ldg(g.vr + i);
                const double V0 = vr / cw0, V1 = vr / cw1;
                const double2 f = ld2(a.f + (o - a.out));
                const double2 di = ld2(a.dinv + (o - a.out));
                acc[0] += V0 * f.x * f.x + V1 * f.y * f.y;
                acc[1] += V0 * r0 * r0 + V1 * r1 * r1;
                acc[2] += V0 * r0 * (di.x * r0) + V1 * r1 * (di.y * r1);
            } else {
                stg2(o, make_double2(qv.x + y0, qv.y + y1));
            }
        };

        issue(ia - 1);  // p plane ia-1 (zeros below the slab)
        issue(ia);
        issue(ia + 1);
        for (int I = ia; I <= ib; I++) {
            cpa_wait_1();  // this thread's copies of stages <= I are done (I+1 may be in flight)
            __syncthreads();
            issue(I + 2);
            corners(I);
            __syncthreads();
            if (I > ia) cells(I - 1);
        }
        __syncthreads();  // the next segment refills the rings
    }

    if (MODE == MODE_PCGA) {
        double v[1] = {acc[0]};
        if (grid_reduce<1>(v, a.scr, TKT_ANISO) && threadIdx.x == 0)
            a.st->pend_sigma = a.st->pend_sigma + v[0];  // <p,L_iso p> (kernel A) + <p,L_par p>
    } else if (MODE == MODE_RESID) {
        if (grid_reduce<3>(acc, a.scr, TKT_ANISO) && threadIdx.x == 0) {
            a.st->pend_ff = acc[0];
            a.st->pend_rr = acc[1];
            a.st->pend_rho = acc[2];
        }
    }
}

// ---------------------------------------------------------------------------
// launchers
// ---------------------------------------------------------------------------
// one resident wave: MAS_ANISO_MINB blocks per SM, each with an equal share of
// the (tile, r-plane) units (bounded by the reduction scratch)
cudaError_t launch_aniso(int mode, const AnisoArgs& a0, cudaStream_t s) {
    AnisoArgs a = a0;
    a.ntj = (a.g.nt + AJ - 1) / AJ;
    a.ntk = (a.g.np + AK - 1) / AK;
    const int tiles = a.ntj * a.ntk;
    static int sms = 0;
    if (!sms) {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        if (sms <= 0) sms = 148;
    }
    long long want = (long long)MAS_ANISO_MINB * sms;
    if (const char* e = getenv("MAS_ABLOCKS")) want = std::max(1, atoi(e));  // experiment hook
    want = std::min<long long>(want, (long long)tiles * a.g.nl);
    want = std::min<long long>(want, a.max_blocks);
    a.chunk = 0;
    a.nchunk = 0;
    const int blocks = (int)want;
    if (blocks <= 0) return cudaErrorInvalidValue;
    static bool attr = false;
    if (!attr) {
        cudaFuncSetAttribute(k_aniso<MODE_APPLY>, cudaFuncAttributeMaxDynamicSharedMemorySize, kAnisoSmem);
        cudaFuncSetAttribute(k_aniso<MODE_RESID>, cudaFuncAttributeMaxDynamicSharedMemorySize, kAnisoSmem);
        cudaFuncSetAttribute(k_aniso<MODE_PCGA>, cudaFuncAttributeMaxDynamicSharedMemorySize, kAnisoSmem);
        attr = true;
    }
    if (mode == MODE_APPLY)
        k_aniso<MODE_APPLY><<<blocks, kThreads, kAnisoSmem, s>>>(a);
    else if (mode == MODE_RESID)
        k_aniso<MODE_RESID><<<blocks, kThreads, kAnisoSmem, s>>>(a);
    else
        k_aniso<MODE_PCGA><<<blocks, kThreads, kAnisoSmem, s>>>(a);
    return cudaGetLastError();
}

cudaError_t launch_aniso_coef(const Geo& g, AnisoTab t, const double* kpar, const double* bhat,
                              double* ca, int* bad, cudaStream_t s) {
    const long long N = (long long)g.nl * g.plane;
    const int blocks = (int)std::min<long long>((N + kThreads - 1) / kThreads, 148LL * 16);
    k_aniso_coef<<<blocks, kThreads, 0, s>>>(g, t, kpar, bhat, ca, bad);
    return cudaGetLastError();
}

cudaError_t launch_aniso_diag(const Geo& g, const double* ca, const double* ca_hi, double* D,
                              double* dinv, int* bad, cudaStream_t s) {
    const long long N = (long long)g.nl * g.plane;
    const int blocks = (int)std::min<long long>((N + kThreads - 1) / kThreads, 148LL * 16);
    k_aniso_diag<<<blocks, kThreads, 0, s>>>(g, ca, ca_hi, D, dinv, bad);
    return cudaGetLastError();
}

}  // namespace mas
