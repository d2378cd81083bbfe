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
// (I = nl: the global outer r-face; J = nt: the south pole / wall)
__device__ __forceinline__ double corner_coef(const Geo& g, const double* ca, int f, int I, int J,
                                              int K) {
    if (I >= g.nl || J >= g.nt) return 0.0;
    if (K >= g.np) K -= g.np;
    const long long N = (long long)g.nl * g.plane;
    return __ldg(ca + f * N + ((long long)I * g.nt + J) * g.np + K);
}

// D += (1/V) sum over the 8 corners of (sr a + st b + sp e)^2  (R26)
__global__ void __launch_bounds__(kThreads) k_aniso_diag(const Geo g, const double* ca, double* D,
                                                         double* dinv, int* bad) {
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
                    const double d = sr * corner_coef(g, ca, 0, I, J, K) +
                                     st * corner_coef(g, ca, 1, I, J, K) +
                                     sp * corner_coef(g, ca, 2, I, J, K);
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
constexpr int NK_IT = (CR * (AK + 1) + kThreads - 1) / kThreads;       // corners
constexpr int NL_IT = (AJ * AK + kThreads - 1) / kThreads;             // cells
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
        // corners (smem offsets into the coefficient / p slots) and cells
        int kc[NK_IT], kp[NK_IT];
        unsigned kown = 0;  // bit s: the corner belongs to this tile (row < height, col < width):
                            // the last row / col is the next tile's first (sigma counts each once)
        for (int s = 0; s < NK_IT; s++) {
            const int t = threadIdx.x + s * kThreads;
            kc[s] = -1;
            kp[s] = 0;
            if (t < (height + 1) * (width + 1)) {
                const int r = t / (width + 1), c = t - r * (width + 1);
                kc[s] = r * CW + c;
                kp[s] = r * PW + c + 1;
                if (r < height && c < width) kown |= 1u << s;
            }
        }
        int lc[NL_IT], lq[NL_IT], lo_[NL_IT];
        double lw[NL_IT];  // 1 / (vt_j vp_k)
        for (int s = 0; s < NL_IT; s++) {
            const int t = threadIdx.x + s * kThreads;
            lc[s] = -1;
            lq[s] = 0;
            lo_[s] = 0;
            lw[s] = 0.0;
            if (t < height * width) {
                const int r = t / width, c = t - r * width;
                lc[s] = r * CW + c;
                lq[s] = r * AK + c;
                lo_[s] = (j0 + r) * g.np + k0 + c;
                lw[s] = 1.0 / (__ldg(g.vt + j0 + r) * __ldg(g.vp + k0 + c));
            }
        }

        // ---- stages ------------------------------------------------------------
        auto issue = [&](int I) {
            if (I <= ib) {
                const unsigned P = sP + (unsigned)((I & 3) * P_SLOT * 8);
                const bool pl = I >= 0 && I < g.nl;
                const double* pb = a.u + (size_t)(pl ? I : 0) * plane;
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
                const bool cl = I >= 0 && I < g.nl;  // plane ia-1 (p only) may be -1
    #pragma unroll
                for (int f = 0; f < 3; f++) {
                    const double* cb = a.ca + f * Nl + (size_t)(cl ? I : 0) * plane;
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
        // (p cols c+1, c+2)
        auto corners = [&](int I) {
            const double* p0 = Ps + ((I - 1) & 3) * P_SLOT;
            const double* p1 = Ps + (I & 3) * P_SLOT;
            double* Cf = Cs + (I & 3) * C_SLOT;
    #pragma unroll
            for (int s = 0; s < NK_IT; s++) {
                if (kc[s] < 0) continue;
                double* c0 = Cf + kc[s];
                const double A0 = c0[0], B0 = c0[CA], E0 = c0[2 * CA];
                const double* q0 = p0 + kp[s];
                const double* q1 = p1 + kp[s];
                const double a00 = q0[0], a01 = q0[1], a10 = q0[PW], a11 = q0[PW + 1];
                const double b00 = q1[0], b01 = q1[1], b10 = q1[PW], b11 = q1[PW + 1];
                const double Dr = ((b00 - a00) + (b01 - a01)) + ((b10 - a10) + (b11 - a11));
                const double Dt = ((a10 - a00) + (a11 - a01)) + ((b10 - b00) + (b11 - b01));
                const double Dp = ((a01 - a00) + (a11 - a10)) + ((b01 - b00) + (b11 - b10));
                const double sc = A0 * Dr + B0 * Dt + E0 * Dp;
                const double A = sc * A0, B = sc * B0, E = sc * E0;
                c0[0] = (A + B) + E;       // st +, sp +
                c0[CA] = (A + B) - E;      // st +, sp -
                c0[2 * CA] = (A - B) + E;  // st -, sp +
                c0[3 * CA] = (A - B) - E;  // st -, sp -
                // corner plane ib is the next chunk's first (or the dead outer face)
                if (MODE == MODE_PCGA && I < ib && ((kown >> s) & 1u)) acc[0] += sc * sc;
            }
        };

        // cells of plane i: corner planes i (sr = +1) and i+1 (sr = -1); corner
        // rows r (st = +1), r+1 (st = -1); corner cols c (sp = +1), c+1 (sp = -1)
        auto cells = [&](int i) {
            const double* lo = Cs + (i & 3) * C_SLOT;
            const double* hi = Cs + ((i + 1) & 3) * C_SLOT;
            const double* Q = Qs + ((i + 3) % 3) * Q_SLOT;
            const double ivr = __ldg(a.ivr + i);
            double* ob = a.out + (size_t)i * plane;
    #pragma unroll
            for (int s = 0; s < NL_IT; s++) {
                if (lc[s] < 0) continue;
                const double* l = lo + lc[s];
                const double* h = hi + lc[s];
                const double sl = (l[0] + l[CA + 1]) + (l[2 * CA + CW] + l[3 * CA + CW + 1]);
                const double sh = (h[3 * CA] + h[2 * CA + 1]) + (h[CA + CW] + h[CW + 1]);
                const double y = (sl - sh) * (ivr * lw[s]);
                const double qv = Q[lq[s]];
                if (MODE == MODE_RESID) {
                    const double rv = qv - y;
                    ob[lo_[s]] = rv;
                    const double V = __ldg(g.vr + i) / lw[s];
                    const double f = a.f[(size_t)i * plane + lo_[s]];
                    acc[0] += V * f * f;
                    acc[1] += V * rv * rv;
                    acc[2] += V * rv * (a.dinv[(size_t)i * plane + lo_[s]] * rv);
                } else {
                    ob[lo_[s]] = qv + y;
                }
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

cudaError_t launch_aniso_diag(const Geo& g, const double* ca, double* D, double* dinv, int* bad,
                              cudaStream_t s) {
    const long long N = (long long)g.nl * g.plane;
    const int blocks = (int)std::min<long long>((N + kThreads - 1) / kThreads, 148LL * 16);
    k_aniso_diag<<<blocks, kThreads, 0, s>>>(g, ca, D, dinv, bad);
    return cudaGetLastError();
}

}  // namespace mas
