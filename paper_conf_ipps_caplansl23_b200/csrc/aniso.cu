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
// kernel A and kernel B are unchanged.  One block per SM, warp-specialised:
// a producer warp streams stages {p plane I with its phi halo, the 3
// corner-coefficient fields of corner plane I, out plane I-1} into a 4-slot
// shared ring with tensor copies (TMA, cuTensorMapEncodeTiled maps, one box
// per field; rows beyond a pole and planes outside the slab arrive as zeros;
// the periodic phi-wrap cells come as 2-wide side boxes); 16 consumer warps
// (one per tile row) compute the corner products and gather them into the
// cells.  Full / empty mbarriers order the two sides.  Bytes per cell (PCGA):
// p 8 + (a, b, e) 24 + q read/write 16 = 48 B.
#include <cuda.h>
#include <cuda_runtime.h>
#include <cudaTypedefs.h>

#include <algorithm>
#include <cmath>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <vector>

#include "mas_internal.h"
#include "reduce.cuh"

namespace mas {

namespace {
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

// D += (1/V) sum over the 8 corners of (sr a + st b + sp e)^2  (R26).  One
// thread per (theta, phi) column marches a chunk of r-planes: the 12 corner
// values (3 fields x 4 corners) of corner plane i+1 become those of plane i
// for the next cell, so a cell loads 12 instead of 24 (same sums, same order).
#ifndef MAS_DIAG_CHUNK
#define MAS_DIAG_CHUNK 8  // sweep at C2a: 4 / 8 / 16 / 32 planes = 81.9 / 77.6 / 85.3 / 107.4 us
#endif
constexpr int kDiagChunk = MAS_DIAG_CHUNK;
__global__ void __launch_bounds__(kThreads) k_aniso_diag(const Geo g, const double* ca, const double* ca_hi,
                                                         double* D, double* dinv, int* bad) {
    const long long cols = g.plane;
    const int nch = (g.nl + kDiagChunk - 1) / kDiagChunk;
    for (long long t = blockIdx.x * (long long)kThreads + threadIdx.x; t < cols * nch;
         t += (long long)gridDim.x * kThreads) {
        const int ch = (int)(t / cols);
        const long long off = t - (long long)ch * cols;
        const int j = (int)(off / g.np), k = (int)(off - (long long)j * g.np);
        const int i0 = ch * kDiagChunk, i1 = min(g.nl, i0 + kDiagChunk);
        // c[di][f][dj][dk]: corner (i + di, j + dj, k + dk), field f
        double c[2][3][2][2];
        auto load_plane = [&](int di, int I) {
#pragma unroll
            for (int f = 0; f < 3; f++)
#pragma unroll
                for (int dj = 0; dj < 2; dj++)
#pragma unroll
                    for (int dk = 0; dk < 2; dk++) c[di][f][dj][dk] = corner_coef(g, ca, ca_hi, f, I, j + dj, k + dk);
        };
        load_plane(0, i0);
        const double vtj = g.vt[j], vpk = g.vp[k];
        for (int i = i0; i < i1; i++) {
            load_plane(1, i + 1);
            double s = 0.0;
            for (int di = 0; di < 2; di++)
                for (int dj = 0; dj < 2; dj++)
                    for (int dk = 0; dk < 2; dk++) {
                        const double sr = di ? -1.0 : 1.0, st = dj ? -1.0 : 1.0, sp = dk ? -1.0 : 1.0;
                        const double d = sr * c[di][0][dj][dk] + st * c[di][1][dj][dk] + sp * c[di][2][dj][dk];
                        s += d * d;
                    }
            const long long P = (long long)i * g.plane + off;
            const double V = g.vr[i] * vtj * vpk;  // the same product order as before
            const double Dn = D[P] + s / V;
            D[P] = Dn;
            dinv[P] = 1.0 / Dn;
            if (!(Dn > 0.0) || !isfinite(Dn)) atomicOr(bad, 1);
#pragma unroll
            for (int f = 0; f < 3; f++)
#pragma unroll
                for (int dj = 0; dj < 2; dj++)
#pragma unroll
                    for (int dk = 0; dk < 2; dk++) c[0][f][dj][dk] = c[1][f][dj][dk];
        }
    }
}

// ---------------------------------------------------------------------------
// the operator term
// ---------------------------------------------------------------------------
__device__ __forceinline__ double2 lds2(const double* p) { return *reinterpret_cast<const double2*>(p); }
__device__ __forceinline__ void sts2(double* p, double2 v) { *reinterpret_cast<double2*>(p) = v; }
__device__ __forceinline__ void stg2(double* p, double2 v) { *reinterpret_cast<double2*>(p) = v; }
__device__ __forceinline__ double2 ld2(const double* p) { return __ldg(reinterpret_cast<const double2*>(p)); }

// ---- warp-specialised pipeline ---------------------------------------------
// One block per SM: 16 cell warps (warp w = tile row w, lane l = the column
// pair 2l, 2l+1), a halo warp (the corner row below the tile and the extra
// corner column) and one producer warp whose lane 0 streams the stages with
// tensor copies (cp.async.bulk.tensor, the TMA engine) into a 4-slot ring,
// signalled by mbarriers (full: the box bytes landed; empty: the 17 consumer
// warps are done with the slot).
namespace {
// out/q arrives as a TMA box per stage (MAS_ANISO_QREG: plain loads by the
// consumers, a tie; the other consumer designs tried are listed in
// profiles/README.md, "k_aniso A/B", and kept in the history up to c1ffbea)
#ifndef MAS_ANISO_WJ
#define MAS_ANISO_WJ 16
#endif
#ifndef MAS_ANISO_BPS
#define MAS_ANISO_BPS 1
#endif
constexpr int WJ = MAS_ANISO_WJ;       // tile rows (one consumer warp each)
constexpr int kAnisoBps = MAS_ANISO_BPS;  // resident blocks per SM (the rings must fit)
constexpr int rup16(int x) { return (x + 15) / 16 * 16; }  // 128-byte multiples of doubles
constexpr int WK = 64;                 // tile columns (32 lanes x 2)
constexpr int NCW = WJ;                // cell warps (warp w: cell row w and corner row w)
constexpr int NXW = NCW + 1;           // consumer warps: + the halo warp (corner row WJ, extra column)
constexpr int WTHREADS = 32 * (NXW + 1);
constexpr int WPR = WJ + 2;            // p rows: j0-1 .. j0+16
constexpr int WPW = WK + 4;            // p row: [k0-2][k0-1][64 cells][k0+64][k0+65]
constexpr int WCR = WJ + 1;            // corner rows
constexpr int WCW = WK + 2;            // corner row: K = k0 .. k0+64 (+1)
constexpr int WCA = WCR * WCW;         // one corner array
// every component of a slot starts 128-byte aligned (tensor-copy destinations)
constexpr int WP_SLOT = rup16(WPR * WPW);  // p box [WJ+2][68] + pad
constexpr int WC_SLOT = rup16(3 * WCA);    // coefficient box [3][WJ+1][66] + pad
#ifdef MAS_ANISO_QREG
constexpr int WQ_SLOT = 0;             // out/q loaded by the consumers (experiment hook)
#else
constexpr int WQ_SLOT = WJ * WK;       // out box [WJ][64]
#endif
constexpr int WPL = rup16(WPR * 2), WPRT = WPL;  // phi-wrap side boxes of p: [WJ+2][2]
constexpr int WCS = rup16(3 * WCR * 2);          // phi-wrap side box of the coefficients: [3][WJ+1][2]
constexpr int O_C = WP_SLOT, O_Q = O_C + WC_SLOT, O_PL = O_Q + WQ_SLOT, O_PR = O_PL + WPL,
              O_CS = O_PR + WPRT;
constexpr int W_SLOT = O_CS + WCS;     // WJ = 16: 5840 doubles
#ifndef MAS_ANISO_SLOTS
#define MAS_ANISO_SLOTS 4
#endif
constexpr int W_NSLOT = MAS_ANISO_SLOTS;  // ring depth (>= 2)
// corner-row exchange between the consumer warps (outside the ring, two
// parities): per corner row and cell column the K-combined A2 and Y (XA, XY),
// and the extra column's (A, B, E) per corner row (XC, padded to 4)
constexpr int XSZ = WCR * WK;          // one parity of XA / XY
constexpr int XCS = WCR * 4;           // one parity of XC
constexpr int O_XA = W_NSLOT * W_SLOT, O_XY = O_XA + 2 * XSZ, O_XC = O_XY + 2 * XSZ;
constexpr int W_SMEM_D = O_XC + 2 * XCS;
// tensor-copy transaction bytes (whole boxes, out-of-bounds elements included)
constexpr unsigned TX_P = WPR * WPW * 8, TX_PS = WPR * 2 * 8, TX_C = 3 * WCR * WCW * 8,
                   TX_CS = 3 * WCR * 2 * 8;
constexpr unsigned TX_Q = WJ * WK * 8;
}  // namespace
constexpr int kAnisoSmem = W_SMEM_D * (int)sizeof(double) + 3 * W_NSLOT * 8;  // 222,880 B

// Tensor maps of one launch (host-encoded, cuTensorMapEncodeTiled): boxes of
// the field u, of its r-slab ghost planes, of the corner coefficients (all 3
// fields in one box), of the corner plane above the slab, and of out.  The
// *_s maps are the 2-wide phi-wrap side boxes (TMA does not wrap).
struct __align__(64) AnisoMaps {
    CUtensorMap u, u_s, lo, lo_s, hi, hi_s, ca, ca_s, cahi, cahi_s, out;
    int has_lo, has_hi, has_cahi, pad;
};

__device__ __forceinline__ unsigned smem_u32(const void* p) { return (unsigned)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(unsigned bar, unsigned count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;\n" ::"r"(bar), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(unsigned bar, unsigned bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;\n" ::"r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(unsigned bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];\n" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void mbar_wait(unsigned bar, unsigned parity) {
    asm volatile(
        "{\n"
        ".reg .pred P1;\n"
        "WAIT_%=:\n"
        "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
        "@!P1 bra WAIT_%=;\n"
        "}\n" ::"r"(bar), "r"(parity) : "memory");
}
// tensor copies (TMA): one box of a tensor map into shared memory, completing
// the box bytes on the mbarrier; out-of-bounds box elements land as zeros
__device__ __forceinline__ void tma3(unsigned dst, const CUtensorMap* m, int c0, int c1, int c2, unsigned bar) {
    asm volatile(
        "cp.async.bulk.tensor.3d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], [%5];\n"
        ::"r"(dst), "l"(m), "r"(c0), "r"(c1), "r"(c2), "r"(bar) : "memory");
}
__device__ __forceinline__ void tma2(unsigned dst, const CUtensorMap* m, int c0, int c1, unsigned bar) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];\n"
        ::"r"(dst), "l"(m), "r"(c0), "r"(c1), "r"(bar) : "memory");
}
__device__ __forceinline__ void tma4(unsigned dst, const CUtensorMap* m, int c0, int c1, int c2, int c3,
                                     unsigned bar) {
    asm volatile(
        "cp.async.bulk.tensor.4d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5}], [%6];\n"
        ::"r"(dst), "l"(m), "r"(c0), "r"(c1), "r"(c2), "r"(c3), "r"(bar) : "memory");
}
__device__ __forceinline__ void fence_proxy_async() {
    asm volatile("fence.proxy.async.shared::cta;\n" ::: "memory");
}
__device__ __forceinline__ void consumer_sync() {  // the 17 consumer warps only
    asm volatile("bar.sync 1, %0;\n" ::"n"(32 * NXW) : "memory");
}

// Per step I (corner plane I, cells of plane I-1), consumer side:
//   wait full(stage I) -> corners(I) -> publish the corner row -> release
//   stage I -> consumer barrier -> cells(I-1).
// A stage I is {p plane I, corner coefficients of corner plane I, out/q plane
// I-1}.  With the corner fluxes (A, B, E) = s_c (a, b, e), a cell sums over
// its 8 corners sr A + st B + sp E (sr, st, sp = +1 where the corner is on
// the cell's low r / theta / phi side, -1 on the high side), so the sum
// separates by direction: the thread combines its corners along K with the
// right lane (shuffle), keeps its own row's B2 + Ed, and publishes A2 and
// Ed - B2 to the warp of the row above through a small two-parity shared
// array; along r the cell carries G+ of its lower corner plane in registers
// from the previous step.  sigma_par = <p, L_par p>_V = sum_c s_c^2
// (V L_par = G^T W K G), summed in the corner phase.
template <int MODE>
__global__ void __launch_bounds__(WTHREADS, kAnisoBps) k_aniso(const AnisoArgs a, const __grid_constant__ AnisoMaps M) {
    extern __shared__ __align__(128) double sm[];
    unsigned long long* bars = reinterpret_cast<unsigned long long*>(sm + W_SMEM_D);
    if (MODE == MODE_PCGA && __ldcg(&a.st->stopped)) {
        if (a.cond && blockIdx.x == 0 && threadIdx.x == 0)
            cudaGraphSetConditional((cudaGraphConditionalHandle)a.cond, 0);
        return;
    }
    const bool p2p = a.p2p.nranks > 0;
    int kit = 0;
    if (MODE == MODE_PCGA && p2p) {
        // P2P: the r-neighbours' p_k edge planes are read in place; wait until
        // every rank's kernel A(k) has published (its p_k is then complete)
        kit = __ldcg(&a.st->k);
        if (threadIdx.x == 0) {
            double v[1];
            p2p_gather_one<1>(a.p2p, MB_A, p2p_seq(__ldcg(&a.st->epoch), kit), v);
        }
        __syncthreads();
        // the neighbours' p_k was written through the generic proxy; the
        // producer reads it with tensor copies (async proxy): order the two
        // before the first cp.async.bulk.tensor of the lo / hi maps
        asm volatile("fence.proxy.async.global;\n" ::: "memory");
    }
    const Geo& g = a.g;
    const int plane = (int)g.plane;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const bool producer = warp == NXW;
    double acc[3] = {0.0, 0.0, 0.0};
    auto P_of = [&](int slot) { return sm + slot * W_SLOT; };
    auto C_of = [&](int slot) { return sm + slot * W_SLOT + O_C; };
    auto Q_of = [&](int slot) { return sm + slot * W_SLOT + O_Q; };
    const unsigned full0 = smem_u32(bars), empty0 = smem_u32(bars + W_NSLOT);

    int par = 0;  // parity of the consumers' corner-row exchange (toggled per barrier step)
    // balanced partition of the (tile, r-plane) units, tile-major (one or two
    // segments per block)
    const long long units = (long long)a.ntj * a.ntk * g.nl;
    long long u0 = units * blockIdx.x / gridDim.x;
    const long long u1 = units * (blockIdx.x + 1) / gridDim.x;
    while (u0 < u1) {
        const int tile = (int)(u0 / g.nl);
        const int ia = (int)(u0 - (long long)tile * g.nl);
        const int ib = (int)min((long long)g.nl, ia + (u1 - u0));
        u0 += ib - ia;
        const int tk = tile % a.ntk, tj = tile / a.ntk;
        const int j0 = tj * WJ, k0 = tk * WK;
        const int height = min(WJ, g.nt - j0), width = min(WK, g.np - k0);  // width is even

        // barriers (the rings need no clearing: every value a consumer reads is
        // written first in the same stage -- whole tensor boxes with zero-filled
        // out-of-bounds parts, side boxes on the tiles that read them)
        if (threadIdx.x == 0) {
            for (int q = 0; q < W_NSLOT; q++) {
                mbar_init(full0 + 8 * q, 1);    // expect_tx by the producer; the tensor bytes
                mbar_init(empty0 + 8 * q, NXW);
            }
        }
        fence_proxy_async();
        __syncthreads();
        // stages ia-1 .. ib; stage number n = I - (ia - 1), slot n % W_NSLOT, use n / W_NSLOT
        const int nst = ib - ia + 2;

        if (producer) {
            // one lane issues the stage's tensor copies: one box per field, plus
            // the 2-wide phi-wrap side boxes on the first / last phi tile (the
            // consumers read the wrap cells from those)
            const bool first = k0 == 0, last = k0 + width == g.np;
            auto p_src = [&](int I) -> int {  // 0 dead, 1 own, 2 lo ghost, 3 hi ghost
                return I >= 0 && I < g.nl ? 1 : (I < 0 ? (M.has_lo ? 2 : 0) : (M.has_hi ? 3 : 0));
            };
            auto c_src = [&](int n, int I) -> int {  // 0 none (stage ia-1), 1 own, 2 above, 3 dead
                return n == 0 ? 0 : (I >= 0 && I < g.nl ? 1 : (M.has_cahi ? 2 : 3));
            };
            auto issue = [&](int n) {
                const int I = ia - 1 + n, slot = n % W_NSLOT;
                if (n >= W_NSLOT) mbar_wait(empty0 + 8 * slot, ((n / W_NSLOT) - 1) & 1);
                const int ps = p_src(I), cs = c_src(n, I);
                const bool ql = I - 1 >= ia && I - 1 < ib;
                double* base = sm + slot * W_SLOT;
                __syncwarp();
                if (lane == 0) {
                    const unsigned full = full0 + 8 * slot;
                    unsigned bytes = 0;
                    // every stage carries a p box: a dead plane (beyond a global r
                    // boundary) is fetched from the own map at its out-of-range
                    // plane index, i.e. as zeros (the corners there have zero
                    // weight, but the ring slot must not hold stale or
                    // uninitialised values: 0 * NaN)
                    bytes += TX_P + (first ? TX_PS : 0u) + (last ? TX_PS : 0u);
                    if (cs) bytes += TX_C + (last ? TX_CS : 0u);
#ifndef MAS_ANISO_QREG
                    if (ql) bytes += TX_Q;
#endif
                    mbar_expect_tx(full, bytes);
                    const unsigned sb = smem_u32(base);
                    const int jr = j0 - 1;
                    if (ps <= 1) {  // own plane, or a dead one (out of range: zeros)
                        tma3(sb, &M.u, k0 - 2, jr, I, full);
                        if (first) tma3(sb + 8 * O_PL, &M.u_s, g.np - 2, jr, I, full);
                        if (last) tma3(sb + 8 * O_PR, &M.u_s, 0, jr, I, full);
                    } else if (ps >= 2) {
                        const CUtensorMap* m = ps == 2 ? &M.lo : &M.hi;
                        const CUtensorMap* m_s = ps == 2 ? &M.lo_s : &M.hi_s;
                        tma2(sb, m, k0 - 2, jr, full);
                        if (first) tma2(sb + 8 * O_PL, m_s, g.np - 2, jr, full);
                        if (last) tma2(sb + 8 * O_PR, m_s, 0, jr, full);
                    }
                    if (cs == 1 || cs == 3) {  // 3: the dead outer face, a box beyond the
                                                 // last plane (read as zeros)
                        const int Ic = cs == 1 ? I : g.nl;
                        tma4(sb + 8 * O_C, &M.ca, k0, j0, Ic, 0, full);
                        if (last) tma4(sb + 8 * O_CS, &M.ca_s, 0, j0, Ic, 0, full);
                    } else if (cs == 2) {
                        tma3(sb + 8 * O_C, &M.cahi, k0, j0, 0, full);
                        if (last) tma3(sb + 8 * O_CS, &M.cahi_s, 0, j0, 0, full);
                    }
#ifndef MAS_ANISO_QREG
                    if (ql) tma3(sb + 8 * O_Q, &M.out, k0, j0, I - 1, full);
#endif
                }
            };
            for (int n = 0; n < nst; n++) issue(n);
        } else {
            // ---- consumers: warp w < WJ owns corner row w and cell row w; the
            // halo warp (w = WJ) owns corner row WJ and the extra corner column
            // (K = k0 + width, one corner per lane = row) ----------------------
            const int w = warp, c2 = 2 * lane;
            const bool first = k0 == 0, last = k0 + width == g.np;
            const bool halo = w == NCW;
            const bool crow = w <= height && c2 < width;     // corner pair in use
            const bool cell_ok = w < height && c2 < width;   // cell pair in use
            const bool edge = c2 + 2 == width;               // right neighbour corner: the extra column
            const bool xlane = halo && lane <= height;       // extra-column corner (row lane, col width)
            double cw0 = 0.0, cw1 = 0.0;  // 1 / (vt_j vp_k) of the two cells
            if (cell_ok) {
                const double vt = __ldg(g.vt + j0 + w);
                cw0 = 1.0 / (vt * __ldg(g.vp + k0 + c2));
                cw1 = 1.0 / (vt * __ldg(g.vp + k0 + c2 + 1));
            }
            // s_c = a Dr + b Dt + e Dp of a corner from its 8 cells (a: plane
            // I-1, b: plane I; [row J-1 / J][column K-1 / K])
            auto corner_s = [&](double a00, double a01, double a10, double a11, double b00, double b01,
                                double b10, double b11, double A0, double B0, double E0) -> double {
                const double Dr = ((b00 - a00) + (b01 - a01)) + ((b10 - a10) + (b11 - a11));
                const double Dt = ((a10 - a00) + (a11 - a01)) + ((b10 - b00) + (b11 - b01));
                const double Dp = ((a01 - a00) + (a11 - a10)) + ((b01 - b00) + (b11 - b10));
                return A0 * Dr + B0 * Dt + E0 * Dp;
            };
            // p of the previous plane carried in registers: rows w, w+1 of the
            // box at columns c2+1 .. c2+3; the extra-column corner's 4 cells
            double x0 = 0.0, y0 = 0.0, e0 = 0.0, e1 = 0.0, e2 = 0.0, e3 = 0.0;
            double2 x12 = make_double2(0.0, 0.0), y12 = x12;
            // G+ of the previous corner plane (the cells' lower-r face), carried
            double2 carry = make_double2(0.0, 0.0);
            double ivr_cur = 0.0;  // 1/vr of the next step's cell plane, loaded one step ahead
            double* XA = sm + O_XA;
            double* XY = sm + O_XY;
            double* XC = sm + O_XC;
            for (int n = 0; n < nst; n++) {
                const int I = ia - 1 + n, slot = n % W_NSLOT;
                const double ivr_here = ivr_cur;
                if (cell_ok && n + 1 >= 2 && n + 1 < nst) ivr_cur = __ldg(a.ivr + I);
                // q / out of plane I-1 (the cells of this step)
                double2 qv = make_double2(0.0, 0.0);
#ifdef MAS_ANISO_QREG
                if (n >= 2 && cell_ok)
                    qv = ld2(a.out + (size_t)(I - 1) * plane + (size_t)(j0 + w) * g.np + k0 + c2);
#endif
                mbar_wait(full0 + 8 * slot, (n / W_NSLOT) & 1);
#ifdef MAS_ANISO_DIAG_NOCOMPUTE
                // diagnostic build (wrong results): the consumers only wait for
                // each stage and release it -- the producer / TMA pipeline alone
                __syncwarp();
                if (lane == 0) mbar_arrive(empty0 + 8 * slot);
                continue;
#endif
                const double* p1 = P_of(slot);
                // p rows w, w+1 (cell rows J-1, J) at cells k0+c2, k0+c2+1; the
                // cell k0+c2-1 from the left lane (lane 0: the box or the wrap box)
                const double* q1 = p1 + w * WPW + c2;
                const double2 X12 = lds2(q1 + 2), Y12 = lds2(q1 + WPW + 2);
                double X0 = __shfl_up_sync(0xffffffffu, X12.y, 1);
                double Y0 = __shfl_up_sync(0xffffffffu, Y12.y, 1);
                if (lane == 0) {
                    X0 = first ? p1[O_PL + 2 * w + 1] : q1[1];
                    Y0 = first ? p1[O_PL + 2 * w + 3] : q1[WPW + 1];
                }
                double E0 = 0.0, E1 = 0.0, E2 = 0.0, E3 = 0.0;
                if (xlane) {  // cells k0+width-1, k0+width (the latter wraps on the last tile)
                    const double* q2 = p1 + lane * WPW + width + 1;
                    E0 = q2[0], E2 = q2[WPW];
                    E1 = last ? p1[O_PR + 2 * lane] : q2[1];
                    E3 = last ? p1[O_PR + 2 * lane + 2] : q2[WPW + 1];
                }
                if (n == 0) {  // stage ia-1: p plane ia-1 only
                    x0 = X0, y0 = Y0, x12 = X12, y12 = Y12, e0 = E0, e1 = E1, e2 = E2, e3 = E3;
                    __syncwarp();
                    if (lane == 0) mbar_arrive(empty0 + 8 * slot);
                    continue;
                }
                // ---- corners (w, c2), (w, c2+1) of plane I ------------------
                const double* Cf = C_of(slot);
                const double* cc = Cf + w * WCW + c2;
                const double2 Ac = lds2(cc), Bc = lds2(cc + WCA), Ec = lds2(cc + 2 * WCA);
                const double s0 = corner_s(x0, x12.x, y0, y12.x, X0, X12.x, Y0, Y12.x, Ac.x, Bc.x, Ec.x);
                const double s1 = corner_s(x12.x, x12.y, y12.x, y12.y, X12.x, X12.y, Y12.x, Y12.y, Ac.y, Bc.y,
                                           Ec.y);
                // sigma: this tile's corners (row < height, col < width) of the
                // segment's own planes (plane ib is the next segment's first)
                if (MODE == MODE_PCGA && I < ib && cell_ok) acc[0] += s0 * s0 + s1 * s1;
                // the corner fluxes (A, B, E) = s_c (a, b, e); a cell sums, over
                // its 8 corners, sr A + st B + sp E (sr, st, sp = +1 on the
                // corner's low side): combine along K with the right lane
                const double Aa = s0 * Ac.x, Ab = s1 * Ac.y, Ba = s0 * Bc.x, Bb = s1 * Bc.y;
                const double Ea = s0 * Ec.x, Eb = s1 * Ec.y;
                double An = __shfl_down_sync(0xffffffffu, Aa, 1);
                double Bn = __shfl_down_sync(0xffffffffu, Ba, 1);
                double En = __shfl_down_sync(0xffffffffu, Ea, 1);
                if (edge) An = 0.0, Bn = 0.0, En = 0.0;  // the extra column, added after the barrier
                const double A2a = Aa + Ab, A2b = Ab + An;
                const double B2a = Ba + Bb, B2b = Bb + Bn;
                const double Eda = Ea - Eb, Edb = Eb - En;
                // corner row w gives its own cell row B2 + Ed (+-A2) and the cell
                // row above Ed - B2 (+-A2): the latter goes to warp w-1
                if (crow && w >= 1) {
                    sts2(XA + par * XSZ + w * WK + c2, make_double2(A2a, A2b));
                    sts2(XY + par * XSZ + w * WK + c2, make_double2(Eda - B2a, Edb - B2b));
                }
                if (xlane) {  // extra-column corner (lane, width)
                    double A, B, E;
                    if (last) {
                        const double* CS = p1 + O_CS;
                        A = CS[2 * lane], B = CS[2 * (WCR + lane)], E = CS[2 * (2 * WCR + lane)];
                    } else {
                        const double* c0 = Cf + lane * WCW + width;
                        A = c0[0], B = c0[WCA], E = c0[2 * WCA];
                    }
                    const double sx = corner_s(e0, e1, e2, e3, E0, E1, E2, E3, A, B, E);
                    double* xo = XC + par * XCS + 4 * lane;
                    sts2(xo, make_double2(sx * A, sx * B));
                    xo[2] = sx * E;
                }
                x0 = X0, y0 = Y0, x12 = X12, y12 = Y12, e0 = E0, e1 = E1, e2 = E2, e3 = E3;
                // q / out of plane I-1 from this stage (read before the release)
#ifndef MAS_ANISO_QREG
                if (n >= 2 && cell_ok) qv = lds2(Q_of(slot) + w * WK + c2);
#endif
                // stage n is no longer read: hand the slot back
                __syncwarp();
                if (lane == 0) mbar_arrive(empty0 + 8 * slot);
                consumer_sync();
                // ---- cells (w, c2..c2+1): corner rows w and w+1 -------------
                if (cell_ok) {
                    const double2 An1 = lds2(XA + par * XSZ + (w + 1) * WK + c2);
                    const double2 Yn1 = lds2(XY + par * XSZ + (w + 1) * WK + c2);
                    const double Sa = (B2a + Eda) + Yn1.x, Ta = A2a + An1.x;
                    double Sb = (B2b + Edb) + Yn1.y, Tb = A2b + An1.y;
                    if (edge) {  // the extra column's corners at rows w, w+1
                        const double* xc0 = XC + par * XCS + 4 * w;
                        const double2 ab0 = lds2(xc0), ab1 = lds2(xc0 + 4);
                        Sb += (ab0.y - xc0[2]) - (ab1.y + xc0[6]);
                        Tb += ab0.x + ab1.x;
                    }
                    // corner plane I is the upper-r face of cell plane I-1 (-A) and
                    // the lower-r face of cell plane I (+A)
                    if (n >= 2) {
                        const double sv0 = carry.x + (Sa - Ta), sv1 = carry.y + (Sb - Tb);
                        const int i = I - 1;
                        const double ivr = ivr_here;  // 1/vr of plane i = I-1
                        const double y0 = sv0 * (ivr * cw0), y1 = sv1 * (ivr * cw1);
                        double* o = a.out + (size_t)i * plane + (size_t)(j0 + w) * g.np + k0 + c2;
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
                    }
                    carry = make_double2(Sa + Ta, Sb + Tb);
                }
                par ^= 1;
            }
        }
        __syncthreads();  // the next segment re-initialises the rings and barriers
    }

    if (MODE == MODE_PCGA) {
        double v[1] = {acc[0]};
        if (grid_reduce<1, WTHREADS>(v, a.scr, TKT_ANISO, p2p) && threadIdx.x == 0) {
            if (p2p)  // kernel B(k) sums every rank's part from MB_C
                p2p_publish(a.p2p, MB_C, p2p_seq(a.st->epoch, kit), v, 1);
            else
                a.st->pend_sigma = a.st->pend_sigma + v[0];  // <p,L_iso p> (kernel A) + <p,L_par p>
        }
    } else if (MODE == MODE_RESID) {
        if (grid_reduce<3, WTHREADS>(acc, a.scr, TKT_ANISO, p2p) && threadIdx.x == 0) {
            a.st->pend_ff = acc[0];
            a.st->pend_rr = acc[1];
            a.st->pend_rho = acc[2];
            if (p2p) {  // the init sums (kernel A(1) reads them from MB_B)
                const double pub[3] = {acc[2], acc[1], acc[0]};  // {rho, rr, ff}
                p2p_publish(a.p2p, MB_B, p2p_seq(a.st->epoch, 0), pub, 3);
            }
        }
    }
}

// ---------------------------------------------------------------------------
// launchers
// ---------------------------------------------------------------------------
// one resident wave: MAS_ANISO_MINB blocks per SM, each with an equal share of
// the (tile, r-plane) units (bounded by the reduction scratch)
static PFN_cuTensorMapEncodeTiled_v12000 tmap_encode_fn() {
    static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
    static std::once_flag once;
    std::call_once(once, [] {
        void* p = nullptr;
        cudaDriverEntryPointQueryResult q{};
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
    });
    return fn;
}

// L2 promotion of the tensor copies (default 64 B).  The boxes are 66-68 doubles wide and
// start 16 B off a 512 B boundary, so a 256 B promotion fetches up to 1.5x the
// row; MAS_TMA_PROMO = 0 | 64 | 128 | 256 selects (experiment hook)
static CUtensorMapL2promotion tma_promotion() {
    static const CUtensorMapL2promotion p = [] {
        const char* e = getenv("MAS_TMA_PROMO");
        const int v = e ? atoi(e) : 64;  // 64 B measured best at C2a (r2j: 53.7 us vs 55.8 at 256 B)
        return v == 0 ? CU_TENSOR_MAP_L2_PROMOTION_NONE
               : v == 64 ? CU_TENSOR_MAP_L2_PROMOTION_L2_64B
               : v == 128 ? CU_TENSOR_MAP_L2_PROMOTION_L2_128B
                          : CU_TENSOR_MAP_L2_PROMOTION_L2_256B;
    }();
    return p;
}

// fp64 tiled tensor map, no swizzle, out-of-bounds elements read as zero
static bool tmap(CUtensorMap* m, const double* base, int rank, const cuuint64_t* dims,
                 const cuuint64_t* strides, const cuuint32_t* box) {
    auto fn = tmap_encode_fn();
    if (!fn || !base) return false;
    const cuuint32_t es[5] = {1, 1, 1, 1, 1};
    return fn(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, (cuuint32_t)rank, const_cast<double*>(base), dims, strides,
              box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, tma_promotion(),
              CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

static bool build_maps(const AnisoArgs& a, AnisoMaps* M) {
    std::memset(M, 0, sizeof(*M));
    const Geo& g = a.g;
    const cuuint64_t np = (cuuint64_t)g.np, nt = (cuuint64_t)g.nt, nl = (cuuint64_t)g.nl;
    const cuuint64_t rs = np * 8, ps = np * nt * 8, fs = np * nt * nl * 8;
    const cuuint64_t d3[3] = {np, nt, nl}, s3[2] = {rs, ps};
    const cuuint64_t d2[2] = {np, nt}, s2[1] = {rs};
    const cuuint64_t d4[4] = {np, nt, nl, 3}, s4[3] = {rs, ps, fs};
    const cuuint64_t dh[3] = {np, nt, 3}, sh[2] = {rs, ps};
    const cuuint32_t bp[3] = {WPW, WPR, 1}, bps[3] = {2, WPR, 1};
    const cuuint32_t bp2[2] = {WPW, WPR}, bps2[2] = {2, WPR};
    const cuuint32_t bc[4] = {WCW, WCR, 1, 3}, bcs[4] = {2, WCR, 1, 3};
    const cuuint32_t bh[3] = {WCW, WCR, 3}, bhs[3] = {2, WCR, 3};
    const cuuint32_t bq[3] = {WK, WJ, 1};
    bool ok = tmap(&M->u, a.u.in, 3, d3, s3, bp) && tmap(&M->u_s, a.u.in, 3, d3, s3, bps) &&
              tmap(&M->ca, a.ca, 4, d4, s4, bc) && tmap(&M->ca_s, a.ca, 4, d4, s4, bcs) &&
              tmap(&M->out, a.out, 3, d3, s3, bq);
    if (ok && a.u.glo) {
        M->has_lo = 1;
        ok = tmap(&M->lo, a.u.glo, 2, d2, s2, bp2) && tmap(&M->lo_s, a.u.glo, 2, d2, s2, bps2);
    }
    if (ok && a.u.ghi) {
        M->has_hi = 1;
        ok = tmap(&M->hi, a.u.ghi, 2, d2, s2, bp2) && tmap(&M->hi_s, a.u.ghi, 2, d2, s2, bps2);
    }
    if (ok && a.ca_hi) {
        M->has_cahi = 1;
        ok = tmap(&M->cahi, a.ca_hi, 3, dh, sh, bh) && tmap(&M->cahi_s, a.ca_hi, 3, dh, sh, bhs);
    }
    return ok;
}

cudaError_t launch_aniso(int mode, const AnisoArgs& a0, cudaStream_t s) {
    AnisoArgs a = a0;
    a.ntj = (a.g.nt + WJ - 1) / WJ;
    a.ntk = (a.g.np + WK - 1) / WK;
    const int tiles = a.ntj * a.ntk;
    long long want = (long long)kAnisoBps * device_sms();  // one resident wave (the rings fill the SM)
    if (const char* e = getenv("MAS_ABLOCKS")) want = std::max(1, atoi(e));  // experiment hook
    want = std::min<long long>(want, (long long)tiles * a.g.nl);
    want = std::min<long long>(want, a.max_blocks);
    a.chunk = 0;
    a.nchunk = 0;
    const int blocks = (int)want;
    if (blocks <= 0) return cudaErrorInvalidValue;
    AnisoMaps M;
    if (!build_maps(a, &M)) {
        set_last_error("k_aniso: cuTensorMapEncodeTiled failed");
        return cudaErrorInvalidValue;
    }
    static DeviceOnce attr;
    cudaError_t e = attr.run([] {
        cudaError_t r = cudaFuncSetAttribute(k_aniso<MODE_APPLY>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                             kAnisoSmem);
        if (r == cudaSuccess)
            r = cudaFuncSetAttribute(k_aniso<MODE_RESID>, cudaFuncAttributeMaxDynamicSharedMemorySize, kAnisoSmem);
        if (r == cudaSuccess)
            r = cudaFuncSetAttribute(k_aniso<MODE_PCGA>, cudaFuncAttributeMaxDynamicSharedMemorySize, kAnisoSmem);
        return r;
    });
    if (e != cudaSuccess) return e;
    if (mode == MODE_APPLY)
        k_aniso<MODE_APPLY><<<blocks, WTHREADS, kAnisoSmem, s>>>(a, M);
    else if (mode == MODE_RESID)
        k_aniso<MODE_RESID><<<blocks, WTHREADS, kAnisoSmem, s>>>(a, M);
    else
        k_aniso<MODE_PCGA><<<blocks, WTHREADS, kAnisoSmem, s>>>(a, M);
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
    const long long N = (long long)((g.nl + kDiagChunk - 1) / kDiagChunk) * g.plane;  // columns x chunks
    const int blocks = (int)std::min<long long>((N + kThreads - 1) / kThreads, 148LL * 16);
    k_aniso_diag<<<blocks, kThreads, 0, s>>>(g, ca, ca_hi, D, dinv, bad);
    return cudaGetLastError();
}

}  // namespace mas
