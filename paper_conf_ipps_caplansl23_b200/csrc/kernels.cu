// kernels.cu — sm_100a kernels of the MAS implicit-parabolic PCG path.
//
// The path is HBM-bound ("highly memory-bound"; DESIGN.md
// §5 roofline), so there are no tensor-core contractions here: every kernel
// streams fp64 fields with 16-byte (double2) coalesced accesses along phi,
// stages (theta,phi) plane tiles with a one-cell halo in a shared-memory
// ring and marches along r (the r-neighbours are the adjacent ring slots).
// Kernel fusion follows the paper's own lesson that OpenACC's fused,
// asynchronous kernels beat the un-fused DC loops:
//
//   k_stencil<MODE_PCGA>  "kernel A":  beta, p = D^-1 r + beta p_old (also on
//       the halo), deferred x += alpha_{k-1} p_old, q = L p, partial <p,q>_V
//   k_pcg_b               "kernel B":  r -= alpha q, z = D^-1 r, <r,z>_V, <r,r>_V
//   k_stencil<MODE_RESID> init:  r = f - L x, <f,f>_V, <r,r>_V, <r,D^-1 r>_V
//   k_stencil<MODE_APPLY> y = L x (mas_op_apply)
//   k_stencil<MODE_CG1>   single-reduction PCG (NEXT-1, Chronopoulos-Gear):
//       s = w + beta s, r -= alpha s, x += alpha p, p = D^-1 r_old + beta p
//       (halo too for s, r), w = L D^-1 r, <r,D^-1 r>, <w,D^-1 r>, <r,r>:
//       ONE kernel and one reduction per iteration (FIRSTK: w0 = L D^-1 r0)
//
// Scalars (alpha, beta, convergence, breakdown) never leave the device: each
// reduction ends in a deterministic "last block" sum (fixed order, no fp64
// atomics) whose result the next kernel reads.  See DESIGN.md §5.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdint>

#include "mas_internal.h"
#include "reduce.cuh"

namespace mas {

#ifndef MAS_TJ
#define MAS_TJ 8
#endif
#ifndef MAS_MINB
#define MAS_MINB 2
#endif
#ifndef MAS_MINB1
#define MAS_MINB1 2
#endif
constexpr int TJ = MAS_TJ;     // theta rows per stencil tile (one warp per row)
constexpr int kSThreads = 32 * TJ;
#ifndef MAS_MAXCHUNK
#define MAS_MAXCHUNK 32
#endif
constexpr int kMaxChunk = MAS_MAXCHUNK;  // r-planes per stencil work item (host picks <= this)
constexpr int TK = 64;         // phi cells per tile (2 per lane, double2)
constexpr int OFF = 2;         // smem column of the first tile cell (16B aligned)
constexpr int ROW = TK + 4;    // smem row length: [pad][halo][64 cells][halo][pad]
constexpr int HROWS = TJ + 2;  // tile rows + 2 halo rows

enum { P_NORMAL = 0, P_FINAL = 1, P_ZERO = 2 };
enum { TKT_STENCIL = 0, TKT_B = 1, TKT_DOT = 2 };

// --------------------------------------------------------------------------
// field access
// --------------------------------------------------------------------------
// The stencil kernels index with 32-bit offsets (the host rejects slabs with
// ncomp * cells >= 2^31): fewer integer instructions on the address path.
__device__ __forceinline__ int plane32(const Geo& g) { return (int)g.plane; }
// --------------------------------------------------------------------------
__device__ __forceinline__ const double* plane_ptr(const Halo& h, int comp, int i, const Geo& g) {
    if (i < 0) return h.glo + (int)comp * h.slo;
    if (i >= g.nl) return h.ghi + (int)comp * h.shi;
    return h.in + ((int)comp * g.nl + i) * plane32(g);
}
__device__ __forceinline__ double2 ld2(const double* p) {
    return __ldg(reinterpret_cast<const double2*>(p));
}
__device__ __forceinline__ double2 lds2(const double* p) { return *reinterpret_cast<const double2*>(p); }
__device__ __forceinline__ void sts2(double* p, double2 v) { *reinterpret_cast<double2*>(p) = v; }
__device__ __forceinline__ void stg2(double* p, double2 v) { *reinterpret_cast<double2*>(p) = v; }
// use-once streams of kernel B (r, q: far larger than L2): evict-first loads
// and stores (A/B: kernel B -3..-5% at C3 and C2; the same hints in kernel A
// measured +2.6% there, so kernel A keeps the default policy)
// kernel A's stores (p, q, x): default policy (MAS_A_STCS, streaming stores,
// measured +2.8% on kernel A)
__device__ __forceinline__ void stg2a(double* p, double2 v) {
#ifdef MAS_A_STCS
    __stcs(reinterpret_cast<double2*>(p), v);
#else
    *reinterpret_cast<double2*>(p) = v;
#endif
}
#ifndef MAS_NO_CS
__device__ __forceinline__ void sts_cs(double* p, double2 v) { __stcs(reinterpret_cast<double2*>(p), v); }
__device__ __forceinline__ double2 ld_cs(const double* p) { return __ldcs(reinterpret_cast<const double2*>(p)); }
#else
__device__ __forceinline__ void sts_cs(double* p, double2 v) { *reinterpret_cast<double2*>(p) = v; }
__device__ __forceinline__ double2 ld_cs(const double* p) { return *reinterpret_cast<const double2*>(p); }
#endif

// Values that the stencil phase of a plane needs besides the smem ring.
template <int NC>
struct OwnRegs {
    double2 c;      // mass term
    double2 f[NC];  // RESID: rhs
    double2 di;     // RESID: 1/D
    double2 rn[NC]; // CG1 scalar: r_k for <r,u>, <r,r> in the stencil phase
};

// Raw inputs of one cell pair (or one cell in .x for a phi-halo column).
template <int NC>
struct Raw {
    double2 u[NC];   // PCGA: r;  APPLY/RESID: x
    double2 po[NC];  // PCGA: p_{k-1}
    double2 di;      // PCGA, CG1: 1/D
    double2 kap;
    double2 wv[NC];  // CG1: w_{k-1} (po holds s_{k-2})
};

template <bool SCALAR>
__device__ __forceinline__ double2 ldv(const double* p) {
    if (SCALAR) return make_double2(__ldg(p), 0.0);
    return ld2(p);
}

// Block-uniform base pointers of plane i of every field the producer reads.
template <int NC>
struct PlanePtrs {
    const double* u[NC];
    const double* po[NC];
    const double* w[NC];
    const double* di;
    const double* kap;
};

template <int MODE, int NC>
__device__ __forceinline__ PlanePtrs<NC> plane_ptrs(const StencilArgs& a, int i, bool first) {
    const Geo& g = a.g;
    PlanePtrs<NC> P;
    P.kap = plane_ptr(a.kappa, 0, i, g);
#pragma unroll
    for (int c = 0; c < NC; c++) P.u[c] = plane_ptr(a.u, c, i, g);
    constexpr bool KRY = MODE == MODE_PCGA || MODE == MODE_CG1;
    P.di = KRY ? plane_ptr(a.dinv, 0, i, g) : nullptr;
#pragma unroll
    for (int c = 0; c < NC; c++) P.po[c] = (KRY && !first) ? plane_ptr(a.pold, c, i, g) : nullptr;
#pragma unroll
    for (int c = 0; c < NC; c++) P.w[c] = (MODE == MODE_CG1 && !first) ? plane_ptr(a.w, c, i, g) : nullptr;
    return P;
}

template <int MODE, int NC, bool SCALAR>
__device__ __forceinline__ void load_raw(const PlanePtrs<NC>& P, int off, bool first, Raw<NC>& R) {
    R.kap = ldv<SCALAR>(P.kap + off);
#pragma unroll
    for (int c = 0; c < NC; c++) R.u[c] = ldv<SCALAR>(P.u[c] + off);
    if (MODE == MODE_PCGA || MODE == MODE_CG1) {
        R.di = ldv<SCALAR>(P.di + off);
        if (!first) {
#pragma unroll
            for (int c = 0; c < NC; c++) R.po[c] = ldv<SCALAR>(P.po[c] + off);
            if (MODE == MODE_CG1) {
#pragma unroll
                for (int c = 0; c < NC; c++) R.wv[c] = ldv<SCALAR>(P.w[c] + off);
            }
        }
    }
}

// Interior planes (no ghost buffer involved): every field is addressed as
// base + comp * Nl + idx with one 32-bit idx = i * plane + offset, so the
// per-load address is a single wide multiply-add on a uniform base.
template <int MODE, int NC, bool SCALAR>
__device__ __forceinline__ void load_raw_in(const StencilArgs& a, int Nl, int idx, bool first, Raw<NC>& R) {
    R.kap = ldv<SCALAR>(a.kappa.in + idx);
#pragma unroll
    for (int c = 0; c < NC; c++) R.u[c] = ldv<SCALAR>(a.u.in + c * Nl + idx);
    if (MODE == MODE_PCGA || MODE == MODE_CG1) {
        R.di = ldv<SCALAR>(a.dinv.in + idx);
        if (!first) {
#pragma unroll
            for (int c = 0; c < NC; c++) R.po[c] = ldv<SCALAR>(a.pold.in + c * Nl + idx);
            if (MODE == MODE_CG1) {
#pragma unroll
                for (int c = 0; c < NC; c++) R.wv[c] = ldv<SCALAR>(a.w.in + c * Nl + idx);
            }
        }
    }
}

// u entering the stencil: APPLY/RESID x;  PCGA p_k = D^-1 r + beta p_{k-1}
template <int MODE, int NC>
__device__ __forceinline__ void finish_raw(Raw<NC>& R, bool first, double beta) {
    if constexpr (MODE == MODE_PCGA) {
#pragma unroll
        for (int c = 0; c < NC; c++) {
            double2 z = make_double2(R.di.x * R.u[c].x, R.di.y * R.u[c].y);
            if (!first) {
                z.x = fma(beta, R.po[c].x, z.x);
                z.y = fma(beta, R.po[c].y, z.y);
            }
            R.u[c] = z;
        }
    }
}

// smem ring buffer of one plane: field f (0..NC-1 = u components, NC = kappa)
__device__ __forceinline__ double* sfield(double* buf, int f) { return buf + f * (HROWS * ROW); }

// Halo item of a thread (plane independent), one scalar cell: threads
// 0..2TK-1 cover the theta halo rows j0-1 and j0+height, threads
// 2TK..2TK+2TJ-1 the periodic phi halo columns.
struct HaloMeta {
    int hoff;  // offset in the plane
    int hidx;        // index in a ring field
    int hkind;       // 0 none, 1 load, 3 zeros (beyond a pole / theta wall),
                     // 4 / 5 load from the lower / upper theta neighbour's row
};

// hkind 4 / 5: the row beyond the local theta range belongs to the theta
// neighbour (2-D decomposition): hoff is then the phi index in that row.
__device__ __forceinline__ HaloMeta halo_meta(const Geo& g, int j0, int k0, int height, int width,
                                              bool tnb_lo, bool tnb_hi, bool diag = false) {
    const int t = threadIdx.x;
    HaloMeta m{0, 0, 0};
    if (t < 2 * TK) {
        const bool top = t < TK;
        const int kk = top ? t : t - TK;
        const int hr = top ? 0 : height + 1;
        const int j = j0 + hr - 1;
        if (kk < width) {
            m.hidx = hr * ROW + OFF + kk;
            m.hkind = (j >= 0 && j < g.nt) ? 1 : j < 0 ? (tnb_lo ? 4 : 3) : (tnb_hi ? 5 : 3);
            m.hoff = m.hkind >= 4 ? k0 + kk : (int)j * g.np + k0 + kk;
        }
    } else if (t < 2 * TK + 2 * TJ) {
        const int q = t - 2 * TK, side = q / TJ, r = q % TJ;
        if (r < height) {
            const int k = side == 0 ? (k0 - 1 + g.np) % g.np : (k0 + width) % g.np;
            m.hidx = (1 + r) * ROW + (side == 0 ? OFF - 1 : OFF + width);
            m.hkind = 1;
            m.hoff = (int)(j0 + r) * g.np + k;
        }
    } else if (diag && t < 2 * TK + 2 * TJ + 4) {
        // the 4 diagonal halo cells (j0-1 | j0+height, k0-1 | k0+width): the
        // corner gradients of the fused field-aligned term need them
        const int q = t - 2 * TK - 2 * TJ, bottom = q >> 1, right = q & 1;
        const int hr = bottom ? height + 1 : 0, j = j0 + hr - 1;
        const int k = right ? (k0 + width) % g.np : (k0 - 1 + g.np) % g.np;
        m.hidx = hr * ROW + (right ? OFF + width : OFF - 1);
        m.hkind = (j >= 0 && j < g.nt) ? 1 : 3;
        m.hoff = (int)j * g.np + k;
    }
    return m;
}

// One plane's loads of this thread, in flight in registers (the software
// pipeline issues plane i+2 before the stencil of plane i).
template <int NC>
struct Stage {
    Raw<NC> R;                          // own double2 pair
    double2 xv[NC];                     // own x (PCGA deferred update; CG1 x_{k-1})
    double2 pp[NC];                     // CG1: own p_{k-2}
    OwnRegs<NC> o;                      // own c (+ f, D^-1 for RESID)
};

// --- cp.async (LDGSTS) for the halo items --------------------------------
// The scalar halo items do not fit in registers next to the own pair's
// in-flight loads (ptxas spilled them, forcing an early wait), so each halo
// thread copies its item into a private shared-memory slot instead:
// layout [field][kHS], fields 0 kappa, 1 1/D, 2.. u[NC], po[NC]
// (+ w[NC] in MODE_CG1).
// (+ the 4 diagonal halo cells for the fused L_par only: the slot stride and
// the extra ghost-plane halo branch cost the 3-component kernel A ~20%)
template <bool LPAR>
constexpr int kHS = 2 * TK + 2 * TJ + (LPAR ? 4 : 0);
__device__ __forceinline__ void cpa8(double* sdst, const double* gsrc) {
    const unsigned sa = (unsigned)__cvta_generic_to_shared(sdst);
    asm volatile("cp.async.ca.shared.global [%0], [%1], 8;\n" ::"r"(sa), "l"(gsrc) : "memory");
}
__device__ __forceinline__ void cpa_commit() { asm volatile("cp.async.commit_group;\n" ::: "memory"); }
__device__ __forceinline__ void cpa_wait_all() { asm volatile("cp.async.wait_group 0;\n" ::: "memory"); }


// theta-neighbour row item (2-D decomposition): same private cp.async slots
// as a local halo item, addresses from the TRows descriptors
__device__ __forceinline__ const double* trow_at(const TRows& T, bool hi, int comp, int i, int k) {
    return hi ? T.hi + comp * T.cs_hi + i * T.ps_hi + k : T.lo + comp * T.cs_lo + i * T.ps_lo + k;
}
template <int MODE, int NC, bool LPAR = false>
__device__ __forceinline__ void trow_issue(const StencilArgs& a, int i, const HaloMeta& hm, bool first,
                                        double* h) {
    const bool hi = hm.hkind == 5;
    const int k = hm.hoff;
    cpa8(h, trow_at(a.tkappa, hi, 0, i, k));
#pragma unroll
    for (int c = 0; c < NC; c++) cpa8(h + (2 + c) * kHS<LPAR>, trow_at(a.tu, hi, c, i, k));
    if (MODE == MODE_PCGA || MODE == MODE_CG1) {
        cpa8(h + kHS<LPAR>, trow_at(a.tdinv, hi, 0, i, k));
        if (!first) {
#pragma unroll
            for (int c = 0; c < NC; c++) cpa8(h + (2 + NC + c) * kHS<LPAR>, trow_at(a.tpold, hi, c, i, k));
        }
    }
}

// PCGA: the two-iteration x update (x read and written by every second kernel
// A, which also reads p_{k-2}) for the scalar operator.  The 3-component kernel
// keeps the one-step update: with p_{k-2} in registers it spills, and loaded
// at commit time it measured 4% slower at C3 (profiles/README.md)
template <int NC>
constexpr bool kX2 = (NC == 1);

// --- L2 prefetch one plane ahead of the register pipeline -----------------
// The own-tile loads of plane i+2 are issued (into registers) before the
// stencil of plane i.  Before that, plane i+3's tile rows are prefetched into
// L2 by the bulk-copy engine (one cp.async.bulk.prefetch per (field, row):
// no registers, no LSU/MIO slots), so the DRAM queue stays fed while the
// block computes and the register loads mostly hit L2.
#ifndef MAS_NO_PREFETCH
#ifndef MAS_PF_DIST
#define MAS_PF_DIST 3
#endif
constexpr int kPfDist = MAS_PF_DIST;  // planes ahead of the stencil plane
// the single-reduction kernel (CG1) streams more fields per plane (w, s and
// its late own-only x, p loads): its prefetched lines must land closer to
// their use or L2 evicts them first (C3 CG1: distance 2 / 3 / 4 = 534 / 474 /
// 426 iters/s; kernel A at 3 is best: 707 against 665 at 2 or 4, r6pfab)
#ifndef MAS_PF_DIST_CG1
#define MAS_PF_DIST_CG1 2
#endif
template <int MODE>
constexpr int kPfDistOf = MODE == MODE_CG1 ? MAS_PF_DIST_CG1 : kPfDist;
#ifndef MAS_PF_SCALAR
#define MAS_PF_SCALAR 0  // the scalar kernel measured slower with the prefetch (r1e)
#endif
// evict_last policy on the prefetched lines (A/B: kernel B -2%, kernel A equal)
__device__ __forceinline__ void l2_prefetch_row(const double* p, int bytes) {
#ifndef MAS_PF_NORMAL
    unsigned long long pol;
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;\n" : "=l"(pol));
    asm volatile("cp.async.bulk.prefetch.L2.global.L2::cache_hint [%0], %1, %2;\n" ::"l"(p), "r"(bytes),
                 "l"(pol)
                 : "memory");
#else
    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;\n" ::"l"(p), "r"(bytes) : "memory");
#endif
}
template <int MODE, int NC>
__device__ __forceinline__ void plane_prefetch(const StencilArgs& a, int i, int j0, int k0, int height,
                                               int width, bool first, bool xupd) {
    const Geo& g = a.g;
    // fields: u[NC], po[NC] (PCGA, not first), x[NC] (xupd), dinv (PCGA), kappa, c
    // (+ CG1: w[NC], the own p[NC])
    constexpr bool KRY = MODE == MODE_PCGA || MODE == MODE_CG1;
    // (+ PCGA, kX2, with the x update: p_{k-2} from the p_k buffer, fields 3NC+3..)
    constexpr int NF = 3 * NC + 3 + (MODE == MODE_CG1 ? 2 * NC : (MODE == MODE_PCGA && kX2<NC> ? NC : 0));
    const int t = threadIdx.x;
    if (t >= NF * TJ) return;
    const int f = t / TJ, w = t - f * TJ;
    if (w >= height) return;
    const int Nl = (int)g.nl * plane32(g);
    const int off = i * plane32(g) + (j0 + w) * g.np + k0;
    const double* base = nullptr;
    if (f < NC) base = a.u.in + f * Nl;
    else if (f < 2 * NC) base = (KRY && !first) ? a.pold.in + (f - NC) * Nl : nullptr;
    else if (f < 3 * NC) base = (KRY && xupd) ? a.x + (f - 2 * NC) * Nl : nullptr;
    else if (f == 3 * NC) base = KRY ? a.dinv.in : nullptr;
    else if (f == 3 * NC + 1) base = a.kappa.in;
    else if (f == 3 * NC + 2) base = a.c;
    else if (MODE == MODE_PCGA) base = (kX2<NC> && xupd) ? a.pnew + (f - 3 * NC - 3) * Nl : nullptr;
    else if (f < 4 * NC + 3) base = (MODE == MODE_CG1 && !first) ? a.w.in + (f - 3 * NC - 3) * Nl : nullptr;
    else base = (MODE == MODE_CG1 && xupd) ? a.pnew + (f - 4 * NC - 3) * Nl : nullptr;
    if (base) l2_prefetch_row(base + off, width * 8);
}
#endif

// CG1, 3 components: the own-only x and p are loaded at commit time (L2 hits:
// the bulk prefetch runs kPfDist planes ahead) instead of one plane ahead in
// registers, which would spill (17 double2 of loads in flight per thread)
template <int NC>
constexpr bool kCg1LateOwn = (NC == 3);
// CG1: where <r_k,u_k> and <r_k,r_k> accumulate.  3 components: at commit
// (r_k is at hand; keeping it to the stencil phase spills); scalar: in the
// stencil phase with r_k carried in OwnRegs (measured 5% faster at C2)
template <int NC>
constexpr bool kCg1DotsAtCommit = (NC == 3);

template <int MODE, int NC, bool LPAR = false>
__device__ __forceinline__ void stage_issue(const StencilArgs& a, int i, int j0, int k0, int height,
                                            int width, const HaloMeta& hm, bool first, bool xupd,
                                            bool halo, bool own_work, Stage<NC>& S, double* hst) {
    const Geo& g = a.g;
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int kc = 2 * lane;
    const int Nl = (int)g.nl * plane32(g);
    const bool interior = (i >= 0) && (i < g.nl);  // uniform: no ghost buffer involved
    const int pl = plane32(g), ipl = i * pl;
    if (w < height && kc < width) {
        const int off = (int)(j0 + w) * g.np + k0 + kc;
        const int o3 = ipl + off;
        if (interior) {
            load_raw_in<MODE, NC, false>(a, Nl, o3, first, S.R);
        } else {
            const PlanePtrs<NC> P = plane_ptrs<MODE, NC>(a, i, first);
            load_raw<MODE, NC, false>(P, off, first, S.R);
        }
        if (own_work) {
            if (a.c) S.o.c = ld2(a.c + o3);
            if ((MODE == MODE_PCGA || (MODE == MODE_CG1 && !kCg1LateOwn<NC>)) && xupd) {
#pragma unroll
                for (int c = 0; c < NC; c++) S.xv[c] = lds2(a.x + c * Nl + o3);
            }
            if (((MODE == MODE_CG1 && !kCg1LateOwn<NC>) || (MODE == MODE_PCGA && kX2<NC>)) && xupd) {
#pragma unroll
                for (int c = 0; c < NC; c++) S.pp[c] = lds2(a.pnew + c * Nl + o3);
            }
            if (MODE == MODE_RESID) {
                S.o.di = ld2(a.dinv.in + o3);
#pragma unroll
                for (int c = 0; c < NC; c++) S.o.f[c] = ld2(a.f + c * Nl + o3);
            }
        }
    }
    if (halo && hm.hkind >= 4 && interior) {
        trow_issue<MODE, NC, LPAR>(a, i, hm, first, hst + threadIdx.x);
    } else if (halo && hm.hkind == 1) {
        double* h = hst + threadIdx.x;
        if (interior) {  // halo planes are stencil planes: always interior here
            const int hi = ipl + (int)hm.hoff;
            cpa8(h, a.kappa.in + hi);
#pragma unroll
            for (int c = 0; c < NC; c++) cpa8(h + (2 + c) * kHS<LPAR>, a.u.in + c * Nl + hi);
            if (MODE == MODE_PCGA || MODE == MODE_CG1) {
                cpa8(h + kHS<LPAR>, a.dinv.in + hi);
                if (!first) {
#pragma unroll
                    for (int c = 0; c < NC; c++)
                        cpa8(h + (2 + NC + c) * kHS<LPAR>, a.pold.in + c * Nl + hi);
                    if (MODE == MODE_CG1) {
#pragma unroll
                        for (int c = 0; c < NC; c++)
                            cpa8(h + (2 + 2 * NC + c) * kHS<LPAR>, a.w.in + c * Nl + hi);
                    }
                }
            }
        } else if (LPAR && MODE == MODE_PCGA) {
            // an r-ghost plane's halo (the fused field-aligned term's corners
            // read it): the ghost copy, or the neighbour's own array in place
            const PlanePtrs<NC> P = plane_ptrs<MODE, NC>(a, i, first);
            const int hi = (int)hm.hoff;
            cpa8(h, P.kap + hi);
#pragma unroll
            for (int c = 0; c < NC; c++) cpa8(h + (2 + c) * kHS<LPAR>, P.u[c] + hi);
            cpa8(h + kHS<LPAR>, P.di + hi);
            if (!first) {
#pragma unroll
                for (int c = 0; c < NC; c++) cpa8(h + (2 + NC + c) * kHS<LPAR>, P.po[c] + hi);
            }
        }
    }
    cpa_commit();
}

template <int MODE, int NC, bool LPAR = false>
__device__ __forceinline__ void stage_commit(const StencilArgs& a, int i, int j0, int k0, int height,
                                             int width, const HaloMeta& hm, bool first, double beta,
                                             double alpha_prev, double alpha_km2, bool xupd, bool halo,
                                             bool own_work,
                                             Stage<NC>& S, double* buf, double2& kown,
                                             OwnRegs<NC>& o, const double* hst, double (&acc)[3]) {
    const Geo& g = a.g;
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int kc = 2 * lane;
    const int Nl = (int)g.nl * plane32(g);
    if (w < height && kc < width) {
        if constexpr (MODE == MODE_CG1) {
            // s_{k-1} = w_{k-1} + beta s_{k-2};  r_k = r_{k-1} - alpha s_{k-1};
            // own: p_{k-1} = D^-1 r_{k-1} + beta p_{k-2};  x_k = x_{k-1} + alpha p_{k-1}
            // (alpha_prev = alpha_{k-1}, beta = beta_{k-1});  ring: u_k = D^-1 r_k
            const int o3 = (int)i * plane32(g) + (int)(j0 + w) * g.np + k0 + kc;
            double V0 = 0.0, V1 = 0.0;
            if (kCg1DotsAtCommit<NC> && own_work) {  // <r_k, u_k>_V and <r_k, r_k>_V (own cells)
                const double vrt = __ldg(g.vr + i) * __ldg(g.vt + j0 + w);
                const double2 vp = ld2(g.vp + k0 + kc);
                V0 = vrt * vp.x;
                V1 = vrt * vp.y;
            }
#pragma unroll
            for (int c = 0; c < NC; c++) {
                double2 rk = S.R.u[c];
                if (!first) {
                    double2 sv;
                    sv.x = fma(beta, S.R.po[c].x, S.R.wv[c].x);
                    sv.y = fma(beta, S.R.po[c].y, S.R.wv[c].y);
                    rk.x = fma(-alpha_prev, sv.x, S.R.u[c].x);
                    rk.y = fma(-alpha_prev, sv.y, S.R.u[c].y);
                    if (own_work) {
                        const double2 pp = kCg1LateOwn<NC> ? lds2(a.pnew + c * Nl + o3) : S.pp[c];
                        double2 pv;
                        pv.x = fma(beta, pp.x, S.R.di.x * S.R.u[c].x);
                        pv.y = fma(beta, pp.y, S.R.di.y * S.R.u[c].y);
                        double2 xv = kCg1LateOwn<NC> ? lds2(a.x + c * Nl + o3) : S.xv[c];
                        xv.x = fma(alpha_prev, pv.x, xv.x);
                        xv.y = fma(alpha_prev, pv.y, xv.y);
                        stg2a(a.sout + c * Nl + o3, sv);
                        stg2a(a.rout + c * Nl + o3, rk);
                        stg2a(a.pnew + c * Nl + o3, pv);
                        stg2a(a.x + c * Nl + o3, xv);
                    }
                }
                S.R.u[c] = make_double2(S.R.di.x * rk.x, S.R.di.y * rk.y);
                if (!kCg1DotsAtCommit<NC>) S.o.rn[c] = rk;
                if (kCg1DotsAtCommit<NC> && own_work) {
                    acc[0] += V0 * rk.x * S.R.u[c].x + V1 * rk.y * S.R.u[c].y;
                    acc[2] += V0 * rk.x * rk.x + V1 * rk.y * rk.y;
                }
            }
        } else {
            finish_raw<MODE, NC>(S.R, first, beta);
        }
        const int idx = (1 + w) * ROW + OFF + kc;
#pragma unroll
        for (int c = 0; c < NC; c++) sts2(sfield(buf, c) + idx, S.R.u[c]);
        sts2(sfield(buf, NC) + idx, S.R.kap);
        kown = S.R.kap;
        if (own_work) {
            o = S.o;
            if constexpr (MODE == MODE_PCGA) {
                const int o3 = (int)i * plane32(g) + (int)(j0 + w) * g.np + k0 + kc;
#pragma unroll
                for (int c = 0; c < NC; c++) {
                    if (xupd) {
                        double2 xv = S.xv[c];
                        if constexpr (kX2<NC>) {
                            // odd k >= 3: x += alpha_{k-2} p_{k-2} + alpha_{k-1} p_{k-1},
                            // the two fmas of two one-step updates (p_{k-2} was loaded
                            // one plane ahead, before p_k overwrites it)
                            xv.x = fma(alpha_km2, S.pp[c].x, xv.x);
                            xv.y = fma(alpha_km2, S.pp[c].y, xv.y);
                        }
                        xv.x = fma(alpha_prev, S.R.po[c].x, xv.x);
                        xv.y = fma(alpha_prev, S.R.po[c].y, xv.y);
                        stg2a(a.x + c * Nl + o3, xv);
                    }
                    stg2a(a.pnew + c * Nl + o3, S.R.u[c]);
                }
            }
        }
    }
    if (halo && (hm.hkind == 1 || hm.hkind >= 4)) {
        cpa_wait_all();  // this thread's own copies; read back below by the same thread
        const double* h = hst + threadIdx.x;
#pragma unroll
        for (int c = 0; c < NC; c++) {
            double u = h[(2 + c) * kHS<LPAR>];
            if (MODE == MODE_PCGA) {
                const double z = h[kHS<LPAR>] * u;
                u = first ? z : fma(beta, h[(2 + NC + c) * kHS<LPAR>], z);
            } else if (MODE == MODE_CG1) {
                if (!first) {  // r_k of the halo cell from its r, s, w of iteration k-1
                    const double sv = fma(beta, h[(2 + NC + c) * kHS<LPAR>], h[(2 + 2 * NC + c) * kHS<LPAR>]);
                    u = fma(-alpha_prev, sv, u);
                }
                u = h[kHS<LPAR>] * u;
            }
            sfield(buf, c)[hm.hidx] = u;
        }
        sfield(buf, NC)[hm.hidx] = h[0];
    } else if (halo && hm.hkind == 3) {
#pragma unroll
        for (int c = 0; c <= NC; c++) sfield(buf, c)[hm.hidx] = 0.0;
    }
}

// Own-cell region of a ring slot as the global-boundary ghost plane:
// u = 0 (homogeneous Dirichlet; irrelevant under Neumann, weight 0) and
// kappa_ghost = kappa_P so that the face kappa is kappa_P (reading R3).
template <int NC>
__device__ __forceinline__ void ghost_plane(double* buf, int height, int width, double2 kP, bool all = false) {
    if (all) {  // the fused L_par corners read the halo of this plane too: zeros
        for (int t = threadIdx.x; t < HROWS * ROW; t += kSThreads) sfield(buf, 0)[t] = 0.0;
    }
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int kc = 2 * lane;
    if (w < height && kc < width) {
        const int idx = (1 + w) * ROW + OFF + kc;
#pragma unroll
        for (int c = 0; c < NC; c++) sts2(sfield(buf, c) + idx, make_double2(0.0, 0.0));
        sts2(sfield(buf, NC) + idx, kP);
    }
}

// Global <f,f>, <r_{k-1},r_{k-1}>, <r_{k-1},z_{k-1}> entering A(k): from
// PcgState (one GPU / NCCL allreduce in place), or summed from the mailbox of
// B(k-1) (init at k = 1) under the P2P transport.  block: every thread of
// the block calls (thread 0 waits, the others read its sums); otherwise the
// calling thread alone.
__device__ __forceinline__ void a_globals(const StencilArgs& a, int kit, double& ff, double& rr,
                                          double& rho1, bool block = false) {
    const PcgState* st = a.st;
    ff = __ldcg(&st->pend_ff);
    rr = __ldcg(&st->pend_rr);
    rho1 = __ldcg(&st->pend_rho);
    if (a.p2p.nranks > 0) {
        __shared__ double sh[3];
        double v[3];
        if (!block || threadIdx.x == 0) {
            p2p_gather_one<3>(a.p2p, MB_B, p2p_seq(__ldcg(&st->epoch), kit - 1), v);
            if (block) sh[0] = v[0], sh[1] = v[1], sh[2] = v[2];
        }
        if (block) {
            __syncthreads();
            v[0] = sh[0], v[1] = sh[1], v[2] = sh[2];
        }
        rho1 = v[0];
        rr = v[1];
        if (kit == 1) ff = v[2];
    }
}

// --------------------------------------------------------------------------
// field-aligned term fused into kernel A (NEXT-4; readings R21-R26; DESIGN.md
// §5.3): the corner coefficients (a, b, e) of one corner plane are staged per
// plane, the corners of the tile computed once into the 4 sign combinations
// c[st,sp] = s a + st s b + sp s e (s = a Dr + b Dt + e Dp), and every cell
// gathers its 8 corners: V (L_par p)_P = sum_lower c[st,sp] - sum_upper
// c[-st,-sp].  Same arithmetic as k_aniso (aniso.cu), one kernel less: p_k
// and q never leave the SM for it (24 of its 48 bytes per cell).
// --------------------------------------------------------------------------
constexpr int LCR = TJ + 1;    // corner rows of a tile (J = j0 .. j0+TJ)
constexpr int LCW = TK + 2;    // corner columns staged (K = k0 .. k0+65; 64 + 1 used)
constexpr int LCA = LCR * LCW; // one corner array
constexpr int kLparSmem = (2 * 3 + 4) * LCA;  // 2 staging buffers of (a, b, e) + 4 combinations

// cp.async of corner plane c's coefficients (rows J = j0 .. j0+height,
// columns K = k0 .. k0+width, K = np wrapping to 0) into buf [3][LCR][LCW];
// rows beyond nt-1 and a plane beyond the slab without a ghost copy are zeros
__device__ __forceinline__ void lpar_coef_issue(const StencilArgs& a, int c, int j0, int k0, int height,
                                                int width, double* buf) {
    const Geo& g = a.g;
    const long long N = (long long)g.nl * g.plane;
    const int pairs = width / 2 + 1;                  // pair m2 < width/2, then the single column width
    const int items = 3 * (height + 1) * pairs;
    for (int t = threadIdx.x; t < items; t += kSThreads) {
        const int f = t / ((height + 1) * pairs), rem = t - f * (height + 1) * pairs;
        const int q = rem / pairs, m2 = rem - q * pairs;
        const int J = j0 + q;
        double* dst = buf + f * LCA + q * LCW + 2 * m2;
        const double* src = nullptr;
        if (J < g.nt) {
            if (c < g.nl) src = a.ca + f * N + (long long)c * g.plane + (long long)J * g.np;
            else if (a.ca_hi) src = a.ca_hi + f * g.plane + (long long)J * g.np;
        }
        if (m2 < width / 2) {
            if (src) {
                const unsigned sa = (unsigned)__cvta_generic_to_shared(dst);
                asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(sa), "l"(src + k0 + 2 * m2)
                             : "memory");
            } else {
                dst[0] = 0.0, dst[1] = 0.0;
            }
        } else {  // column width: K = k0 + width (np -> 0)
            const int K = (k0 + width) % g.np;
            if (src) cpa8(dst, src + K);
            else dst[0] = 0.0;
        }
    }
    cpa_commit();
}

// corners of corner plane c (cells c-1 | c in ring slots lo | hi) into the 4
// combination arrays cmb [4][LCR][LCW]
__device__ __forceinline__ void lpar_corners(const double* lo, const double* hi, const double* cf, double* cmb,
                                             int height, int width) {
    const int cols = width + 1, n = (height + 1) * cols;
    for (int t = threadIdx.x; t < n; t += kSThreads) {
        const int q = t / cols, m = t - q * cols;
        const int r0 = q * ROW + OFF + m - 1, r1 = r0 + ROW;  // cell rows J-1 | J, columns K-1 | K
        const double a00 = lo[r0], a01 = lo[r0 + 1], a10 = lo[r1], a11 = lo[r1 + 1];
        const double b00 = hi[r0], b01 = hi[r0 + 1], b10 = hi[r1], b11 = hi[r1 + 1];
        const double Dr = ((b00 - a00) + (b01 - a01)) + ((b10 - a10) + (b11 - a11));
        const double Dt = ((a10 - a00) + (a11 - a01)) + ((b10 - b00) + (b11 - b01));
        const double Dp = ((a01 - a00) + (a11 - a10)) + ((b01 - b00) + (b11 - b10));
        const int ci = q * LCW + m;
        const double A0 = cf[ci], B0 = cf[LCA + ci], E0 = cf[2 * LCA + ci];
        const double sc = A0 * Dr + B0 * Dt + E0 * Dp;
        const double A = sc * A0, B = sc * B0, E = sc * E0;
        cmb[ci] = (A + B) + E;            // st +, sp +
        cmb[LCA + ci] = (A + B) - E;      // st +, sp -
        cmb[2 * LCA + ci] = (A - B) + E;  // st -, sp +
        cmb[3 * LCA + ci] = (A - B) - E;  // st -, sp -
    }
}

// --------------------------------------------------------------------------
// the fused stencil kernel
// --------------------------------------------------------------------------
// One block = one (TJ x TK) theta-phi tile x one chunk of r-planes.  It
// marches along r keeping the last three produced planes (p and kappa with
// halo) in a shared-memory ring: slot(i) = (i - ia + 1) % 3.  Per plane:
//   produce(i+1): global loads of r, p_old, D^-1, kappa (+x, c for own cells)
//                 -> p_{i+1} into the ring (and x-update / p store)
//   sync; stencil(i) from the ring only (r-neighbours = adjacent slots); sync
// FIRSTK: kernel A of iteration 1 (p = D^-1 r, no x update) is its own
// instantiation, so the per-plane code of every other iteration carries no
// first-iteration branches.
// LPAR: the field-aligned term fused in (MODE_PCGA, NC = 1): q = L_iso p +
// L_par p and <p, q> of both in one pass.
template <int MODE, int NC, bool FIRSTK = false, bool LPAR = false>
__global__ void __launch_bounds__(kSThreads, NC == 1 ? MAS_MINB1 : MAS_MINB) k_stencil(const StencilArgs a) {
    extern __shared__ __align__(16) double smem[];
    constexpr int BUF = (NC + 1) * HROWS * ROW;
    static_assert(!LPAR || (MODE == MODE_PCGA && NC == 1), "fused L_par: scalar kernel A only");
    const Geo& g = a.g;
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;

    // ---- PCG scalars (all threads read the same device values) ----------
    int pmode = P_NORMAL;
    bool first = false;
    // CG1: the global sums of kernel k-1 and, on a stop, its status / count
    double cg_g1 = 0.0, cg_d1 = 0.0, cg_rr1 = 0.0;
    int cg_status = -1, cg_iters = 0;
    double beta = 0.0, alpha_prev = 0.0;
    double alpha_km2 = 0.0;  // PCGA: alpha_{k-2} (saved by A(k-1))
    int kit = 0;
    const bool p2p = a.p2p.nranks > 0;
    __shared__ double final_g[3];
    if (MODE == MODE_PCGA) {
        // one round trip: everything A(k) needs sits in PcgState (written by
        // earlier kernels; read through L2)
        const PcgState* st = a.st;
        if (__ldcg(&st->stopped)) {
            // already decided (possibly before the graph's while loop started):
            // end the loop
            if (a.cond && blockIdx.x == 0 && threadIdx.x == 0)
                cudaGraphSetConditional((cudaGraphConditionalHandle)a.cond, 0);
            return;
        }
        kit = __ldcg(&st->k);
        double ff, rr, rho1;
        a_globals(a, kit, ff, rr, rho1, true);
        final_g[0] = ff, final_g[1] = rr, final_g[2] = rho1;  // for the stop branch below
        const double rho2 = __ldcg(&st->rho_prev);
        const double sig1 = __ldcg(&st->sigma_prev);
        first = (kit == 1);
        if (kit >= 2) alpha_prev = rho2 / sig1;
        if (kit >= 3) alpha_km2 = __ldcg(&st->alpha_save);
        if (first && ff == 0.0)
            pmode = P_ZERO;
        else if (sqrt(rr) <= __ldcg(&st->tol) * sqrt(ff) || kit > __ldcg(&st->maxit))
            pmode = P_FINAL;
        else if (!first)
            beta = rho1 / rho2;
    } else if (MODE == MODE_CG1) {
        // single reduction: kernel k (k >= 1) finds in PcgState the GLOBAL sums
        // of kernel k-1 (gamma_{k-1}, delta_{k-1}, ||r_{k-1}||^2; allreduced in
        // place between the kernels on r-slabs) and the gamma_{k-2}, alpha_{k-2}
        // kernel k-1 saved.  Every block takes the same decision: stop (r_{k-1}
        // met tol, maxit reached, breakdown), else alpha_{k-1}, beta_{k-1}.
        const PcgState* st = a.st;
        if (__ldcg(&st->stopped)) {
            if (a.cond && blockIdx.x == 0 && threadIdx.x == 0)
                cudaGraphSetConditional((cudaGraphConditionalHandle)a.cond, 0);
            return;
        }
        kit = __ldcg(&st->k);
        double ff = __ldcg(&st->pend_ff);
        // P2P transport: the global sums come from the mailbox, summed in rank
        // order (the init's from k_stencil<RESID>'s slot B {rho, rr, ff};
        // kernel k-1's {gamma, delta, ||r||^2} from slot A / C by its parity)
        double pv[3] = {0.0, 0.0, 0.0};
        if (p2p) {
            __shared__ double sh_pv[3];
            if (threadIdx.x == 0) {
                const unsigned long long ep = __ldcg(&st->epoch);
                if (FIRSTK) p2p_gather_one<3>(a.p2p, MB_B, p2p_seq(ep, 0), pv);
                else p2p_gather_one<3>(a.p2p, ((kit - 1) & 1) ? MB_C : MB_A, p2p_seq(ep, kit - 1), pv);
                sh_pv[0] = pv[0], sh_pv[1] = pv[1], sh_pv[2] = pv[2];
            }
            __syncthreads();
            pv[0] = sh_pv[0], pv[1] = sh_pv[1], pv[2] = sh_pv[2];
            if (FIRSTK) ff = pv[2];
        }
        if (FIRSTK) {  // the init: k = 0; r0 from k_stencil<RESID>
            const double rr = p2p ? pv[1] : __ldcg(&st->pend_rr);
            final_g[0] = ff, final_g[1] = rr, final_g[2] = 0.0;
            if (ff == 0.0)
                pmode = P_ZERO;
            else if (sqrt(rr) <= __ldcg(&st->tol) * sqrt(ff) || __ldcg(&st->maxit) == 0)
                pmode = P_FINAL;
        } else {
            cg_g1 = p2p ? pv[0] : __ldcg(&st->pend_rho);
            cg_d1 = p2p ? pv[1] : __ldcg(&st->pend_sigma);
            cg_rr1 = p2p ? pv[2] : __ldcg(&st->pend_rr);
            if (kit >= 2 && sqrt(cg_rr1) <= __ldcg(&st->tol) * sqrt(ff)) {
                pmode = P_FINAL, cg_status = MAS_OK, cg_iters = kit - 1;
            } else if (kit >= 2 && kit - 1 >= __ldcg(&st->maxit)) {
                pmode = P_FINAL, cg_status = MAS_NOT_CONVERGED, cg_iters = kit - 1;
            } else {
                const double b = kit >= 2 ? cg_g1 / __ldcg(&st->cg_gamma) : 0.0;
                const double den = kit >= 2 ? cg_d1 - b * cg_g1 / __ldcg(&st->cg_alpha) : cg_d1;  // <p,Lp>
                if (!(den > 0.0) || !isfinite(den)) {
                    pmode = P_FINAL, cg_status = MAS_ERR_BREAKDOWN, cg_iters = kit >= 2 ? kit - 1 : 1;
                } else {
                    beta = b;                     // beta_{k-1}
                    alpha_prev = cg_g1 / den;     // alpha_{k-1}
                }
            }
        }
    }
    // the deferred x update.  PCGA, scalar (kX2): every other kernel A, odd
    // k >= 3, applies the last two steps, x += alpha_{k-2} p_{k-2} + alpha_{k-1}
    // p_{k-1} (the same two fmas as two one-step updates; x read and written
    // every second iteration only, p_{k-2} read then).  PCGA,
    // 3 components: every kernel A, x += alpha_{k-1} p_{k-1}.  CG1: every kernel.
    const bool xupd = MODE == MODE_PCGA ? (!FIRSTK && (!kX2<NC> || ((kit & 1) && kit >= 3)))
                                        : (MODE == MODE_CG1 && !FIRSTK);
    if (MODE == MODE_PCGA && pmode == P_NORMAL && FIRSTK != first) __trap();  // host dispatch bug

    // ---- work item ------------------------------------------------------
    // work item; a split launch (multi-GPU seam overlap) covers either the
    // interior chunks 1..nchunk-2 or the edge chunks 0 and nchunk-1
    const int T = a.ntk * a.ntj;
    const int item = a.part == 1 ? T + (int)blockIdx.x
                     : a.part == 2 ? ((int)blockIdx.x < T ? (int)blockIdx.x : T * (a.nchunk - 2) + (int)blockIdx.x)
                                   : (int)blockIdx.x;
    const int tk = item % a.ntk;
    const int tj = (item / a.ntk) % a.ntj;
    const int ch = item / (a.ntk * a.ntj);
    const int j0 = tj * TJ, k0 = tk * TK;
    const int height = min(TJ, g.nt - j0), width = min(TK, g.np - k0);
    const int ia = ch * a.chunk, ib = min(ia + a.chunk, g.nl);
    const int kc = 2 * lane;
    const bool own = (w < height) && (kc < width);
    const int j = j0 + w, k = k0 + kc;
    const int off = (int)j * g.np + k;
    const int Nl = (int)g.nl * plane32(g);

    double acc[3] = {0.0, 0.0, 0.0};

    if ((MODE == MODE_PCGA || MODE == MODE_CG1) && pmode != P_NORMAL) {
        // final deferred update x += alpha_{k-1} p_{k-1} (or x = 0 if f == 0)
        if (own) {
            for (int i = ia; i < ib; i++) {
#pragma unroll
                for (int c = 0; c < NC; c++) {
                    double* xp = a.x + c * Nl + (int)i * plane32(g) + off;
                    if (pmode == P_ZERO) {
                        stg2(xp, make_double2(0.0, 0.0));
                    } else if (MODE == MODE_PCGA && kit >= 2) {
                        // the pending steps of the two-iteration update: alpha_{k-1}
                        // p_{k-1}, and for odd k also alpha_{k-2} p_{k-2} (still in
                        // the p_k buffer: this kernel writes no p_k)
                        const double2 po = ld2(plane_ptr(a.pold, c, i, g) + off);
                        double2 xv = lds2(xp);
                        if (kX2<NC> && (kit & 1)) {
                            const double2 pp = lds2(a.pnew + c * Nl + (int)i * plane32(g) + off);
                            xv.x = fma(alpha_km2, pp.x, xv.x);
                            xv.y = fma(alpha_km2, pp.y, xv.y);
                        }
                        xv.x = fma(alpha_prev, po.x, xv.x);
                        xv.y = fma(alpha_prev, po.y, xv.y);
                        stg2(xp, xv);
                    }
                }
            }
        }
        double v1[1] = {0.0};
        if (grid_reduce<1, kSThreads>(v1, a.scr, TKT_STENCIL) && threadIdx.x == 0 && a.part != 1) {
            PcgState* st = a.st;
            const double ff = final_g[0], rr = final_g[1], rho1 = final_g[2];
            // PCGA: A(k) stops at iterate k-1;  CG1: kernel k at iterate k-1 (its
            // init, k = 0, at iterate 0)
            const int hk = MODE == MODE_CG1 ? (FIRSTK ? 0 : kit - 1) : kit - 1;
            a.rr_hist[hk] = (MODE == MODE_CG1 && !FIRSTK) ? cg_rr1 : rr;
            a.rho_hist[hk] = (MODE == MODE_CG1 && !FIRSTK) ? cg_g1 : rho1;
            if (MODE == MODE_CG1 && !FIRSTK) {
                st->iters = cg_iters;
                st->relres = sqrt(cg_rr1) / sqrt(st->pend_ff);
                st->status = cg_status;
            } else if (pmode == P_ZERO) {
                st->iters = 0;
                st->relres = 0.0;
                st->status = MAS_OK;
                a.rr_hist[0] = 0.0;
            } else {
                const bool conv = sqrt(rr) <= st->tol * sqrt(ff);
                st->iters = hk;
                st->relres = sqrt(rr) / sqrt(ff);
                st->status = conv ? MAS_OK : MAS_NOT_CONVERGED;
            }
            __threadfence();
            st->stopped = 1;
            if (a.host_flag) {
                __threadfence_system();
                *(volatile int*)a.host_flag = MODE == MODE_CG1 ? kit + 1 : kit;  // CG1: launch number
            }
            if (a.cond) cudaGraphSetConditional((cudaGraphConditionalHandle)a.cond, 0);
        }
        return;
    }

    // 4-slot ring: stencil(i) reads slots i-1, i, i+1 while plane i+2's loads
    // are in flight; plane i+2 is committed into the slot of plane i-2, so
    // one barrier per plane suffices.
    auto slot = [&](int i) { return smem + ((i - ia + 1) & 3) * BUF; };
    // private cp.async slots of the halo items: static shared memory, so the
    // shared-window address needs no runtime conversion
    __shared__ __align__(16) double hst_arr[(2 + (MODE == MODE_CG1 ? 3 : 2) * NC) * kHS<LPAR>];
    auto real_plane = [&](int p) { return !(p == g.nl && g.glob_hi); };

    // 1-D geometry of this work item staged in shared memory once (visible to
    // the stencil after the first barrier of the march)
    __shared__ __align__(16) double sgR[4][kMaxChunk];
    __shared__ __align__(16) double sgT[4][TJ];
    __shared__ __align__(16) double sgP[3][TK];
    for (int t = threadIdx.x; t < kMaxChunk; t += kSThreads) {
        const int i = min(ia + t, g.nl - 1);
        sgR[0][t] = g.wRm[i];
        sgR[1][t] = g.wRp[i];
        sgR[2][t] = g.irc2[i];
        sgR[3][t] = g.vr[i];
    }
    for (int t = threadIdx.x; t < TJ; t += kSThreads) {
        const int jj = min(j0 + t, g.nt - 1);
        sgT[0][t] = g.wTm[jj];
        sgT[1][t] = g.wTp[jj];
        sgT[2][t] = g.isc2[jj];
        sgT[3][t] = g.vt[jj];
    }
    for (int t = threadIdx.x; t < TK; t += kSThreads) {
        const int kk = min(k0 + t, g.np - 1);
        sgP[0][t] = g.wPm[kk];
        sgP[1][t] = g.wPp[kk];
        sgP[2][t] = g.vp[kk];
    }

#ifndef MAS_NO_PREFETCH
    // the planes the march reaches before its first in-loop prefetch
    if (NC == 3 || MAS_PF_SCALAR)
        for (int ip = ia + 1; ip < min(ia + kPfDistOf<MODE>, ib); ip++)
            plane_prefetch<MODE, NC>(a, ip, j0, k0, height, width, FIRSTK, xupd);
#endif
    // ---- prologue: planes ia-1 (own cells only) and ia --------------------
    OwnRegs<NC> oc, on;  // own-cell stencil inputs for the current / next plane
    double2 kown = make_double2(0.0, 0.0), kdummy;
    const bool lo_ghost = (ia == 0) && g.glob_lo;
    const HaloMeta hm = halo_meta(g, j0, k0, height, width, a.tkappa.lo != nullptr,
                                  a.tkappa.hi != nullptr, LPAR);
    // fused L_par: coefficient staging [2][3][LCR][LCW], combinations [4][LCR][LCW]
    double* const lcf = smem + 4 * BUF;
    double* const lcmb = lcf + 2 * 3 * LCA;
    double lpart0 = 0.0, lpart1 = 0.0;  // the lower-corner (corner plane i) part of this pair's L_par p
    double lcw0 = 0.0, lcw1 = 0.0;      // 1 / (vt_j vp_k) of the pair
    if (LPAR && own) {
        const double vt = __ldg(g.vt + j);
        lcw0 = 1.0 / (vt * __ldg(g.vp + k));
        lcw1 = 1.0 / (vt * __ldg(g.vp + k + 1));
    }
    // planes ia-1 (own cells only) and ia: both loads in flight together
    Stage<NC> S0, S;
    // (fused L_par: plane ia-1's halo is a corner input too, so it is loaded
    // in the prologue; the halo item copies of ia-1 and ia go one after the
    // other through the same private slots)
    if (!lo_ghost) {
        stage_issue<MODE, NC, LPAR>(a, ia - 1, j0, k0, height, width, hm, FIRSTK, false, LPAR, false, S0, hst_arr);
        if (LPAR)
            stage_commit<MODE, NC, LPAR>(a, ia - 1, j0, k0, height, width, hm, FIRSTK, beta, alpha_prev, alpha_km2, false,
                                   true, false, S0, slot(ia - 1), kdummy, on, hst_arr, acc);
    }
    stage_issue<MODE, NC, LPAR>(a, ia, j0, k0, height, width, hm, FIRSTK, xupd, true, true, S, hst_arr);
    if (!lo_ghost && !LPAR)
        stage_commit<MODE, NC, LPAR>(a, ia - 1, j0, k0, height, width, hm, FIRSTK, beta, alpha_prev, alpha_km2, false,
                               false, false, S0, slot(ia - 1), kdummy, on, hst_arr, acc);
    stage_commit<MODE, NC, LPAR>(a, ia, j0, k0, height, width, hm, FIRSTK, beta, alpha_prev, alpha_km2, xupd, true, true,
                           S, slot(ia), kown, oc, hst_arr, acc);
    if (lo_ghost) ghost_plane<NC>(slot(ia - 1), height, width, kown, LPAR);
    if (LPAR) {  // corner plane ia (cells ia-1 | ia): its lower-corner part for plane ia
        lpar_coef_issue(a, ia, j0, k0, height, width, lcf + (ia & 1) * 3 * LCA);
        cpa_wait_all();
        __syncthreads();
        lpar_corners(sfield(slot(ia - 1), 0), sfield(slot(ia), 0), lcf + (ia & 1) * 3 * LCA, lcmb, height,
                     width);
        __syncthreads();
        if (own) {
            const double* h = lcmb + w * LCW + kc;
            const double2 l0 = lds2(h), l2 = lds2(h + 2 * LCA + LCW);
            lpart0 = (l0.x + h[LCA + 1]) + (l2.x + h[3 * LCA + LCW + 1]);
            lpart1 = (l0.y + h[LCA + 2]) + (l2.y + h[3 * LCA + LCW + 2]);
        }
    }
    if (real_plane(ia + 1))
        stage_issue<MODE, NC, LPAR>(a, ia + 1, j0, k0, height, width, hm, FIRSTK, xupd && (ia + 1 < ib),
                              LPAR || ia + 1 < ib, ia + 1 < ib, S, hst_arr);
    if (LPAR) lpar_coef_issue(a, ia + 1, j0, k0, height, width, lcf + ((ia + 1) & 1) * 3 * LCA);

    for (int i = ia; i < ib; i++) {
        // commit plane i+1 (its loads were issued one plane earlier)
        if (real_plane(i + 1))
            stage_commit<MODE, NC, LPAR>(a, i + 1, j0, k0, height, width, hm, FIRSTK, beta, alpha_prev,
                                   alpha_km2, xupd && (i + 1 < ib), LPAR || i + 1 < ib, i + 1 < ib, S, slot(i + 1),
                                   kown, on, hst_arr, acc);
        else
            ghost_plane<NC>(slot(i + 1), height, width, kown, LPAR);
        if (LPAR) cpa_wait_all();  // the coefficient copies of corner plane i+1 (every thread)
        // issue plane i+2 (registers and private cp.async slots only): its
        // latency overlaps the stencil of plane i.  Issuing it before the
        // barrier measured faster for the scalar kernel and slower for the
        // 3-component one (tools/abtest.sh), hence the split.
        constexpr bool kIssueEarly = (NC == 1);
        if (kIssueEarly && i + 2 <= ib && real_plane(i + 2))
            stage_issue<MODE, NC, LPAR>(a, i + 2, j0, k0, height, width, hm, FIRSTK, xupd && (i + 2 < ib),
                                  LPAR || i + 2 < ib, i + 2 < ib, S, hst_arr);
        if (LPAR && i + 2 <= ib) lpar_coef_issue(a, i + 2, j0, k0, height, width, lcf + ((i + 2) & 1) * 3 * LCA);
        __syncthreads();
        if (LPAR) {  // corner plane i+1 (cells i | i+1) into the combinations
            lpar_corners(sfield(slot(i), 0), sfield(slot(i + 1), 0), lcf + ((i + 1) & 1) * 3 * LCA, lcmb,
                         height, width);
            __syncthreads();
        }
#ifndef MAS_NO_PREFETCH
        // 3-component kernels only: for the scalar kernel (C2: 256 work items,
        // under one wave) it measured slower (tools/abtest.sh)
        if ((NC == 3 || MAS_PF_SCALAR) && i + kPfDistOf<MODE> < ib)
            plane_prefetch<MODE, NC>(a, i + kPfDistOf<MODE>, j0, k0, height, width, FIRSTK, xupd);
#endif
        if (!kIssueEarly && i + 2 <= ib && real_plane(i + 2))
            stage_issue<MODE, NC, LPAR>(a, i + 2, j0, k0, height, width, hm, FIRSTK, xupd && (i + 2 < ib),
                                  i + 2 < ib, i + 2 < ib, S, hst_arr);

        if (own) {
            const double* S0 = slot(i);
            const double* Sm = slot(i - 1);
            const double* Sp = slot(i + 1);
            const int idx = (1 + w) * ROW + OFF + kc;
            // 1-D geometry from the block's shared-memory copy (no global latency per plane)
            const int ir = i - ia;
            const double wrm = sgR[0][ir], wrp = sgR[1][ir], irc = sgR[2][ir], vri = sgR[3][ir];
            const double wtm = sgT[0][w], wtp = sgT[1][w], isc = sgT[2][w], vtj = sgT[3][w];
            const double2 wpm2 = lds2(&sgP[0][kc]), wpp2 = lds2(&sgP[1][kc]), vpk2 = lds2(&sgP[2][kc]);
            const double wpm[2] = {wpm2.x, wpm2.y}, wpp[2] = {wpp2.x, wpp2.y}, vpk[2] = {vpk2.x, vpk2.y};

            const double2 kP = lds2(sfield(const_cast<double*>(S0), NC) + idx);
            const double2 kM = lds2(sfield(const_cast<double*>(Sm), NC) + idx);
            const double2 kN = lds2(sfield(const_cast<double*>(Sp), NC) + idx);
            const double2 kS = lds2(sfield(const_cast<double*>(S0), NC) + idx - ROW);
            const double2 kT = lds2(sfield(const_cast<double*>(S0), NC) + idx + ROW);
            const double kL = sfield(const_cast<double*>(S0), NC)[idx - 1];
            const double kR = sfield(const_cast<double*>(S0), NC)[idx + 2];
            const double it = irc * wtm, ip = irc * wtp, ic = irc * isc;
            // face coefficients a_f = w_f * (kappa_P + kappa_N)/2, cells e = 0, 1
            const double aRm0 = wrm * (0.5 * (kP.x + kM.x)), aRm1 = wrm * (0.5 * (kP.y + kM.y));
            const double aRp0 = wrp * (0.5 * (kP.x + kN.x)), aRp1 = wrp * (0.5 * (kP.y + kN.y));
            const double aTm0 = it * (0.5 * (kP.x + kS.x)), aTm1 = it * (0.5 * (kP.y + kS.y));
            const double aTp0 = ip * (0.5 * (kP.x + kT.x)), aTp1 = ip * (0.5 * (kP.y + kT.y));
            const double aPm0 = ic * wpm[0] * (0.5 * (kP.x + kL));
            const double aPm1 = ic * wpm[1] * (0.5 * (kP.y + kP.x));
            const double aPp0 = ic * wpp[0] * (0.5 * (kP.x + kP.y));
            const double aPp1 = ic * wpp[1] * (0.5 * (kP.y + kR));
            const double V0 = vri * vtj * vpk[0], V1 = vri * vtj * vpk[1];
            const double2 cP = a.c ? oc.c : make_double2(0.0, 0.0);
            const int pofs = (int)i * plane32(g) + off;
            // vector-Laplacian curvature terms (3 components, NEXT-2, R31): the
            // mass term of component m gains kappa_P * (2/r^2 | 1/(r sin)^2)
            const bool curv = NC == 3 && a.curv;
            const double cmr = 2.0 * irc, cma = ic;
#pragma unroll
            for (int c = 0; c < NC; c++) {
                const double* s0 = sfield(const_cast<double*>(S0), c);
                const double2 u = lds2(s0 + idx);
                const double2 uM = lds2(sfield(const_cast<double*>(Sm), c) + idx);
                const double2 uN = lds2(sfield(const_cast<double*>(Sp), c) + idx);
                const double2 uS = lds2(s0 + idx - ROW);
                const double2 uT = lds2(s0 + idx + ROW);
                const double uL = s0[idx - 1], uR = s0[idx + 2];
                double L0 = cP.x * u.x, L1 = cP.y * u.y;
                if (curv) {
                    const double cm = c == 0 ? cmr : cma;
                    L0 = fma(kP.x * cm, u.x, L0);
                    L1 = fma(kP.y * cm, u.y, L1);
                }
                L0 = fma(aRm0, u.x - uM.x, L0);
                L1 = fma(aRm1, u.y - uM.y, L1);
                L0 = fma(aRp0, u.x - uN.x, L0);
                L1 = fma(aRp1, u.y - uN.y, L1);
                L0 = fma(aTm0, u.x - uS.x, L0);
                L1 = fma(aTm1, u.y - uS.y, L1);
                L0 = fma(aTp0, u.x - uT.x, L0);
                L1 = fma(aTp1, u.y - uT.y, L1);
                L0 = fma(aPm0, u.x - uL, L0);
                L1 = fma(aPm1, u.y - u.x, L1);
                L0 = fma(aPp0, u.x - u.y, L0);
                L1 = fma(aPp1, u.y - uR, L1);
                const int o = c * Nl + pofs;
                if (MODE == MODE_RESID) {
                    const double r0 = oc.f[c].x - L0, r1 = oc.f[c].y - L1;
                    stg2(a.out + o, make_double2(r0, r1));
                    acc[0] += V0 * oc.f[c].x * oc.f[c].x + V1 * oc.f[c].y * oc.f[c].y;
                    acc[1] += V0 * r0 * r0 + V1 * r1 * r1;
                    acc[2] += V0 * r0 * (oc.di.x * r0) + V1 * r1 * (oc.di.y * r1);
                } else {
                    if constexpr (LPAR) {
                        // upper corners (corner plane i+1) from the combinations, lower
                        // ones (plane i) gathered one step earlier; then plane i+1's lower part
                        const double* h = lcmb + w * LCW + kc;
                        const double2 h3 = lds2(h + 3 * LCA), h1 = lds2(h + LCA + LCW);
                        const double up0 = (h3.x + h[2 * LCA + 1]) + (h1.x + h[LCW + 1]);
                        const double up1 = (h3.y + h[2 * LCA + 2]) + (h1.y + h[LCW + 2]);
                        const double iv = __ldg(a.ivr + i);
                        L0 += (lpart0 - up0) * (iv * lcw0);
                        L1 += (lpart1 - up1) * (iv * lcw1);
                        const double2 l0 = lds2(h), l2 = lds2(h + 2 * LCA + LCW);
                        lpart0 = (l0.x + h[LCA + 1]) + (l2.x + h[3 * LCA + LCW + 1]);
                        lpart1 = (l0.y + h[LCA + 2]) + (l2.y + h[3 * LCA + LCW + 2]);
                    }
                    stg2a(a.out + o, make_double2(L0, L1));
                    if (MODE == MODE_PCGA) acc[0] += V0 * u.x * L0 + V1 * u.y * L1;
                    // CG1: delta = <w,u> (+ gamma = <r,u>, <r,r> unless accumulated at commit)
                    if (MODE == MODE_CG1) {
                        acc[1] += V0 * L0 * u.x + V1 * L1 * u.y;
                        if (!kCg1DotsAtCommit<NC>) {
                            const double2 rk = oc.rn[c];
                            acc[0] += V0 * rk.x * u.x + V1 * rk.y * u.y;
                            acc[2] += V0 * rk.x * rk.x + V1 * rk.y * rk.y;
                        }
                    }
                }
            }
        }
        oc = on;
    }

    // ---- reductions -------------------------------------------------------
    if (MODE == MODE_RESID) {
        if (grid_reduce<3, kSThreads>(acc, a.scr, TKT_STENCIL, p2p) && threadIdx.x == 0) {
            PcgState* st = a.st;
            st->pend_ff = acc[0];
            st->pend_rr = acc[1];
            st->pend_rho = acc[2];
            if (p2p && !a.nopub) {  // (with the field-aligned term k_aniso<RESID> publishes)
                const double pub[3] = {acc[2], acc[1], acc[0]};  // {rho, rr, ff}
                p2p_publish(a.p2p, MB_B, p2p_seq(st->epoch, 0), pub, 3);
            }
        }
    } else if (MODE == MODE_CG1) {
        if (grid_reduce<3, kSThreads>(acc, a.scr, TKT_STENCIL, p2p) && threadIdx.x == 0) {
            // the single reduction of iteration k: this rank's gamma_k, delta_k,
            // ||r_k||^2 (summed over the ranks before kernel k+1 reads them).
            // Kernel k+1 decides; here the values it needs besides them.
            PcgState* st = a.st;
            if (!FIRSTK) {
                st->cg_gamma = cg_g1;        // gamma_{k-1}
                st->cg_alpha = alpha_prev;   // alpha_{k-1}
                a.rr_hist[kit - 1] = cg_rr1;
                a.rho_hist[kit - 1] = cg_g1;
                a.sigma_hist[kit - 1] = cg_d1;
            }
            st->pend_rho = acc[0];
            st->pend_sigma = acc[1];
            st->pend_rr = acc[2];
            st->k = kit + 1;
            if (p2p) {
                if (FIRSTK) st->pend_ff = final_g[0];  // the global ||f||^2 for every later kernel
                // the single reduction of iteration k: this rank's partials to
                // every rank's mailbox (slots alternate by parity: a rank publishes
                // k+2 only after every rank has consumed k)
                const double pub[3] = {acc[0], acc[1], acc[2]};
                p2p_publish(a.p2p, (kit & 1) ? MB_C : MB_A, p2p_seq(st->epoch, kit), pub, 3);
            }
        }
    } else if (MODE == MODE_PCGA) {
        double v[1] = {acc[0]};
        if (grid_reduce<1, kSThreads>(v, a.scr, TKT_STENCIL, p2p) && threadIdx.x == 0) {
            PcgState* st = a.st;
            if (a.part == 1) {
                st->sigma_part = v[0];  // completed by the edge launch
            } else {
                double ff, rr, rho1;
                a_globals(a, kit, ff, rr, rho1);
                st->pend_sigma = a.part == 2 ? st->sigma_part + v[0] : v[0];
                a.rr_hist[kit - 1] = rr;
                a.rho_hist[kit - 1] = rho1;
                st->rho_prev = rho1;  // rho_{k-1}, read as rho_{(k+1)-2} by A(k+1)
                st->alpha_save = alpha_prev;  // alpha_{k-1}: A(k+1)'s alpha_{k-2}, B(k)'s fix-up
                if (p2p) {
                    // globals for B(k) (alpha, breakdown report) and later A's
                    st->pend_rho = rho1;
                    st->pend_rr = rr;
                    st->pend_ff = ff;
                    p2p_publish(a.p2p, MB_A, p2p_seq(st->epoch, kit), v, 1);
                }
            }
        }
    }
}
// --------------------------------------------------------------------------
// kernel B: r -= alpha q ; z = D^-1 r ; <r,z>_V, <r,r>_V
// --------------------------------------------------------------------------
// TN (theta-node placement, NEXT-2 R29-R30): kernel B also does the pole pass
// on q that k_pole_avg did between kernel A and kernel B -- one block per
// (plane, pole) row forms the phi average of q with k_pole_avg's arithmetic
// (same bits), then updates that row with it; the main loop skips pole rows.
template <int NC, bool TN = false>
__global__ void __launch_bounds__(kThreads) k_pcg_b(const StreamArgs a) {
    const PcgState* vst = a.st;
    if (__ldcg(&vst->stopped)) {
        if (a.cond && blockIdx.x == 0 && threadIdx.x == 0)
            cudaGraphSetConditional((cudaGraphConditionalHandle)a.cond, 0);
        return;
    }
    const Geo& g = a.g;
    const int kit = __ldcg(&vst->k);
    const bool p2p = a.p2p.nranks > 0;
    double sigma = __ldcg(&vst->pend_sigma);
    if (p2p) {  // the allreduce of A(k): sigma_k (thread 0 waits, the block reads)
        __shared__ double sh_sigma;
        if (threadIdx.x == 0) {
            double v[1];
            const unsigned long long seq = p2p_seq(__ldcg(&vst->epoch), kit);
            p2p_gather_one<1>(a.p2p, MB_A, seq, v);
            if (a.aniso) {  // + the field-aligned part, summed over the ranks by k_aniso(k)
                double u[1];
                p2p_gather_one<1>(a.p2p, MB_C, seq, u);
                v[0] = v[0] + u[0];
            }
            sh_sigma = v[0];
        }
        __syncthreads();
        sigma = sh_sigma;
    }
    const bool brk = !(sigma > 0.0) || !isfinite(sigma) || (a.brk_at > 0 && kit == a.brk_at);
    const double alpha = __ldcg(&vst->pend_rho) / sigma;  // rho_{k-1} / sigma_k
    double acc[2] = {0.0, 0.0};
    if (kX2<NC> && brk && a.x && kit >= 2 && !(kit & 1)) {
        // breakdown at an even k: A(k) left x at x_{k-2} (two-iteration
        // update); the solve reports x_{k-1} = x_{k-2} + alpha_{k-1} p_{k-1}
        const double am1 = __ldcg(&vst->alpha_save);
        const double* pk1 = a.p[(kit - 1) & 1];
        const long long n = (long long)a.ncomp * g.nl * g.plane;
        for (long long e = blockIdx.x * (long long)blockDim.x + threadIdx.x; e < n;
             e += (long long)gridDim.x * blockDim.x)
            a.x[e] = fma(am1, pk1[e], a.x[e]);
    }
    if (TN && !brk) {
        // the pole rows (j = 0, nt-1 of the theta-node rows), block-uniform loop
        const long long Nl = (long long)g.nl * g.plane;
        __shared__ double pws[2][kThreads / 32];
        __shared__ double pavg;
        for (int u = blockIdx.x; u < 2 * g.nl; u += gridDim.x) {
            const int il = u >> 1, row = (u & 1) ? g.nt - 1 : 0;
            const long long base = ((long long)il * g.nt + row) * g.np;
            const double wrow = __ldg(g.vr + il) * __ldg(g.vt + row);
            for (int c = 0; c < NC; c++) {
                const double* qr = a.q + c * Nl + base;
                double* rr = a.r + c * Nl + base;
                // q, r, 1/D and the phi weights of the thread's cells, loaded
                // together (one round trip; rows of up to 4 * kThreads cells)
                constexpr int PK = 4;
                double qv[PK], rv0[PK], dv[PK], vp[PK];
                const bool fits = g.np <= PK * kThreads;
#pragma unroll
                for (int t = 0; t < PK; t++) {
                    const int k = threadIdx.x + t * kThreads;
                    const bool in = fits && k < g.np;
                    qv[t] = in ? qr[k] : 0.0;
                    rv0[t] = in ? rr[k] : 0.0;
                    dv[t] = in ? __ldg(a.dinv + base + k) : 0.0;
                    vp[t] = in ? __ldg(g.vp + k) : 0.0;
                }
                double sq = 0.0, sw = 0.0;
                if (fits) {
#pragma unroll
                    for (int t = 0; t < PK; t++)
                        if (threadIdx.x + t * kThreads < g.np) sq = fma(vp[t], qv[t], sq), sw += vp[t];
                } else {
                    for (int k = threadIdx.x; k < g.np; k += kThreads) {
                        const double dp = __ldg(g.vp + k);
                        sq = fma(dp, qr[k], sq);
                        sw += dp;
                    }
                }
                sq = warp_sum(sq);
                sw = warp_sum(sw);
                if ((threadIdx.x & 31) == 0) pws[0][threadIdx.x >> 5] = sq, pws[1][threadIdx.x >> 5] = sw;
                __syncthreads();
                if (threadIdx.x == 0) {
                    double ts = 0.0, tw = 0.0;
                    for (int t = 0; t < kThreads / 32; t++) ts += pws[0][t], tw += pws[1][t];
                    pavg = ts / tw;
                }
                __syncthreads();
                const double qbar = pavg;
                if (fits) {
#pragma unroll
                    for (int t = 0; t < PK; t++) {
                        const int k = threadIdx.x + t * kThreads;
                        if (k < g.np) {
                            const double rv = fma(-alpha, qbar, rv0[t]);
                            rr[k] = rv;
                            const double V = wrow * vp[t];
                            acc[0] += V * rv * (dv[t] * rv);
                            acc[1] += V * rv * rv;
                        }
                    }
                } else {
                    for (int k = threadIdx.x; k < g.np; k += kThreads) {
                        const double rv = fma(-alpha, qbar, rr[k]);
                        rr[k] = rv;
                        const double V = wrow * __ldg(g.vp + k);
                        acc[0] += V * rv * (__ldg(a.dinv + base + k) * rv);
                        acc[1] += V * rv * rv;
                    }
                }
                __syncthreads();  // pavg / pws reused by the next component or row
            }
        }
    }
    if (!brk) {
        const long long Nl = (long long)g.nl * g.plane;
        const int rows = g.nl * g.nt;
        const int half = g.np >> 1;
        // a block covers rpi whole (r,theta) rows per step when a row has
        // fewer double2 pairs than the block has threads
        const int tpr = min(kThreads, half), rpi = kThreads / tpr;
        const int sub = threadIdx.x / tpr, col = threadIdx.x - sub * tpr;
        if (sub >= rpi) goto reduce;
#ifndef MAS_B_NO_U2
        if constexpr (NC == 1) {
            // scalar operator (C2: 4 M cells, ~7 rows per block): two rows per
            // step, all six loads in flight before the arithmetic
            const int stride = gridDim.x * rpi;
            for (int row = blockIdx.x * rpi + sub; row < rows; row += 2 * stride) {
                int row1 = row, row2 = row + stride;
                bool two = row2 < rows;
                if (TN) {  // pole rows were done above
                    const int jj1 = row1 % g.nt, jj2 = row2 % g.nt;
                    const bool p1 = jj1 == 0 || jj1 == g.nt - 1, p2 = two && (jj2 == 0 || jj2 == g.nt - 1);
                    if (p2) two = false;
                    if (p1) {
                        if (!two) continue;
                        row1 = row2;
                        two = false;
                    }
                }
                const int i1 = row1 / g.nt, j1 = row1 - i1 * g.nt;
                const int i2 = two ? row2 / g.nt : i1, j2 = two ? row2 - i2 * g.nt : j1;
                const double w1 = __ldg(g.vr + i1) * __ldg(g.vt + j1);
                const double w2 = __ldg(g.vr + i2) * __ldg(g.vt + j2);
                const long long b1 = (long long)row1 * g.np, b2 = (long long)(two ? row2 : row1) * g.np;
                for (int h = col; h < half; h += tpr) {
                    const int k = 2 * h;
                    const double2 d1 = ld2(a.dinv + b1 + k), r1 = ld_cs(a.r + b1 + k), q1 = ld_cs(a.q + b1 + k);
                    double2 d2 = make_double2(0.0, 0.0), r2 = d2, q2 = d2;
                    if (two) {
                        d2 = ld2(a.dinv + b2 + k);
                        r2 = ld_cs(a.r + b2 + k);
                        q2 = ld_cs(a.q + b2 + k);
                    }
                    const double vp0 = __ldg(g.vp + k), vp1 = __ldg(g.vp + k + 1);
                    double2 rv = r1;
                    rv.x = fma(-alpha, q1.x, rv.x);
                    rv.y = fma(-alpha, q1.y, rv.y);
                    sts_cs(a.r + b1 + k, rv);
                    acc[0] += w1 * vp0 * rv.x * (d1.x * rv.x) + w1 * vp1 * rv.y * (d1.y * rv.y);
                    acc[1] += w1 * vp0 * rv.x * rv.x + w1 * vp1 * rv.y * rv.y;
                    if (two) {
                        double2 rw = r2;
                        rw.x = fma(-alpha, q2.x, rw.x);
                        rw.y = fma(-alpha, q2.y, rw.y);
                        sts_cs(a.r + b2 + k, rw);
                        acc[0] += w2 * vp0 * rw.x * (d2.x * rw.x) + w2 * vp1 * rw.y * (d2.y * rw.y);
                        acc[1] += w2 * vp0 * rw.x * rw.x + w2 * vp1 * rw.y * rw.y;
                    }
                }
            }
        } else
#endif
        for (int row = blockIdx.x * rpi + sub; row < rows; row += gridDim.x * rpi) {
            const int i = row / g.nt, j = row - i * g.nt;
            if (TN && (j == 0 || j == g.nt - 1)) continue;  // pole rows were done above
            const double wrow = __ldg(g.vr + i) * __ldg(g.vt + j);
            const long long base = (long long)row * g.np;
            for (int h = col; h < half; h += tpr) {
                const int k = 2 * h;
                const double2 di = ld2(a.dinv + base + k);
                const double V0 = wrow * __ldg(g.vp + k), V1 = wrow * __ldg(g.vp + k + 1);
                double2 r[NC], q[NC];
#pragma unroll
                for (int c = 0; c < NC; c++) {
                    r[c] = ld_cs(a.r + c * Nl + base + k);
                    q[c] = ld_cs(a.q + c * Nl + base + k);
                }
#pragma unroll
                for (int c = 0; c < NC; c++) {
                    double2 rv = r[c];
                    rv.x = fma(-alpha, q[c].x, rv.x);
                    rv.y = fma(-alpha, q[c].y, rv.y);
                    sts_cs(a.r + c * Nl + base + k, rv);
                    const double z0 = di.x * rv.x, z1 = di.y * rv.y;
                    acc[0] += V0 * rv.x * z0 + V1 * rv.y * z1;
                    acc[1] += V0 * rv.x * rv.x + V1 * rv.y * rv.y;
                }
            }
        }
    }
reduce:
    if (grid_reduce<2>(acc, a.scr, TKT_B, p2p) && threadIdx.x == 0) {
        PcgState* st = a.st;
        if (brk) {
            st->iters = kit;
            st->relres = sqrt(st->pend_rr) / sqrt(st->pend_ff);
            st->status = MAS_ERR_BREAKDOWN;
            a.rr_hist[kit - 1] = st->pend_rr;
            __threadfence();
            st->stopped = 1;
            if (a.host_flag) {
                __threadfence_system();
                *(volatile int*)a.host_flag = kit;
            }
            if (a.cond) cudaGraphSetConditional((cudaGraphConditionalHandle)a.cond, 0);
        } else {
            a.sigma_hist[kit] = sigma;
            st->sigma_prev = sigma;
            st->pend_rho = acc[0];
            st->pend_rr = acc[1];
            st->k = kit + 1;
            if (p2p) p2p_publish(a.p2p, MB_B, p2p_seq(st->epoch, kit), acc, 2);
        }
    }
}

// --------------------------------------------------------------------------
// setup kernels
// --------------------------------------------------------------------------
__device__ __forceinline__ double kap_at(const Halo& h, int i, long long off, const Geo& g) {
    return __ldg(plane_ptr(h, 0, i, g) + off);
}

// D = c + sum_f a_f (Dirichlet faces included via kappa_ghost = kappa_P),
// dinv = 1/D; flags negative / non-finite coefficients and D <= 0.
__global__ void __launch_bounds__(kThreads) k_diag(const Geo g, const Halo kappa, const TRows tk,
                                                   const double* c, double* D, double* dinv, int* bad) {
    const long long Nl = (long long)g.nl * g.plane;
    for (long long P = blockIdx.x * (long long)kThreads + threadIdx.x; P < Nl;
         P += (long long)gridDim.x * kThreads) {
        const int i = (int)(P / g.plane);
        const long long off = P - (long long)i * g.plane;
        const int j = (int)(off / g.np), k = (int)(off - (long long)j * g.np);
        const double kp = kappa.in[P];
        const double cp = c ? c[P] : 0.0;
        const double kim = (i == 0 && g.glob_lo) ? kp : kap_at(kappa, i - 1, off, g);
        const double kip = (i == g.nl - 1 && g.glob_hi) ? kp : kap_at(kappa, i + 1, off, g);
        // beyond the local theta rows: the theta neighbour's row, else 0 (pole / wall, weight 0)
        const double kjm = j > 0 ? kappa.in[P - g.np] : tk.lo ? tk.lo[(long long)i * tk.ps_lo + k] : 0.0;
        const double kjp = j < g.nt - 1 ? kappa.in[P + g.np]
                                        : tk.hi ? tk.hi[(long long)i * tk.ps_hi + k] : 0.0;
        const int km = k == 0 ? g.np - 1 : k - 1, kq = k == g.np - 1 ? 0 : k + 1;
        const double kkm = kappa.in[P - k + km], kkp = kappa.in[P - k + kq];
        const double irc = g.irc2[i];
        double s = cp;
        s += g.wRm[i] * (0.5 * (kp + kim));
        s += g.wRp[i] * (0.5 * (kp + kip));
        s += irc * g.wTm[j] * (0.5 * (kp + kjm));
        s += irc * g.wTp[j] * (0.5 * (kp + kjp));
        s += irc * g.isc2[j] * g.wPm[k] * (0.5 * (kp + kkm));
        s += irc * g.isc2[j] * g.wPp[k] * (0.5 * (kp + kkp));
        if (D) D[P] = s;
        dinv[P] = 1.0 / s;
        const bool ok = (kp >= 0.0) && isfinite(kp) && (cp >= 0.0) && isfinite(cp) && (s > 0.0) &&
                        isfinite(s);
        if (!ok) atomicOr(bad, 1);
    }
}

// f += w_b kappa_P u_b on a Dirichlet boundary plane (inner: plane 0, wRm;
// outer: plane nl-1, wRp).
__global__ void k_dirichlet(const Geo g, int ncomp, const double* kappa, const double* ub, int outer,
                            double* f) {
    const long long plane = g.plane;
    const long long Nl = (long long)g.nl * plane;
    const int i = outer ? g.nl - 1 : 0;
    const double wgt = outer ? g.wRp[i] : g.wRm[i];
    for (long long t = blockIdx.x * (long long)blockDim.x + threadIdx.x; t < plane * ncomp;
         t += (long long)gridDim.x * blockDim.x) {
        const int c = (int)(t / plane);
        const long long off = t - c * plane;
        const long long P = (long long)i * plane + off;
        f[c * Nl + P] += wgt * kappa[P] * ub[t];
    }
}

__global__ void __launch_bounds__(kThreads) k_dot(const Geo g, int ncomp, const double* x,
                                                  const double* y, Scratch scr, double* out) {
    double acc[1] = {0.0};
    const long long Nl = (long long)g.nl * g.plane;
    const int rows = g.nl * g.nt;
    for (int row = blockIdx.x; row < rows; row += gridDim.x) {
        const int i = row / g.nt, j = row - i * g.nt;
        const double wrow = g.vr[i] * g.vt[j];
        const long long base = (long long)row * g.np;
        for (int k = threadIdx.x; k < g.np; k += kThreads) {
            const double V = wrow * g.vp[k];
            for (int c = 0; c < ncomp; c++) acc[0] += V * x[c * Nl + base + k] * y[c * Nl + base + k];
        }
    }
    if (grid_reduce<1>(acc, scr, TKT_DOT) && threadIdx.x == 0) *out = acc[0];
}

// Per-radius array reduction, the paper's Listings 3-5 (P:428-445,
// P:592-645): sum0(i) = sum_j array(i,j) * w(j), here with the angular index
// (j,k) and a caller-supplied weight (reading R27).  MAS's OpenACC version
// uses atomic updates; the paper's DC rewrite reduces each i in an inner
// loop.  On the GPU: one block per (component, r-plane), double2 loads, a
// fixed-order block tree (deterministic, no atomics).
__global__ void __launch_bounds__(kThreads) k_radial_sums(const Geo g, const double* x, const double* w,
                                                          double* out) {
    __shared__ double ws[kThreads / 32];
    const int b = blockIdx.x;  // m * nl + i
    const long long plane = g.plane;
    const double* xp = x + (long long)b * plane;
    // four independent pairs in flight per thread, summed in a fixed order
    double s4[4] = {0.0, 0.0, 0.0, 0.0};
    long long e = 2 * threadIdx.x;
    for (; e + 6 * kThreads < plane; e += 8 * kThreads) {
        double2 xv[4], wv[4];
#pragma unroll
        for (int u = 0; u < 4; u++) {
            xv[u] = ld2(xp + e + 2 * u * kThreads);
            wv[u] = ld2(w + e + 2 * u * kThreads);
        }
#pragma unroll
        for (int u = 0; u < 4; u++) {
            s4[u] = fma(wv[u].x, xv[u].x, s4[u]);
            s4[u] = fma(wv[u].y, xv[u].y, s4[u]);
        }
    }
    for (; e < plane; e += 2 * kThreads) {
        const double2 xv = ld2(xp + e), wv = ld2(w + e);
        s4[0] = fma(wv.x, xv.x, s4[0]);
        s4[0] = fma(wv.y, xv.y, s4[0]);
    }
    double s = (s4[0] + s4[1]) + (s4[2] + s4[3]);
    s = warp_sum(s);
    if ((threadIdx.x & 31) == 0) ws[threadIdx.x >> 5] = s;
    __syncthreads();
    if (threadIdx.x == 0) {
        double t = 0.0;
        for (int q = 0; q < kThreads / 32; q++) t += ws[q];
        out[b] = t;
    }
}

// --------------------------------------------------------------------------
// theta-node placement (NEXT-2, readings R29-R30): the pole
// rows 0 and nt (local rows 0 and g.nt-1) hold one value per radius.  The
// stencil kernels compute each phi slot k of a pole row as its own polar-cap
// slice (volume V_k = rC^2 dr A dp_k); the cap balance is the dp-weighted
// phi average of the slices -- the paper's per-radius sum0 array reduction
// (Listings 3-5) -- written back to every slot.
// One block per (component, plane, pole); fixed-order tree (deterministic).
// dinv != nullptr (the Jacobi diagonal, ncomp = 1): dinv = 1 / average too.
// --------------------------------------------------------------------------
__global__ void __launch_bounds__(kThreads) k_pole_avg(const Geo g, double* y, double* dinv, int plane_lo,
                                                        int nplanes) {
    __shared__ double ws[2][kThreads / 32];
    __shared__ double avg;
    const int pole = blockIdx.x & 1;
    const int q = blockIdx.x >> 1;             // comp * nplanes + plane
    const int comp = q / nplanes, il = plane_lo + q % nplanes;
    const int row = pole ? g.nt - 1 : 0;
    double* yr = y + ((long long)comp * g.nl + il) * g.plane + (long long)row * g.np;
    double s = 0.0, w = 0.0;
    for (int k = threadIdx.x; k < g.np; k += kThreads) {
        const double dp = __ldg(g.vp + k);
        s = fma(dp, yr[k], s);
        w += dp;
    }
    s = warp_sum(s);
    w = warp_sum(w);
    if ((threadIdx.x & 31) == 0) ws[0][threadIdx.x >> 5] = s, ws[1][threadIdx.x >> 5] = w;
    __syncthreads();
    if (threadIdx.x == 0) {
        double ts = 0.0, tw = 0.0;
        for (int t = 0; t < kThreads / 32; t++) ts += ws[0][t], tw += ws[1][t];
        avg = ts / tw;
    }
    __syncthreads();
    const double a = avg;
    for (int k = threadIdx.x; k < g.np; k += kThreads) {
        yr[k] = a;
        if (dinv) dinv[(long long)il * g.plane + (long long)row * g.np + k] = 1.0 / a;
    }
}

// <f,f>_V, <r,r>_V, <r,D^-1 r>_V of the init (after the pole rows of r were
// averaged) into PcgState: the values k_stencil<RESID> computed per slot are
// replaced.  Same grid-stride row order as kernel B.
__global__ void __launch_bounds__(kThreads) k_init_dots(const Geo g, int ncomp, const double* f, const double* r,
                                                         const double* dinv, Scratch scr, PcgState* st) {
    double acc[3] = {0.0, 0.0, 0.0};
    const long long Nl = (long long)g.nl * g.plane;
    const int rows = g.nl * g.nt;
    for (int row = blockIdx.x; row < rows; row += gridDim.x) {
        const int i = row / g.nt, j = row - i * g.nt;
        const double wrow = g.vr[i] * g.vt[j];
        const long long base = (long long)row * g.np;
        for (int k = threadIdx.x; k < g.np; k += kThreads) {
            const double V = wrow * g.vp[k], di = dinv[base + k];
            for (int c = 0; c < ncomp; c++) {
                const double fv = f[c * Nl + base + k], rv = r[c * Nl + base + k];
                acc[0] += V * fv * fv;
                acc[1] += V * rv * rv;
                acc[2] += V * rv * (di * rv);
            }
        }
    }
    if (grid_reduce<3>(acc, scr, TKT_DOT) && threadIdx.x == 0) {
        st->pend_ff = acc[0];
        st->pend_rr = acc[1];
        st->pend_rho = acc[2];
    }
}

// a[i] = 1 + 0.25 * h(i) / 1024 with h a multiplicative hash: finite,
// positive, non-constant values (kernel-replay timing inputs; mas_op_kernel_bench)
__global__ void k_fill_test(double* a, long long n) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n;
         i += (long long)gridDim.x * blockDim.x)
        a[i] = 1.0 + 0.25 * (double)(((unsigned long long)i * 2654435761ull) % 1024ull) / 1024.0;
}

// read-only sweep over a buffer larger than L2: evicts the working set and
// leaves only clean lines behind (a memset flush would leave dirty lines whose
// write-back the timed kernel would pay); kernel-replay timing
__global__ void k_l2_sweep(const double* a, long long n, double* sink) {
    double acc = 0.0;
    for (long long i = 2 * (blockIdx.x * (long long)blockDim.x + threadIdx.x); i + 1 < n;
         i += 2LL * gridDim.x * blockDim.x) {
        const double2 v = __ldcg(reinterpret_cast<const double2*>(a + i));  // L2-allocating (not evict-first)
        acc += v.x + v.y;
    }
    if (acc == -1.0) *sink = acc;  // keeps the loads; never true for the 0 / 1 fill
}

cudaError_t launch_l2_sweep(const double* a, long long n, double* sink, cudaStream_t s) {
    k_l2_sweep<<<148 * 8, 256, 0, s>>>(a, n, sink);
    return cudaGetLastError();
}

cudaError_t launch_fill_test(double* a, long long n, cudaStream_t s) {
    k_fill_test<<<148 * 8, 256, 0, s>>>(a, n);
    return cudaGetLastError();
}

// --------------------------------------------------------------------------
// launchers
// --------------------------------------------------------------------------
cudaError_t launch_pole_avg(const Geo& g, int ncomp, double* y, double* dinv, int plane_lo, int nplanes,
                            cudaStream_t s) {
    if (nplanes <= 0) return cudaSuccess;
    k_pole_avg<<<2 * ncomp * nplanes, kThreads, 0, s>>>(g, y, dinv, plane_lo, nplanes);
    return cudaGetLastError();
}

cudaError_t launch_init_dots(const Geo& g, int ncomp, const double* f, const double* r, const double* dinv,
                             Scratch scr, PcgState* st, int nblocks, cudaStream_t s) {
    k_init_dots<<<nblocks, kThreads, 0, s>>>(g, ncomp, f, r, dinv, scr, st);
    return cudaGetLastError();
}
cudaError_t launch_radial_sums(const Geo& g, int ncomp, const double* x, const double* w, double* out,
                               cudaStream_t s) {
    const int blocks = ncomp * g.nl;
    if (blocks <= 0) return cudaErrorInvalidValue;
    k_radial_sums<<<blocks, kThreads, 0, s>>>(g, x, w, out);
    return cudaGetLastError();
}

int stencil_blocks(const Geo& g, int chunk) {
    const int ntj = (g.nt + TJ - 1) / TJ, ntk = (g.np + TK - 1) / TK;
    const int nch = (g.nl + chunk - 1) / chunk;
    return ntj * ntk * nch;
}

template <int MODE, int NC, bool FIRSTK = false, bool LPAR = false>
static cudaError_t launch_one(const StencilArgs& a0, cudaStream_t s) {
    StencilArgs a = a0;
    a.ntj = (a.g.nt + TJ - 1) / TJ;
    a.ntk = (a.g.np + TK - 1) / TK;
    a.nchunk = (a.g.nl + a.chunk - 1) / a.chunk;
    const int smem = (4 * (NC + 1) * HROWS * ROW + (LPAR ? kLparSmem : 0)) * (int)sizeof(double);
    static DeviceOnce attr;
    cudaError_t e = attr.run([&] {
        return cudaFuncSetAttribute(k_stencil<MODE, NC, FIRSTK, LPAR>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                    smem);
    });
    if (e != cudaSuccess) return e;
    const int T = a.ntj * a.ntk;
    const int blocks = a.part == 1 ? T * (a.nchunk - 2) : a.part == 2 ? 2 * T : T * a.nchunk;
    if (blocks <= 0) return cudaErrorInvalidValue;
    k_stencil<MODE, NC, FIRSTK, LPAR><<<blocks, kSThreads, smem, s>>>(a);
    return cudaGetLastError();
}

cudaError_t launch_stencil(int mode, int ncomp, const StencilArgs& a, cudaStream_t s, bool first) {
    if (ncomp == 1) {
        if (mode == MODE_APPLY) return launch_one<MODE_APPLY, 1>(a, s);
        if (mode == MODE_RESID) return launch_one<MODE_RESID, 1>(a, s);
        if (mode == MODE_CG1) return first ? launch_one<MODE_CG1, 1, true>(a, s) : launch_one<MODE_CG1, 1>(a, s);
        if (a.ca)  // the field-aligned term fused into kernel A
            return first ? launch_one<MODE_PCGA, 1, true, true>(a, s) : launch_one<MODE_PCGA, 1, false, true>(a, s);
        return first ? launch_one<MODE_PCGA, 1, true>(a, s) : launch_one<MODE_PCGA, 1>(a, s);
    }
    if (ncomp == 3) {
        if (mode == MODE_APPLY) return launch_one<MODE_APPLY, 3>(a, s);
        if (mode == MODE_RESID) return launch_one<MODE_RESID, 3>(a, s);
        if (mode == MODE_CG1) return first ? launch_one<MODE_CG1, 3, true>(a, s) : launch_one<MODE_CG1, 3>(a, s);
        return first ? launch_one<MODE_PCGA, 3, true>(a, s) : launch_one<MODE_PCGA, 3>(a, s);
    }
    return cudaErrorInvalidValue;
}

// the per-block partial sums of a stacked solve (mas_stack_solve) into their
// sum, written back to every block's PcgState: the "allreduce" over the blocks
// of the stacked vector (R34).  Offsets in doubles: 0 sigma;
// 1..3 rho, rr, ff (PcgState layout)
__global__ void k_stack_sum(const StackStates s, int off, int cnt) {
    const int t = threadIdx.x;
    if (t >= cnt) return;
    double v = 0.0;
    for (int m = 0; m < s.n; m++) v += __ldcg(reinterpret_cast<const double*>(s.st[m]) + off + t);
    for (int m = 0; m < s.n; m++) reinterpret_cast<double*>(s.st[m])[off + t] = v;
}

cudaError_t launch_stack_sum(const StackStates& s, int off, int cnt, cudaStream_t stream) {
    if (s.n < 1 || s.n > kMaxStack || cnt < 1 || cnt > 32) return cudaErrorInvalidValue;
    k_stack_sum<<<1, 32, 0, stream>>>(s, off, cnt);
    return cudaGetLastError();
}

cudaError_t launch_pcg_b(const StreamArgs& a, int nblocks, cudaStream_t s) {
    if (a.ncomp == 1 && a.tnode)
        k_pcg_b<1, true><<<nblocks, kThreads, 0, s>>>(a);
    else if (a.ncomp == 3 && a.tnode)
        k_pcg_b<3, true><<<nblocks, kThreads, 0, s>>>(a);
    else if (a.ncomp == 1)
        k_pcg_b<1><<<nblocks, kThreads, 0, s>>>(a);
    else if (a.ncomp == 3)
        k_pcg_b<3><<<nblocks, kThreads, 0, s>>>(a);
    else
        return cudaErrorInvalidValue;
    return cudaGetLastError();
}

cudaError_t launch_diag(const Geo& g, Halo kappa, TRows tkappa, const double* c, double* D,
                        double* dinv, int* bad, cudaStream_t s) {
    const long long Nl = (long long)g.nl * g.plane;
    const int blocks = (int)std::min<long long>((Nl + kThreads - 1) / kThreads, 148LL * 16);
    k_diag<<<blocks, kThreads, 0, s>>>(g, kappa, tkappa, c, D, dinv, bad);
    return cudaGetLastError();
}

// first / last theta rows of every plane of a field, packed [2][ncomp][nl][np]
__global__ void k_pack_rows(const Geo g, int ncomp, const double* in, double* out) {
    const long long n = (long long)ncomp * g.nl * g.np;  // per side
    for (long long t = blockIdx.x * (long long)blockDim.x + threadIdx.x; t < 2 * n;
         t += (long long)gridDim.x * blockDim.x) {
        const int side = t >= n;
        const long long u = t - side * n;
        const long long ci = u / g.np;  // comp * nl + i
        const int k = (int)(u - ci * g.np);
        const int j = side ? g.nt - 1 : 0;
        out[t] = in[ci * g.plane + (long long)j * g.np + k];
    }
}

cudaError_t launch_pack_rows(const Geo& g, int ncomp, const double* in, double* out, cudaStream_t s) {
    const long long n = 2LL * ncomp * g.nl * g.np;
    const int blocks = (int)std::min<long long>((n + 255) / 256, 148LL * 8);
    k_pack_rows<<<blocks, 256, 0, s>>>(g, ncomp, in, out);
    return cudaGetLastError();
}

cudaError_t launch_dirichlet(const Geo& g, int ncomp, const double* kappa, const double* ub, int outer,
                             double* f, cudaStream_t s) {
    const long long n = g.plane * ncomp;
    const int blocks = (int)std::min<long long>((n + 255) / 256, 148LL * 8);
    k_dirichlet<<<blocks, 256, 0, s>>>(g, ncomp, kappa, ub, outer, f);
    return cudaGetLastError();
}

__global__ void k_rank_sum(double* out, const double* stage, int nranks, int n) {
    const int t = threadIdx.x;
    if (t < n) {
        double s = 0.0;
        for (int r = 0; r < nranks; r++) s += stage[8 * r + t];
        out[t] = s;
    }
}

cudaError_t launch_rank_sum(double* out, const double* stage, int nranks, int n, cudaStream_t s) {
    k_rank_sum<<<1, 32, 0, s>>>(out, stage, nranks, n);
    return cudaGetLastError();
}

cudaError_t launch_dot(const Geo& g, int ncomp, const double* a, const double* b, Scratch scr,
                       double* out, int nblocks, cudaStream_t s) {
    k_dot<<<nblocks, kThreads, 0, s>>>(g, ncomp, a, b, scr, out);
    return cudaGetLastError();
}

}  // namespace mas
