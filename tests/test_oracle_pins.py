"""Pins for the ORACLE (oracle/mas_ref.c) against what mathematics fixes.

The paper (Caplan et al. 2023) prints no formula or value for this path
(SURVEY.md §0, §8(c)), so the oracle is pinned by closed forms, invariants,
special cases reducing to library routines, and brute force on tiny grids —
chosen so that a dropped term, a wrong sign/index or a transposed metric
factor fails at least one of them (DESIGN.md §3.3 maps each pin to the
mistakes it catches).  None of these tests retype the oracle's face formula.
"""
import math

import numpy as np
import pytest
import scipy.linalg
import scipy.sparse.linalg

from paper_conf_ipps_caplansl23_b200 import workloads as W


def tiny_mesh(nr=3, nt=4, np_=6, r0=1.0, r1=2.0, R=3.0):
    return W.stretched_mesh(nr, nt, np_, r0, r1, R)


def rand_coeffs(shape, seed):
    rng = np.random.default_rng(seed)
    kappa = rng.uniform(0.5, 2.0, size=shape)
    c = rng.uniform(0.1, 1.0, size=shape)
    return kappa, c


def dense_matrix(o, kappa, c, ncomp=1):
    n = o.N * ncomp
    A = np.empty((n, n))
    e = np.zeros(n)
    for col in range(n):
        e[:] = 0.0
        e[col] = 1.0
        A[:, col] = o.apply(kappa, c, e.reshape((ncomp,) + o.shape)).ravel()
    return A


# ---------------------------------------------------------------------------
# metrics: closed forms
# ---------------------------------------------------------------------------
def test_volume_sum_converges_to_shell_volume(oracle_mod):
    """sum_P V_P -> (4 pi/3)(r1^3 - r0^3) at O(h^2) (midpoint metrics, R4);
    theta factor sum_j sin(tC) dt -> 2."""
    exact = 4.0 * math.pi / 3.0 * (2.0 ** 3 - 1.0)
    errs = []
    for n in (8, 16, 32):
        m = W.stretched_mesh(n, 2 * n, 2 * n, 1.0, 2.0, 3.0)
        o = oracle_mod.Oracle(m, W.DIRICHLET, W.DIRICHLET)
        errs.append(abs(o.volumes().sum() - exact) / exact)
    assert errs[-1] < 2e-3
    orders = [math.log2(errs[i] / errs[i + 1]) for i in range(2)]
    assert min(orders) > 1.8, (errs, orders)


def test_volumes_positive_and_separable(oracle_mod):
    m = tiny_mesh(4, 6, 8)
    V = oracle_mod.Oracle(m, 0, 1).volumes()
    assert (V > 0).all()
    # uniform phi: volumes are phi-independent up to rounding of dp
    assert np.allclose(V, V[:, :, :1], rtol=1e-13, atol=0)
    # north/south symmetric theta mesh => V(j) = V(nt-1-j)
    assert np.allclose(V, V[:, ::-1, :], rtol=1e-12, atol=0)


# ---------------------------------------------------------------------------
# operator: constants, symmetry, definiteness, conservation
# ---------------------------------------------------------------------------
def test_L_of_constant_is_c_bitwise_neumann(oracle_mod):
    """Neumann-Neumann: every u_P - u_N is exactly 0, so L 1 == c bitwise."""
    m = W.stretched_mesh(6, 8, 10)
    o = oracle_mod.Oracle(m, W.NEUMANN, W.NEUMANN)
    kappa, c = rand_coeffs(o.shape, 3)
    y = o.apply(kappa, c, np.ones((1,) + o.shape))
    assert np.array_equal(y[0], c)


def test_L_of_constant_dirichlet_only_boundary_planes(oracle_mod):
    """With Dirichlet r-faces L 1 - c is zero (bitwise) off the boundary planes,
    positive on them, and equals the Dirichlet-rhs helper with u_b = 1."""
    m = W.stretched_mesh(6, 8, 10)
    o = oracle_mod.Oracle(m, W.DIRICHLET, W.DIRICHLET)
    kappa, c = rand_coeffs(o.shape, 4)
    y = o.apply(kappa, c, np.ones((1,) + o.shape))[0] - c
    assert np.array_equal(y[1:-1], np.zeros_like(y[1:-1]))
    assert (y[0] > 0).all() and (y[-1] > 0).all()
    ones = np.ones((1,) + o.shape[1:])
    b = o.dirichlet_rhs(kappa, np.zeros((1,) + o.shape), ones, ones)[0]
    np.testing.assert_allclose(y, b, rtol=1e-14, atol=0)


@pytest.mark.parametrize("bc", [(0, 0), (0, 1), (1, 1)])
@pytest.mark.parametrize("shape", [(3, 4, 6), (5, 7, 8), (12, 16, 20)])
def test_symmetry_in_V_inner_product(oracle_mod, bc, shape):
    """<L u, w>_V == <u, L w>_V (R9): catches any one-sided conductance."""
    m = W.stretched_mesh(*shape)
    o = oracle_mod.Oracle(m, *bc)
    kappa, c = rand_coeffs(shape, 5)
    rng = np.random.default_rng(6)
    u = rng.standard_normal((1,) + shape)
    w = rng.standard_normal((1,) + shape)
    Lu, Lw = o.apply(kappa, c, u), o.apply(kappa, c, w)
    lhs, rhs = o.dot(Lu, w), o.dot(u, Lw)
    scale = math.sqrt(o.dot(Lu, Lu) * o.dot(w, w))
    assert abs(lhs - rhs) <= 1e-14 * scale


@pytest.mark.parametrize("shape", [(3, 4, 6), (4, 6, 8)])
@pytest.mark.parametrize("bc", [(0, 1), (0, 0)])
def test_dense_VL_symmetric_and_positive_definite(oracle_mod, shape, bc):
    m = W.stretched_mesh(*shape)
    o = oracle_mod.Oracle(m, *bc)
    kappa, c = rand_coeffs(shape, 7)
    A = dense_matrix(o, kappa, c)
    V = o.volumes().ravel()
    VA = V[:, None] * A
    assert np.abs(VA - VA.T).max() <= 1e-15 * np.abs(VA).max() * 10
    S = np.sqrt(V)[:, None] * A / np.sqrt(V)[None, :]
    ev = np.linalg.eigvalsh(0.5 * (S + S.T))
    assert ev.min() > 0
    # kappa > 0, c = 0, Neumann-Neumann: exactly one zero mode (the constant)
    o2 = oracle_mod.Oracle(m, 1, 1)
    A2 = dense_matrix(o2, kappa, np.zeros(shape))
    S2 = np.sqrt(V)[:, None] * A2 / np.sqrt(V)[None, :]
    ev2 = np.linalg.eigvalsh(0.5 * (S2 + S2.T))
    assert abs(ev2[0]) < 1e-12 * ev2[-1] and ev2[1] > 1e-8 * ev2[-1]


def test_flux_sum_conservation(oracle_mod):
    """sum_P V_P (L u - c u)_P = 0 for Neumann-Neumann (interior fluxes
    telescope); with Dirichlet it equals the boundary conductance sum."""
    shape = (8, 10, 12)
    m = W.stretched_mesh(*shape)
    kappa, c = rand_coeffs(shape, 8)
    u = np.random.default_rng(9).standard_normal((1,) + shape)
    o = oracle_mod.Oracle(m, 1, 1)
    V = o.volumes()
    terms = V * (o.apply(kappa, c, u)[0] - c * u[0])
    assert abs(terms.sum()) <= 1e-13 * np.abs(terms).sum()
    od = oracle_mod.Oracle(m, 0, 0)
    terms = V * (od.apply(kappa, c, u)[0] - c * u[0])
    # boundary term: G_b u_P summed over both Dirichlet faces == V * rhs helper
    # with u_b = u on the boundary planes
    b = od.dirichlet_rhs(kappa, np.zeros((1,) + shape), u[:, 0], u[:, -1])[0]
    assert abs(terms.sum() - (V * b).sum()) <= 1e-13 * np.abs(terms).sum()


def test_phi_shift_equivariance(oracle_mod):
    shape = (5, 6, 16)
    m = W.stretched_mesh(*shape)
    o = oracle_mod.Oracle(m, 0, 1)
    rng = np.random.default_rng(10)
    kappa = np.broadcast_to(rng.uniform(0.5, 2, size=shape[:2])[:, :, None], shape).copy()
    c = np.broadcast_to(rng.uniform(0.1, 1, size=shape[:2])[:, :, None], shape).copy()
    u = rng.standard_normal((1,) + shape)
    for s in (1, 5):
        a = o.apply(kappa, c, np.roll(u, s, axis=-1))
        b = np.roll(o.apply(kappa, c, u), s, axis=-1)
        np.testing.assert_allclose(a, b, rtol=0, atol=1e-13 * np.abs(b).max())


@pytest.mark.parametrize("mode", [1, 3, 7])
def test_phi_fourier_eigenrelation(oracle_mod, mode):
    """u = cos(m phi) with phi-independent kappa: the r and theta differences
    vanish exactly, and the periodic phi part is the discrete eigenvalue
    kappa * 2(1 - cos m dphi) / (rC^2 sin^2(tC) dphi^2) (closed form)."""
    shape = (4, 6, 24)
    m = W.stretched_mesh(*shape)
    o = oracle_mod.Oracle(m, 1, 1)
    kap = np.random.default_rng(11).uniform(0.5, 2, size=shape[:2])
    kappa = np.broadcast_to(kap[:, :, None], shape).copy()
    c = np.zeros(shape)
    u = np.broadcast_to(np.cos(mode * m.pC)[None, None, :], shape)[None].copy()
    dphi = 2 * math.pi / shape[2]
    lam = (kappa * 2 * (1 - math.cos(mode * dphi))
           / (m.rC[:, None, None] ** 2 * np.sin(m.tC)[None, :, None] ** 2 * dphi ** 2))
    np.testing.assert_allclose(o.apply(kappa, c, u)[0], lam * u[0], rtol=0,
                               atol=1e-13 * np.abs(lam).max())


def test_theta_only_operator_is_legendre_like(oracle_mod):
    """u = cos(theta) (the l = 1 harmonic), kappa = 1: the continuum value of
    -div grad u is 2 cos(theta)/r^2.  On a fine uniform theta mesh the
    discrete operator converges to it at O(h^2) away from and AT the poles
    (pole faces carry no flux, R5)."""
    errs = []
    for nt in (32, 64, 128):
        m = W.stretched_mesh(1, nt, 4, 1.0, 1.001, 1.0, a=0.0)
        o = oracle_mod.Oracle(m, 1, 1)
        shape = o.shape
        u = np.broadcast_to(np.cos(m.tC)[None, :, None], shape)[None].copy()
        y = o.apply(np.ones(shape), np.zeros(shape), u)[0]
        exact = 2 * np.cos(m.tC)[None, :, None] / m.rC[:, None, None] ** 2
        V = o.volumes()
        errs.append(math.sqrt((V * (y - exact) ** 2).sum() / V.sum()))
    orders = [math.log2(errs[i] / errs[i + 1]) for i in range(2)]
    assert min(orders) > 1.4, (errs, orders)


# ---------------------------------------------------------------------------
# discretisation: manufactured solution (closed form, sympy-checked forcing)
# ---------------------------------------------------------------------------
def test_mms_forcing_closed_form_matches_sympy():
    sp = pytest.importorskip("sympy")
    r, t, p = sp.symbols("r t p", positive=True)
    u = sp.exp(-r) * (1 + sp.sin(t) ** 2 * sp.cos(2 * p) + sp.sin(t) * sp.sin(p) / 2)
    k = r ** 2
    div = (sp.diff(r ** 2 * k * sp.diff(u, r), r) / r ** 2
           + sp.diff(sp.sin(t) * k * sp.diff(u, t), t) / (r ** 2 * sp.sin(t))
           + sp.diff(k * sp.diff(u, p), p) / (r ** 2 * sp.sin(t) ** 2))
    f = sp.lambdify((r, t, p), -div, "numpy")
    rng = np.random.default_rng(0)
    pts = rng.uniform([1, 0.1, 0], [2, 3.0, 6.2], size=(50, 3)).T
    np.testing.assert_allclose(W.mms_forcing(*pts), f(*pts), rtol=1e-12, atol=1e-14)


def test_mms_second_order_and_c1_iterations(oracle_mod):
    """C1 problem: RMS_V error vs u* at O(h^2); survey-time SciPy prototype
    (independent code) saw 1.475e-3 / 3.544e-4 / 8.700e-5 and 63/134/299
    Jacobi-PCG iterations at tol 1e-12 (scipy's strict <)."""
    errs, its = [], []
    for (nr, nt, np_) in ((8, 12, 16), (16, 24, 32), (32, 48, 64)):
        prob = W.mms_problem(nr, nt, np_)
        rc, x, it, rel, hist = oracle_mod.solve_problem(prob)
        assert rc == oracle_mod.OK and rel <= 1e-12
        o = oracle_mod.Oracle.for_problem(prob)
        V = o.volumes()
        e = x[0] - prob.extra["exact"][0]
        errs.append(math.sqrt((V * e * e).sum() / V.sum()))
        its.append(it)
    np.testing.assert_allclose(errs, [1.475e-3, 3.544e-4, 8.700e-5], rtol=0.01)
    orders = [math.log2(errs[i] / errs[i + 1]) for i in range(2)]
    assert min(orders) > 1.8
    for got, want in zip(its, (63, 134, 299)):
        assert abs(got - want) <= 2, its


# ---------------------------------------------------------------------------
# solver: brute force, library routines, special cases
# ---------------------------------------------------------------------------
@pytest.mark.parametrize("bc", [(0, 1), (0, 0)])
def test_pcg_matches_dense_solve(oracle_mod, bc):
    shape = (4, 6, 8)
    m = W.stretched_mesh(*shape)
    o = oracle_mod.Oracle(m, *bc)
    kappa, c = rand_coeffs(shape, 12)
    A = dense_matrix(o, kappa, c)
    f = np.random.default_rng(13).standard_normal((1,) + shape)
    xd = np.linalg.solve(A, f.ravel())
    rc, x, it, rel, hist = o.pcg(kappa, c, f, np.zeros_like(f), 1e-13, 1000)
    assert rc == oracle_mod.OK
    assert it <= A.shape[0] + 10
    V = o.volumes().ravel()
    err = math.sqrt((V * (x.ravel() - xd) ** 2).sum() / (V * xd ** 2).sum())
    assert err <= 1e-10


def test_pcg_matches_scipy_cg(oracle_mod):
    """Same system through scipy.sparse.linalg.cg on V^1/2 L V^-1/2 with the
    Jacobi preconditioner: iteration count within 1 and x within 1e-10."""
    shape = (6, 8, 10)
    m = W.stretched_mesh(*shape)
    o = oracle_mod.Oracle(m, 0, 1)
    kappa, c = rand_coeffs(shape, 14)
    kappa *= 50.0  # make it take a few dozen iterations
    A = dense_matrix(o, kappa, c)
    V = o.volumes().ravel()
    s = np.sqrt(V)
    S = s[:, None] * A / s[None, :]
    S = 0.5 * (S + S.T)
    f = np.random.default_rng(15).standard_normal((1,) + shape)
    Dg = np.diag(A)
    count = [0]
    y, info = scipy.sparse.linalg.cg(S, s * f.ravel(), rtol=1e-12, atol=0.0, maxiter=1000,
                                     M=scipy.sparse.diags(1.0 / Dg),
                                     callback=lambda _: count.__setitem__(0, count[0] + 1))
    assert info == 0
    rc, x, it, rel, hist = o.pcg(kappa, c, f, np.zeros_like(f), 1e-12, 1000)
    assert rc == oracle_mod.OK
    assert abs(it - count[0]) <= 1
    xs = y / s
    err = math.sqrt((V * (x.ravel() - xs) ** 2).sum() / (V * xs ** 2).sum())
    assert err <= 1e-10
    # the Jacobi diagonal equals the assembled diagonal
    np.testing.assert_allclose(o.diag(kappa, c).ravel(), Dg, rtol=1e-14, atol=0)


def test_mass_only_converges_in_one_iteration(oracle_mod):
    """kappa == 0: L = diag(c) = D, the Jacobi-preconditioned system is the
    identity, so PCG stops after exactly 1 iteration with x = f/c."""
    shape = (4, 5, 6)
    m = W.stretched_mesh(*shape)
    o = oracle_mod.Oracle(m, 0, 1)
    c = np.random.default_rng(16).uniform(0.1, 3, size=shape)
    f = np.random.default_rng(17).standard_normal((2,) + shape)
    rc, x, it, rel, hist = o.pcg(np.zeros(shape), c, f, np.zeros_like(f), 1e-12, 50)
    assert rc == oracle_mod.OK and it == 1
    np.testing.assert_allclose(x, f / c[None], rtol=4e-16, atol=0)


def test_zero_rhs_and_exact_start(oracle_mod):
    shape = (3, 4, 6)
    m = W.stretched_mesh(*shape)
    o = oracle_mod.Oracle(m, 0, 1)
    kappa, c = rand_coeffs(shape, 18)
    x0 = np.ones((1,) + shape)
    rc, x, it, rel, hist = o.pcg(kappa, c, np.zeros_like(x0), x0, 1e-12, 10)
    assert rc == oracle_mod.OK and it == 0 and (x == 0).all()
    # x0 already the solution: stops at k = 0
    f = o.apply(kappa, c, x0)
    rc, x, it, rel, hist = o.pcg(kappa, c, f, x0, 1e-12, 10)
    assert rc == oracle_mod.OK and it == 0 and np.array_equal(x, x0)


def test_radial_problem_reduces_to_tridiagonal(oracle_mod):
    """r-only kappa, c, f: theta/phi differences vanish exactly, the solution
    is r-only and equals the direct banded solve of the 1-D operator read off
    the oracle's own action on r-only vectors (columns of a 1-D matrix)."""
    nr, nt, np_ = 10, 6, 8
    m = W.stretched_mesh(nr, nt, np_, 1.0, 3.0, 5.0)
    o = oracle_mod.Oracle(m, 0, 1)
    rng = np.random.default_rng(19)
    kr = rng.uniform(0.5, 2, nr)
    cr = rng.uniform(0.1, 1, nr)
    fr = rng.standard_normal(nr)
    B = lambda a: np.broadcast_to(a[:, None, None], (nr, nt, np_)).copy()
    kappa, c, f = B(kr), B(cr), B(fr)[None]
    # 1-D matrix from r-only unit vectors; it must be tridiagonal
    A = np.zeros((nr, nr))
    for i in range(nr):
        e = np.zeros(nr)
        e[i] = 1
        y = o.apply(kappa, c, B(e)[None])[0]
        assert np.allclose(y, y[:, :1, :1], rtol=1e-13, atol=1e-13 * np.abs(y).max())
        A[:, i] = y[:, 0, 0]
    assert np.abs(np.triu(A, 2)).max() == 0 and np.abs(np.tril(A, -2)).max() == 0
    ab = np.zeros((3, nr))
    ab[0, 1:] = np.diag(A, 1)
    ab[1] = np.diag(A)
    ab[2, :-1] = np.diag(A, -1)
    xr = scipy.linalg.solve_banded((1, 1), ab, fr)
    rc, x, it, rel, hist = o.pcg(kappa, c, f, np.zeros_like(f), 1e-14, 500)
    assert rc == oracle_mod.OK
    np.testing.assert_allclose(x[0], B(xr), rtol=1e-11, atol=1e-11 * np.abs(xr).max())


# ---------------------------------------------------------------------------
# decomposition: virtual r-slabs == monolithic
# ---------------------------------------------------------------------------
@pytest.mark.parametrize("P", [2, 3, 4, 8])
def test_slab_apply_bitwise_and_vranks_pcg(oracle_mod, P):
    shape = (9, 6, 8)
    m = W.stretched_mesh(*shape)
    o = oracle_mod.Oracle(m, 0, 1)
    kappa, c = rand_coeffs(shape, 20)
    x = np.random.default_rng(21).standard_normal((3,) + shape)
    y = o.apply(kappa, c, x)
    plane = shape[1] * shape[2]
    for rank in range(P):
        i0, nl = oracle_mod.partition(shape[0], P, rank)
        lo, hi = max(i0 - 1, 0), min(i0 + nl + 1, shape[0])
        kext = np.zeros((nl + 2,) + shape[1:])
        xext = np.zeros((3, nl + 2) + shape[1:])
        kext[lo - (i0 - 1): hi - (i0 - 1)] = kappa[lo:hi]
        xext[:, lo - (i0 - 1): hi - (i0 - 1)] = x[:, lo:hi]
        ys = o.apply_slab(i0, nl, kext, c[i0:i0 + nl], xext)
        assert np.array_equal(ys, y[:, i0:i0 + nl])
    prob_f = y  # any rhs
    rc1, x1, it1, _, _ = o.pcg(kappa * 30, c, prob_f, np.zeros_like(x), 1e-12, 500)
    rcP, xP, itP, _, _ = o.pcg(kappa * 30, c, prob_f, np.zeros_like(x), 1e-12, 500, nranks=P)
    assert rc1 == rcP == oracle_mod.OK
    assert abs(it1 - itP) <= 1
    V = o.volumes()
    err = math.sqrt((V * (x1 - xP) ** 2).sum() / (V * x1 ** 2).sum())
    assert err <= 1e-10


def test_partition_tiles_the_r_range(oracle_mod):
    for nr in (1, 7, 256, 320):
        for P in range(1, min(nr, 9) + 1):
            parts = [oracle_mod.partition(nr, P, p) for p in range(P)]
            assert parts[0][0] == 0
            for (a, n), (b, _) in zip(parts, parts[1:]):
                assert a + n == b
            assert parts[-1][0] + parts[-1][1] == nr
            assert max(n for _, n in parts) - min(n for _, n in parts) <= 1


# ---------------------------------------------------------------------------
# decomposition: (r, theta) blocks == monolithic (NEXT-3)
# ---------------------------------------------------------------------------
def block_ext(a, i0, nl, j0, ntl):
    """[.., nl+2, ntl+2, np] copy of a block with one ghost plane / row per
    side from the global array (zeros beyond the global index range)."""
    nr, nt = a.shape[-3], a.shape[-2]
    ext = np.zeros(a.shape[:-3] + (nl + 2, ntl + 2, a.shape[-1]))
    ilo, ihi = max(i0 - 1, 0), min(i0 + nl + 1, nr)
    jlo, jhi = max(j0 - 1, 0), min(j0 + ntl + 1, nt)
    ext[..., ilo - (i0 - 1):ihi - (i0 - 1), jlo - (j0 - 1):jhi - (j0 - 1), :] = \
        a[..., ilo:ihi, jlo:jhi, :]
    return ext


@pytest.mark.parametrize("pr,pt", [(1, 2), (2, 2), (3, 3), (1, 6)])
@pytest.mark.parametrize("bc", [(0, 1), (1, 1)])
def test_block_apply_bitwise(oracle_mod, pr, pt, bc):
    shape = (9, 13, 8)
    m = W.stretched_mesh(*shape)
    o = oracle_mod.Oracle(m, *bc)
    kappa, c = rand_coeffs(shape, 22)
    x = np.random.default_rng(23).standard_normal((3,) + shape)
    y = o.apply(kappa, c, x)
    dots = []
    for rr in range(pr):
        i0, nl = oracle_mod.partition(shape[0], pr, rr)
        for rt in range(pt):
            j0, ntl = oracle_mod.partition(shape[1], pt, rt)
            yb = o.apply_block(i0, nl, j0, ntl, block_ext(kappa, i0, nl, j0, ntl),
                               c[i0:i0 + nl, j0:j0 + ntl], block_ext(x, i0, nl, j0, ntl))
            assert np.array_equal(yb, y[:, i0:i0 + nl, j0:j0 + ntl])
            xb = np.ascontiguousarray(x[:, i0:i0 + nl, j0:j0 + ntl])
            dots.append(o.dot_block(i0, nl, j0, ntl, xb, xb))
    assert abs(sum(dots) - o.dot(x, x)) <= 1e-14 * o.dot(x, x)


# ---------------------------------------------------------------------------
# per-cell sampler (the full-size C2/C3 checker) == the whole-field operator
# ---------------------------------------------------------------------------
def _boundary_class_indices(shape, ncomp, rng, n_random):
    """Flat comp-major indices m*N + P covering every boundary class: the r
    boundary planes (i = 0, nr-1), the pole rows (j = 0, nt-1), the phi wrap
    columns (k = 0, np-1), the GPU tile and chunk edges (j = 7, 8, 15, 16;
    k = 63, 64, 127, 128; i = 31, 32), all their combinations (corners), for
    every component, plus n_random uniform cells."""
    nr, nt, np_ = shape
    N = nr * nt * np_

    def cand(n, edges):
        return sorted({e for e in (0, 1, n - 2, n - 1, *edges) if 0 <= e < n})

    I = cand(nr, (31, 32, 33))
    J = cand(nt, (7, 8, 15, 16))
    K = cand(np_, (63, 64, 127, 128))
    idx = [m * N + (i * nt + j) * np_ + k for m in range(ncomp) for i in I for j in J for k in K]
    idx += list(rng.integers(0, ncomp * N, size=n_random))
    return np.unique(np.asarray(idx, dtype=np.int64))


@pytest.mark.parametrize("shape,ncomp,bc", [
    ((5, 6, 8), 3, (0, 1)),          # every cell of a tiny grid, all 3 components
    ((40, 20, 132), 1, (0, 0)),      # ragged tile/chunk edges, Dirichlet both ends
    ((34, 18, 130), 3, (1, 1)),      # Neumann both ends, 3 components
    ((33, 17, 66), 3, (0, 1)),       # odd nr / nt
])
def test_apply_cells_equals_apply_bitwise(oracle_mod, shape, ncomp, bc):
    """mas_ref_op_apply_cells re-decodes flat indices (m, i, j, k) on its own;
    it must return exactly the values of the whole-field mas_ref_op_apply
    (itself pinned above) at every sampled cell, boundary classes included.
    An index-decoding slip (i/j swapped, component offset, phi wrap) fails."""
    m = W.stretched_mesh(*shape)
    o = oracle_mod.Oracle(m, *bc)
    kappa, c = rand_coeffs(shape, 11)
    rng = np.random.default_rng(12)
    x = rng.uniform(-1.0, 1.0, size=(ncomp,) + shape)
    y = o.apply(kappa, c, x).ravel()
    N = o.N
    if ncomp * N <= 4096:
        idx = np.arange(ncomp * N, dtype=np.int64)
    else:
        idx = _boundary_class_indices(shape, ncomp, rng, 2000)
    assert idx.size >= min(ncomp * N, 2000)
    got = o.apply_cells(kappa, c, x, idx)
    assert np.array_equal(got, y[idx]), np.abs(got - y[idx]).max()
    # and with no mass term (c = NULL), as the full-size tests may pass
    y0 = o.apply(kappa, np.zeros(shape), x).ravel()
    assert np.array_equal(o.apply_cells(kappa, None, x, idx), y0[idx])
