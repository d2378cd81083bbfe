"""Pins for the oracle's theta-node placement with pole unknowns
(mas_ref_tn_*, readings R29-R30 in DESIGN.md §3.5).

The paper prints only that the grid is staggered and that MAS
sums arrays per radius (Listings 3-5); the operator is pinned by
what mathematics fixes:
* metrics: the slots' volumes (interior rows + polar-cap slices) sum to the
  shell volume at O(h^2);
* constants and conservation: L 1 = c bitwise on interior rows (and to
  rounding on the pole rows), sum_P V (L u - c u) = 0 for Neumann-Neumann;
* the pole is one point: pole rows of L u are phi-constant bitwise;
* symmetry / definiteness of the reduced operator (pole = one unknown per
  radius) under the V-weighted inner product, one zero mode for c = 0 NN;
* closed forms through the pole: L cos(theta) = 2 cos(theta) / r^2 at
  O(h^2) on every row including both poles; an MMS with a Cartesian-smooth
  u* (cos theta, sin^2 theta cos 2 phi, sin theta sin phi terms) with the
  sympy-checked forcing, second order in L2_V and in max norm incl. poles;
* the Dirichlet-rhs helper equals L 1 - c on the boundary planes;
* PCG on it equals the dense solve of the reduced system; kappa = 0 takes
  exactly one iteration."""
import math

import numpy as np
import pytest

from paper_conf_ipps_caplansl23_b200 import workloads as W


def mesh(nr, nt, np_, r0=1.0, r1=2.0, R=3.0):
    return W.stretched_mesh(nr, nt, np_, r0, r1, R)


def replicate_poles(a):
    a = np.array(a, dtype=np.float64)
    a[..., 0, :] = a[..., 0, :1]
    a[..., -1, :] = a[..., -1, :1]
    return a


def rand_coeffs(shape, seed):
    rng = np.random.default_rng(seed)
    return rng.uniform(0.5, 2.0, size=shape), rng.uniform(0.1, 1.0, size=shape)


def test_tn_volumes_converge_to_shell(oracle_mod):
    exact = 4.0 * math.pi / 3.0 * 7.0
    errs = []
    for n in (8, 16, 32):
        o = oracle_mod.Oracle(mesh(n, 2 * n, 2 * n), 1, 1)
        errs.append(abs(o.tn_volumes().sum() - exact) / exact)
    orders = [math.log2(errs[i] / errs[i + 1]) for i in range(2)]
    assert errs[-1] < 1e-3 and min(orders) > 1.8, (errs, orders)


def test_tn_constant_and_replication(oracle_mod):
    o = oracle_mod.Oracle(mesh(6, 8, 12), 1, 1)
    kappa, c = rand_coeffs(o.tn_shape, 3)
    c = replicate_poles(c)
    y = o.tn_apply(kappa, c, np.ones((1,) + o.tn_shape))[0]
    assert np.array_equal(y[:, 1:-1], c[:, 1:-1])  # interior rows: bitwise
    np.testing.assert_allclose(y[:, [0, -1]], c[:, [0, -1]], rtol=4e-16, atol=0)
    # pole rows of L u are phi-constant (the pole is one point), for any u
    # with phi-constant pole rows, kappa and c arbitrary per slot
    kappa, c = rand_coeffs(o.tn_shape, 4)
    u = replicate_poles(np.random.default_rng(5).standard_normal((3,) + o.tn_shape))
    y = o.tn_apply(kappa, c, u)
    for row in (0, -1):
        assert np.array_equal(y[:, :, row, :], np.broadcast_to(y[:, :, row, :1], y[:, :, row, :].shape))


def reduced_basis(shape):
    """Basis of the reduced space: one vector per interior slot, one
    phi-replicated vector per (radius, pole)."""
    nr, nt1, np_ = shape
    vecs = []
    for i in range(nr):
        for j in range(nt1):
            if j in (0, nt1 - 1):
                e = np.zeros(shape)
                e[i, j, :] = 1.0
                vecs.append(e)
            else:
                for k in range(np_):
                    e = np.zeros(shape)
                    e[i, j, k] = 1.0
                    vecs.append(e)
    return vecs


def reduced(vec_field, shape):
    """Coordinates of a replicated field in the reduced basis."""
    nr, nt1, np_ = shape
    out = []
    for i in range(nr):
        for j in range(nt1):
            if j in (0, nt1 - 1):
                out.append(vec_field[i, j, 0])
            else:
                out.extend(vec_field[i, j, :])
    return np.array(out)


@pytest.mark.parametrize("bc", [(0, 1), (1, 1), (0, 0)])
def test_tn_reduced_operator_symmetric_positive(oracle_mod, bc):
    o = oracle_mod.Oracle(mesh(3, 4, 6), *bc)
    sh = o.tn_shape
    kappa, c = rand_coeffs(sh, 6)
    basis = reduced_basis(sh)
    A = np.stack([reduced(o.tn_apply(kappa, c, e[None])[0], sh) for e in basis], axis=1)
    Vs = o.tn_volumes()
    Vr = reduced(Vs, sh).copy()
    nr, nt1, np_ = sh
    # a pole unknown weighs its whole cap: sum over its slices
    idx = 0
    for i in range(nr):
        for j in range(nt1):
            if j in (0, nt1 - 1):
                Vr[idx] = Vs[i, j, :].sum()
                idx += 1
            else:
                idx += np_
    VA = Vr[:, None] * A
    assert np.abs(VA - VA.T).max() <= 1e-14 * np.abs(VA).max()
    S = np.sqrt(Vr)[:, None] * A / np.sqrt(Vr)[None, :]
    ev = np.linalg.eigvalsh(0.5 * (S + S.T))
    assert ev.min() > 0
    if bc == (1, 1):  # c = 0, Neumann-Neumann: exactly one zero mode (the constant)
        A0 = np.stack([reduced(o.tn_apply(kappa, np.zeros(sh), e[None])[0], sh) for e in basis], axis=1)
        S0 = np.sqrt(Vr)[:, None] * A0 / np.sqrt(Vr)[None, :]
        ev0 = np.linalg.eigvalsh(0.5 * (S0 + S0.T))
        assert abs(ev0[0]) < 1e-12 * ev0[-1] and ev0[1] > 1e-8 * ev0[-1]


@pytest.mark.parametrize("bc", [(0, 1), (1, 1)])
def test_tn_symmetry_and_flux_conservation(oracle_mod, bc):
    o = oracle_mod.Oracle(mesh(8, 10, 12), *bc)
    sh = o.tn_shape
    kappa, c = rand_coeffs(sh, 7)
    rng = np.random.default_rng(8)
    u = replicate_poles(rng.standard_normal((1,) + sh))
    w = replicate_poles(rng.standard_normal((1,) + sh))
    Lu, Lw = o.tn_apply(kappa, c, u), o.tn_apply(kappa, c, w)
    scale = math.sqrt(o.tn_dot(Lu, Lu) * o.tn_dot(w, w))
    assert abs(o.tn_dot(Lu, w) - o.tn_dot(u, Lw)) <= 1e-14 * scale
    if bc == (1, 1):
        z = o.tn_apply(kappa, np.zeros(sh), u)
        V = o.tn_volumes()
        terms = (V[None] * z).ravel()
        assert abs(terms.sum()) <= 1e-13 * np.abs(terms).sum()


def test_tn_polar_cap_closed_form(oracle_mod):
    """u = cos(theta), kappa = 1, c = 0, Neumann r-faces: the r-fluxes vanish
    and -laplace(cos theta) = 2 cos(theta) / r^2 on every row, poles (+-2/r^2)
    included, at second order."""
    errs_pole, errs_int = [], []
    for n in (16, 32, 64):
        m = mesh(4, n, 2 * n)
        o = oracle_mod.Oracle(m, 1, 1)
        sh = o.tn_shape
        u = np.broadcast_to(np.cos(m.tF)[None, :, None], sh).copy()
        y = o.tn_apply(np.ones(sh), np.zeros(sh), u[None])[0]
        ex = 2.0 * np.cos(m.tF)[None, :, None] / m.rC[:, None, None] ** 2
        err = np.abs(y - ex)
        errs_pole.append(err[:, [0, -1]].max())
        errs_int.append(err[:, 1:-1].max())
    for e in (errs_pole, errs_int):
        orders = [math.log2(e[i] / e[i + 1]) for i in range(2)]
        assert orders[-1] > 1.8, (e, orders)


def u_star(r, t, p):
    return np.exp(-r) * (1.0 + np.cos(t) + np.sin(t) ** 2 * np.cos(2 * p) + 0.5 * np.sin(t) * np.sin(p))


def forcing(r, t, p):
    """-div(r^2 grad u*) in spherical coordinates (checked with sympy below)."""
    a = r * r - 4 * r
    return -np.exp(-r) * (a + (a - 2) * np.cos(t) + (a - 6) * np.sin(t) ** 2 * np.cos(2 * p)
                          + 0.5 * (a - 2) * np.sin(t) * np.sin(p))


def test_tn_mms_forcing_matches_sympy():
    sp = pytest.importorskip("sympy")
    r, t, p = sp.symbols("r t p", positive=True)
    u = sp.exp(-r) * (1 + sp.cos(t) + sp.sin(t) ** 2 * sp.cos(2 * p) + sp.Rational(1, 2) * sp.sin(t) * sp.sin(p))
    k = r ** 2
    div = (sp.diff(r ** 2 * k * sp.diff(u, r), r) / r ** 2
           + sp.diff(sp.sin(t) * k * sp.diff(u, t) / r, t) / (r * sp.sin(t))
           + sp.diff(k * sp.diff(u, p) / (r * sp.sin(t)), p) / (r * sp.sin(t)))
    f = sp.lambdify((r, t, p), -div, "numpy")
    rng = np.random.default_rng(0)
    pts = rng.uniform([1.0, 0.1, 0.0], [2.0, 3.0, 6.28], size=(20, 3))
    for rr, tt, pp in pts:
        assert abs(f(rr, tt, pp) - forcing(rr, tt, pp)) <= 1e-12 * max(1.0, abs(forcing(rr, tt, pp)))


def test_tn_mms_second_order_through_the_poles(oracle_mod):
    errs2, errsm = [], []
    for n in (8, 16, 32):
        m = mesh(n, n + n // 2, 2 * n, 1.0, 2.0, 4.0)
        o = oracle_mod.Oracle(m, 0, 0)
        sh = o.tn_shape
        R, T, P = np.meshgrid(m.rC, m.tF, m.pC, indexing="ij")
        kappa = R ** 2
        f = forcing(R, T, P)[None]
        # the pole rows of f: phi-constant (the forcing is smooth there)
        f = replicate_poles(f)
        Tb, Pb = np.meshgrid(m.tF, m.pC, indexing="ij")
        ubi = u_star(m.rF[0], Tb, Pb)[None]
        ubo = u_star(m.rF[-1], Tb, Pb)[None]
        rhs = o.tn_dirichlet_rhs(kappa, f, ubi, ubo)
        rc, x, it, rel, _ = o.tn_pcg(kappa, np.zeros(sh), rhs, np.zeros((1,) + sh), 1e-13, 20000)
        assert rc == oracle_mod.OK
        ue = u_star(R, T, P)
        V = o.tn_volumes()
        e = x[0] - ue
        errs2.append(math.sqrt((V * e * e).sum() / V.sum()))
        errsm.append(np.abs(e).max())
        # the pole values themselves
        assert np.abs(e[:, [0, -1]]).max() <= 2.0 * np.abs(e).max()
    for es in (errs2, errsm):
        orders = [math.log2(es[i] / es[i + 1]) for i in range(2)]
        assert min(orders) > 1.8, (es, orders)


def test_tn_dirichlet_rhs_is_the_boundary_term(oracle_mod):
    o = oracle_mod.Oracle(mesh(5, 6, 8), 0, 0)
    sh = o.tn_shape
    kappa, c = rand_coeffs(sh, 9)
    c = replicate_poles(c)
    y = o.tn_apply(kappa, c, np.ones((1,) + sh))[0] - c
    ones = np.ones((1,) + sh[1:])
    b = o.tn_dirichlet_rhs(kappa, np.zeros((1,) + sh), ones, ones)[0]
    np.testing.assert_allclose(y[1:-1], 0.0, atol=1e-15 * np.abs(c).max())
    np.testing.assert_allclose(y[[0, -1]], b[[0, -1]], rtol=1e-13, atol=1e-15)
    np.testing.assert_array_equal(b[1:-1], 0.0)


@pytest.mark.parametrize("bc", [(0, 1), (0, 0)])
def test_tn_pcg_matches_dense_solve(oracle_mod, bc):
    o = oracle_mod.Oracle(mesh(3, 4, 6), *bc)
    sh = o.tn_shape
    kappa, c = rand_coeffs(sh, 10)
    basis = reduced_basis(sh)
    A = np.stack([reduced(o.tn_apply(kappa, c, e[None])[0], sh) for e in basis], axis=1)
    f = replicate_poles(np.random.default_rng(11).standard_normal((1,) + sh))
    xd = np.linalg.solve(A, reduced(f[0], sh))
    rc, x, it, rel, _ = o.tn_pcg(kappa, c, f, np.zeros_like(f), 1e-13, 1000)
    assert rc == oracle_mod.OK and it <= len(basis) + 10
    xr = reduced(x[0], sh)
    assert np.abs(xr - xd).max() <= 1e-10 * np.abs(xd).max()
    # pole rows of the solution stay phi-constant
    for row in (0, -1):
        assert np.array_equal(x[0, :, row, :], np.broadcast_to(x[0, :, row, :1], x[0, :, row, :].shape))


def test_tn_mass_only_one_iteration(oracle_mod):
    o = oracle_mod.Oracle(mesh(4, 6, 8), 0, 1)
    sh = o.tn_shape
    c = replicate_poles(np.random.default_rng(12).uniform(0.1, 3, size=sh))
    f = replicate_poles(np.random.default_rng(13).standard_normal((2,) + sh))
    rc, x, it, rel, _ = o.tn_pcg(np.zeros(sh), c, f, np.zeros_like(f), 1e-12, 50)
    assert rc == oracle_mod.OK and it == 1
    np.testing.assert_allclose(x, f / c[None], rtol=1e-15, atol=0)
