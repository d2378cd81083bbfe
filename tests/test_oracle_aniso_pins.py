"""Pins for the ORACLE's field-aligned conduction operator L_par (SURVEY.md
§8(f) NEXT-4; readings R21-R26 in oracle/mas_ref.c and DESIGN.md §3.4).

The paper prints no formula for MAS's thermal conduction (P:748-750 names the
thermodynamic model only; P:1212-1216 cites the implicit Krylov schemes), so
L_par is pinned by what mathematics fixes: exact null spaces (constants, the
checkerboard mode of the 8-cell corner gradient, variation perpendicular to
b), symmetry and semi-definiteness, the assembled diagonal, a manufactured
solution whose forcing sympy derives from the continuous operator
-div(kpar b (b.grad u)) in spherical coordinates (observed order >= 1.8), and
scipy's CG / a dense solve on the assembled system.  A swapped b component,
a wrong metric factor (r, sin theta, h), a sign error or an index slip in the
corner stencil fails at least one of them.
"""
import math

import numpy as np
import pytest
import scipy.sparse.linalg

from paper_conf_ipps_caplansl23_b200 import workloads as W


def rand_corner_fields(shape, seed, unit=False):
    rng = np.random.default_rng(seed)
    kpar = rng.uniform(0.5, 2.0, size=shape)
    b = rng.standard_normal((3,) + shape)
    if unit:
        b /= np.linalg.norm(b, axis=0)
    return kpar, b


def dense(fn, n, shape):
    A = np.empty((n, n))
    e = np.zeros(n)
    for col in range(n):
        e[:] = 0.0
        e[col] = 1.0
        A[:, col] = fn(e.reshape((1,) + shape)).ravel()
    return A


@pytest.fixture(params=[(3, 4, 6), (5, 6, 8)])
def tiny(request, oracle_mod):
    shape = request.param
    m = W.stretched_mesh(*shape, r0=1.0, r1=2.0, R=3.0)
    return oracle_mod.Oracle(m, 0, 1), shape


def test_constant_is_in_the_null_space_bitwise(tiny):
    o, shape = tiny
    kpar, b = rand_corner_fields(shape, 1)
    y = o.aniso_apply(kpar, b, np.full((1,) + shape, 3.25))
    assert np.all(y == 0.0)


def test_checkerboard_is_in_the_null_space_bitwise(tiny):
    """The 8-cell corner gradient averages 4 differences per direction: the
    (-1)^(i+j+k) mode has zero gradient at every corner (the known null mode
    of the symmetric corner scheme; needs np even, R7)."""
    o, shape = tiny
    kpar, b = rand_corner_fields(shape, 2)
    i, j, k = np.meshgrid(*[np.arange(n) for n in shape], indexing="ij")
    u = ((-1.0) ** (i + j + k))[None]
    assert np.all(o.aniso_apply(kpar, b, u) == 0.0)


@pytest.mark.parametrize("axis", [0, 1, 2])
def test_variation_perpendicular_to_b_carries_no_flux(oracle_mod, axis):
    """b along coordinate direction `axis` and u independent of that
    coordinate: every corner difference along `axis` is exactly zero, so
    b.g = 0 and L_par u = 0 exactly, whatever u does in the other two
    directions.  Catches a b component paired with the wrong gradient."""
    shape = (5, 6, 8)
    m = W.stretched_mesh(*shape, r0=1.0, r1=2.0, R=3.0)
    o = oracle_mod.Oracle(m, 0, 1)
    kpar, _ = rand_corner_fields(shape, 3)
    b = np.zeros((3,) + shape)
    b[axis] = np.random.default_rng(4).uniform(0.5, 1.5, size=shape)
    u = np.random.default_rng(5).standard_normal(shape)
    u = np.repeat(np.take(u, [0], axis=axis), shape[axis], axis=axis)[None]
    y = o.aniso_apply(kpar, b, u)
    assert np.all(y == 0.0)
    # ... while a b with a component along another axis does see it
    b2 = b.copy()
    b2[(axis + 1) % 3] = 0.7
    assert np.abs(o.aniso_apply(kpar, b2, u)).max() > 1e-3


def test_symmetric_and_positive_semidefinite(tiny):
    o, shape = tiny
    kpar, b = rand_corner_fields(shape, 6)
    n = o.N
    A = dense(lambda x: o.aniso_apply(kpar, b, x), n, shape)
    V = o.volumes().ravel()
    VA = V[:, None] * A
    assert np.abs(VA - VA.T).max() <= 1e-14 * np.abs(VA).max()
    s = np.sqrt(V)
    ev = np.linalg.eigvalsh(0.5 * ((s[:, None] * A / s[None, :]) + (s[:, None] * A / s[None, :]).T))
    assert ev.min() >= -1e-12 * ev.max()
    # the null space holds at least the constant and the checkerboard
    assert (np.abs(ev) <= 1e-12 * ev.max()).sum() >= 2
    # R26: the Jacobi diagonal contribution is the assembled diagonal
    np.testing.assert_allclose(o.aniso_diag(kpar, b).ravel(), np.diag(A), rtol=1e-14, atol=0)


def test_symmetry_random_vectors_moderate_grid(oracle_mod):
    shape = (9, 12, 16)
    m = W.stretched_mesh(*shape)
    o = oracle_mod.Oracle(m, 0, 1)
    kpar, b = rand_corner_fields(shape, 7, unit=True)
    rng = np.random.default_rng(8)
    u, w = rng.standard_normal((2, 1) + shape)
    Lu, Lw = o.aniso_apply(kpar, b, u), o.aniso_apply(kpar, b, w)
    lhs, rhs = o.dot(Lu, w), o.dot(u, Lw)
    scale = math.sqrt(o.dot(Lu, Lu) * o.dot(w, w))
    assert abs(lhs - rhs) <= 1e-14 * scale
    assert o.dot(Lu, u) > 0.0


# ---------------------------------------------------------------------------
# discretisation: manufactured solution against the continuous operator
# ---------------------------------------------------------------------------
R0, R1 = 1.0, 2.0


def _mms_sympy():
    sp = pytest.importorskip("sympy")
    r, t, p = sp.symbols("r t p", positive=True)
    G = 1 + sp.sin(t) ** 2 * sp.cos(2 * p) + sp.sin(t) * sp.sin(p) / 2
    # u* has zero value-variation and zero r-derivative on both r boundaries,
    # so b.grad u* = 0 there (the no-boundary-flux reading R24)
    u = 1 + 4 * (r - R0) ** 2 * (R1 - r) ** 2 * G
    Br = 1 / r ** 2 + sp.Rational(6, 10) * sp.cos(t) / r ** 3
    Bt = sp.Rational(3, 10) * sp.sin(t) / r ** 3
    Bp = -sp.sin(t) / (2 * r)
    nB = sp.sqrt(Br ** 2 + Bt ** 2 + Bp ** 2)
    b = (Br / nB, Bt / nB, Bp / nB)
    kpar = r ** 2
    grad = (sp.diff(u, r), sp.diff(u, t) / r, sp.diff(u, p) / (r * sp.sin(t)))
    bg = sum(bi * gi for bi, gi in zip(b, grad))
    F = [kpar * bi * bg for bi in b]
    div = (sp.diff(r ** 2 * F[0], r) / r ** 2 + sp.diff(sp.sin(t) * F[1], t) / (r * sp.sin(t))
           + sp.diff(F[2], p) / (r * sp.sin(t)))
    fu = sp.lambdify((r, t, p), u, "numpy")
    ff = sp.lambdify((r, t, p), u - div, "numpy")  # c = 1: f = u* + L_par u*
    return fu, ff


def test_mms_second_order(oracle_mod):
    """(1 + L_par) u = f with f from sympy; L_iso switched off (kappa = 0),
    b = the axisymmetric spiral + dipole field (W.spiral_dipole_field with
    b0 = 0), kpar = r^2 at the corners.  RMS_V error of the PCG solution at
    O(h^2) on 8x12x16 -> 16x24x32 -> 32x48x64."""
    fu, ff = _mms_sympy()
    errs = []
    for (nr, nt, np_) in ((8, 12, 16), (16, 24, 32), (32, 48, 64)):
        m = W.stretched_mesh(nr, nt, np_, r0=R0, r1=R1, R=2.0)
        o = oracle_mod.Oracle(m, 0, 1)
        r, t, p = np.meshgrid(m.rC, m.tC, m.pC, indexing="ij")
        rc, tc, pc = np.meshgrid(m.rF[:-1], m.tF[:-1], m.pF[:-1], indexing="ij")
        b = W.spiral_dipole_field(rc, tc, pc, omega=0.5, dip=0.3, b0=0.0)
        kpar = rc ** 2
        shape = (nr, nt, np_)
        f = ff(r, t, p)[None]
        rcd, x, it, rel, _ = o.pcg_aniso(np.zeros(shape), np.ones(shape), kpar, b, f,
                                         np.zeros_like(f), 1e-13, 20000)
        assert rcd == oracle_mod.OK
        V = o.volumes()
        e = x[0] - fu(r, t, p)
        errs.append(math.sqrt((V * e * e).sum() / V.sum()))
    orders = [math.log2(errs[i] / errs[i + 1]) for i in range(2)]
    assert min(orders) >= 1.8, (errs, orders)


# ---------------------------------------------------------------------------
# solver on L_iso + L_par: brute force and a library routine
# ---------------------------------------------------------------------------
def test_pcg_aniso_matches_dense_solve_and_scipy_cg(oracle_mod):
    shape = (5, 6, 8)
    m = W.stretched_mesh(*shape, r0=1.0, r1=2.0, R=3.0)
    o = oracle_mod.Oracle(m, 0, 1)
    rng = np.random.default_rng(9)
    kappa = rng.uniform(0.01, 0.02, size=shape)
    c = rng.uniform(0.1, 1.0, size=shape)
    kpar, b = rand_corner_fields(shape, 10, unit=True)
    kpar *= 20.0
    n = o.N
    A = dense(lambda x: o.apply(kappa, c, x) + o.aniso_apply(kpar, b, x), n, shape)
    f = rng.standard_normal((1,) + shape)
    V = o.volumes().ravel()
    xd = np.linalg.solve(A, f.ravel())
    rc, x, it, rel, _ = o.pcg_aniso(kappa, c, kpar, b, f, np.zeros_like(f), 1e-12, 2000)
    assert rc == oracle_mod.OK
    err = math.sqrt((V * (x.ravel() - xd) ** 2).sum() / (V * xd ** 2).sum())
    assert err <= 1e-10
    # scipy CG on the symmetrised system with the assembled Jacobi diagonal
    s = np.sqrt(V)
    S = s[:, None] * A / s[None, :]
    S = 0.5 * (S + S.T)
    Dg = np.diag(A)
    np.testing.assert_allclose(o.diag(kappa, c).ravel() + o.aniso_diag(kpar, b).ravel(), Dg,
                               rtol=1e-14)
    count = [0]
    y, info = scipy.sparse.linalg.cg(S, s * f.ravel(), rtol=1e-12, atol=0.0, maxiter=2000,
                                     M=scipy.sparse.diags(1.0 / Dg),
                                     callback=lambda _: count.__setitem__(0, count[0] + 1))
    assert info == 0 and abs(it - count[0]) <= 1, (it, count[0])
    xs = y / s
    assert math.sqrt((V * (x.ravel() - xs) ** 2).sum() / (V * xs ** 2).sum()) <= 1e-10


def test_aniso_workload_shapes_and_unit_b(oracle_mod):
    prob = W.aniso_conduction_problem(8, 8, 16)
    assert prob.kpar.shape == (8, 8, 16) and prob.bhat.shape == (3, 8, 8, 16)
    np.testing.assert_allclose(np.linalg.norm(prob.bhat, axis=0), 1.0, rtol=1e-14)
    assert np.all(prob.kpar > 0)
