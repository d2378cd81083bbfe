"""Pins for the oracle's vector-Laplacian curvature terms of the 3-component
viscosity operator (mas_ref_op_apply_curv / mas_ref_pcg_solve_curv; NEXT-2,
reading R31 in DESIGN.md §3.7).

Each curvature factor is pinned by an exact vector Laplacian of a field whose
other components vanish (so the omitted coupling terms are zero there):
* r:     v = r-hat (the unit radial field):  -lap v = 2 r-hat / r^2, exact on
         the grid (the scalar part of a constant vanishes bitwise);
* phi:   v = r sin(theta) phi-hat (rigid rotation, Cartesian (-y, x, 0)):
         lap v = 0, so the curvature term cancels the scalar Laplacian of
         v_phi at second order;
* theta: v = r^2 sin(theta) theta-hat (Cartesian (xz, yz, -(x^2+y^2))):
         lap v = (0, 0, -4), whose theta component is 4 sin(theta): the
         discrete theta component of L v -> -4 sin(theta) at second order.
Plus: V-symmetry, and PCG = the dense solve."""
import math

import numpy as np
import pytest

from paper_conf_ipps_caplansl23_b200 import workloads as W


def fields(m, comp, fn):
    R, T, P = np.meshgrid(m.rC, m.tC, m.pC, indexing="ij")
    v = np.zeros((3,) + R.shape)
    v[comp] = fn(R, T, P)
    return v, R, T


def test_curv_radial_unit_field_exact(oracle_mod):
    m = W.stretched_mesh(6, 8, 10, 1.0, 2.0, 3.0)
    o = oracle_mod.Oracle(m, 1, 1)
    v, R, T = fields(m, 0, lambda R, T, P: np.ones_like(R))
    sh = R.shape
    y = o.apply_curv(np.ones(sh), np.zeros(sh), v)
    np.testing.assert_allclose(y[0], 2.0 / R ** 2, rtol=2e-16, atol=0)
    assert np.array_equal(y[1:], np.zeros_like(y[1:]))


def _orders(errs):
    return [math.log2(errs[i] / errs[i + 1]) for i in range(len(errs) - 1)]


def test_curv_rigid_rotation_is_harmonic(oracle_mod):
    errs = []
    for n in (16, 32, 64):
        m = W.stretched_mesh(n // 2, n, 2 * n, 1.0, 2.0, 3.0)
        o = oracle_mod.Oracle(m, 1, 1)
        v, R, T = fields(m, 2, lambda R, T, P: R * np.sin(T))
        sh = R.shape
        y = o.apply_curv(np.ones(sh), np.zeros(sh), v)
        V = o.volumes()
        # Neumann r-faces: the r-flux of v_phi = r sin(theta) does not vanish
        # on the boundary planes; compare the interior planes
        sl = slice(1, -1)
        errs.append(math.sqrt((V[sl] * y[2, sl] ** 2).sum() / V[sl].sum()))
        assert np.array_equal(y[:2], np.zeros_like(y[:2]))
    assert min(_orders(errs)) > 1.7, errs


def test_curv_theta_component_closed_form(oracle_mod):
    errs = []
    for n in (16, 32, 64):
        m = W.stretched_mesh(n // 2, n, 2 * n, 1.0, 2.0, 3.0)
        o = oracle_mod.Oracle(m, 1, 1)
        v, R, T = fields(m, 1, lambda R, T, P: R * R * np.sin(T))
        sh = R.shape
        y = o.apply_curv(np.ones(sh), np.zeros(sh), v)
        V = o.volumes()
        sl = slice(1, -1)
        e = y[1, sl] - (-4.0 * np.sin(T[sl]))
        errs.append(math.sqrt((V[sl] * e ** 2).sum() / V[sl].sum()))
    assert min(_orders(errs)) > 1.7, errs


def test_curv_symmetric_and_pcg_dense(oracle_mod):
    shape = (3, 4, 6)
    m = W.stretched_mesh(*shape)
    o = oracle_mod.Oracle(m, 0, 1)
    rng = np.random.default_rng(3)
    kappa, c = rng.uniform(0.5, 2.0, size=shape), rng.uniform(0.1, 1.0, size=shape)
    n = 3 * o.N
    A = np.empty((n, n))
    e = np.zeros(n)
    for col in range(n):
        e[:] = 0.0
        e[col] = 1.0
        A[:, col] = o.apply_curv(kappa, c, e.reshape((3,) + shape)).ravel()
    V = np.tile(o.volumes().ravel(), 3)
    VA = V[:, None] * A
    assert np.abs(VA - VA.T).max() <= 1e-14 * np.abs(VA).max()
    S = np.sqrt(V)[:, None] * A / np.sqrt(V)[None, :]
    assert np.linalg.eigvalsh(0.5 * (S + S.T)).min() > 0
    f = rng.standard_normal((3,) + shape)
    xd = np.linalg.solve(A, f.ravel()).reshape(f.shape)
    rc, x, it, rel, _ = o.pcg_curv(kappa, c, f, np.zeros_like(f), 1e-13, 1000)
    assert rc == oracle_mod.OK
    Vv = o.volumes()[None]
    assert math.sqrt((Vv * (x - xd) ** 2).sum() / (Vv * xd ** 2).sum()) <= 1e-10
    # the curvature terms differ from the plain operator only on the diagonal
    x0 = rng.standard_normal((3,) + shape)
    d = o.apply_curv(kappa, c, x0) - o.apply(kappa, c, x0)
    assert np.abs(d - np.diag(A - np.stack([o.apply(kappa, c, ee.reshape((3,) + shape)).ravel()
                                            for ee in np.eye(n)], axis=1)).reshape(x0.shape) * x0).max() \
        <= 1e-13 * np.abs(d).max()
