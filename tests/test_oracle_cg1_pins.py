"""Pins for the oracle's single-reduction PCG (mas_ref_pcg_solve_cg1, the
Chronopoulos-Gear form of NEXT-1, reading R28 in DESIGN.md).

The paper prints no solver detail ("Krylov solvers"), so the
variant is pinned by what mathematics fixes about it:
* brute force: on tiny grids it solves the assembled system (numpy) to 1e-10;
* equivalence: in exact arithmetic its iterates ARE the standard Jacobi-PCG
  iterates (mas_ref_pcg_solve, itself pinned by tests/test_oracle_pins.py),
  so at a fixed iteration count k = 1..8 x_k agrees to rounding, and the
  residual histories agree over the first iterations; a dropped term of the
  alpha recurrence (d - b g / a), a wrong s or p update fails these;
* special cases: mass-only converges in exactly one iteration with x = f/c,
  zero rhs gives x = 0, an exact start stops at k = 0;
* iteration counts at tol 1e-12 on C1/C2/C3-shaped problems within +-2 of
  the standard PCG (rounding differs, SURVEY §8(f) NEXT-1's band)."""
import math

import numpy as np
import pytest

from paper_conf_ipps_caplansl23_b200 import workloads as W


def rand_coeffs(shape, seed):
    rng = np.random.default_rng(seed)
    return rng.uniform(0.5, 2.0, size=shape), rng.uniform(0.1, 1.0, size=shape)


def rel_V(V, a, b):
    V = V[None]
    return math.sqrt((V * (a - b) ** 2).sum() / (V * b ** 2).sum())


@pytest.mark.parametrize("bc", [(0, 1), (0, 0), (1, 1)])
def test_cg1_matches_dense_solve(oracle_mod, bc):
    shape = (4, 6, 8)
    o = oracle_mod.Oracle(W.stretched_mesh(*shape), *bc)
    kappa, c = rand_coeffs(shape, 21)
    n = o.N
    A = np.empty((n, n))
    e = np.zeros(n)
    for col in range(n):
        e[:] = 0.0
        e[col] = 1.0
        A[:, col] = o.apply(kappa, c, e.reshape((1,) + shape)).ravel()
    f = np.random.default_rng(22).standard_normal((1,) + shape)
    xd = np.linalg.solve(A, f.ravel()).reshape(f.shape)
    rc, x, it, rel, hist = o.pcg_cg1(kappa, c, f, np.zeros_like(f), 1e-13, 1000)
    assert rc == oracle_mod.OK and it <= n + 10
    assert rel_V(o.volumes(), x, xd) <= 1e-10


@pytest.mark.parametrize("ncomp", [1, 3])
def test_cg1_iterates_equal_standard_pcg(oracle_mod, ncomp):
    """Fixed iteration counts (tol = 0): x_k of both recurrences agree to
    rounding for k = 1..8; the residual histories agree to 1e-9."""
    prob = W.viscosity_problem(8, 12, 16) if ncomp == 3 else W.conduction_problem(8, 12, 16)
    o = oracle_mod.Oracle.for_problem(prob)
    f = o.dirichlet_rhs(prob.kappa, prob.f, prob.ub_inner, prob.ub_outer)
    V = o.volumes()
    for k in range(1, 9):
        rs, xs, its, _, hs = o.pcg(prob.kappa, prob.c, f, prob.x0, 0.0, k)
        rc, xc, itc, _, hc = o.pcg_cg1(prob.kappa, prob.c, f, prob.x0, 0.0, k)
        assert rs == rc == oracle_mod.NOT_CONVERGED and its == itc == k
        dx = rel_V(V, xc - prob.x0, xs - prob.x0)  # the correction x_k - x0
        assert dx <= 1e-11, (k, dx)
        np.testing.assert_allclose(hc, hs, rtol=1e-9, atol=0)


@pytest.mark.parametrize("mk", ["mms", "conduction", "viscosity"])
def test_cg1_iteration_counts_within_two(oracle_mod, mk):
    prob = {"mms": lambda: W.mms_problem(16, 24, 32),
            "conduction": lambda: W.conduction_problem(16, 24, 64),
            "viscosity": lambda: W.viscosity_problem(16, 24, 64)}[mk]()
    rs, xs, its, _, _ = oracle_mod.solve_problem(prob)
    rc, xc, itc, relc, _ = oracle_mod.solve_problem(prob, cg1=True)
    assert rs == rc == oracle_mod.OK
    assert abs(itc - its) <= 2, (itc, its)
    assert relc <= prob.tol
    assert rel_V(oracle_mod.Oracle.for_problem(prob).volumes(), xc, xs) <= 1e-9


def test_cg1_special_cases(oracle_mod):
    shape = (4, 5, 6)
    o = oracle_mod.Oracle(W.stretched_mesh(*shape), 0, 1)
    c = np.random.default_rng(23).uniform(0.1, 3, size=shape)
    f = np.random.default_rng(24).standard_normal((3,) + shape)
    # kappa == 0: L = D, exactly one iteration, x = f / c
    rc, x, it, rel, hist = o.pcg_cg1(np.zeros(shape), c, f, np.zeros_like(f), 1e-12, 50)
    assert rc == oracle_mod.OK and it == 1
    np.testing.assert_allclose(x, f / c[None], rtol=4e-16, atol=0)
    kappa, c = rand_coeffs(shape, 25)
    x0 = np.ones((1,) + shape)
    rc, x, it, rel, hist = o.pcg_cg1(kappa, c, np.zeros_like(x0), x0, 1e-12, 10)
    assert rc == oracle_mod.OK and it == 0 and (x == 0).all()
    fx = o.apply(kappa, c, x0)
    rc, x, it, rel, hist = o.pcg_cg1(kappa, c, fx, x0, 1e-12, 10)
    assert rc == oracle_mod.OK and it == 0 and np.array_equal(x, x0)
    rc, x, it, rel, hist = o.pcg_cg1(kappa, c, fx + 1.0, x0, 1e-12, 0)
    assert rc == oracle_mod.NOT_CONVERGED and it == 0 and np.array_equal(x, x0)
