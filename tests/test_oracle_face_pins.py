"""Pins for the oracle's face-centred placements (NEXT-2, readings R32-R33
in DESIGN.md §3.8): r nodes (v_r's location, mas_ref_rn_*) and phi nodes
(v_phi's location, mas_ref_pn_*: the cell-centred operator on the dual phi
mesh).  Pinned by what mathematics fixes:
* the node volumes fill the shell between rC_0 and rC_{nr-1} (r nodes) /
  the whole shell (phi nodes) at O(h^2);
* L 1 = c bitwise (Neumann-Neumann), V-symmetry and definiteness, flux
  conservation;
* the manufactured solution of C1 evaluated AT the nodes (Dirichlet data at
  the boundary nodes rF_0 / rF_nr), second order in L2_V and max norm;
* PCG = the dense solve."""
import math

import numpy as np
import pytest

from paper_conf_ipps_caplansl23_b200 import workloads as W


def mesh(nr, nt, np_, R=3.0):
    return W.stretched_mesh(nr, nt, np_, 1.0, 2.0, R)


def phi_stretched(m, b=0.6):
    """the same mesh with a smooth non-uniform periodic phi mesh
    (pF = 2 pi s + b sin 2 pi s): the phi nodes are then off the dual cells'
    midpoints by O(h^2), and the dual tables differ from the cell ones"""
    import dataclasses
    n = len(m.pF) - 1
    s = np.arange(n + 1, dtype=np.float64) / n
    pF = 2.0 * math.pi * s + b * np.sin(2.0 * math.pi * s)
    pF[0], pF[-1] = 0.0, 2.0 * math.pi
    return dataclasses.replace(m, pF=pF, pC=0.5 * (pF[1:] + pF[:-1]))


def rand(shape, seed):
    rng = np.random.default_rng(seed)
    return rng.uniform(0.5, 2.0, size=shape), rng.uniform(0.1, 1.0, size=shape)


def orders(e):
    return [math.log2(e[i] / e[i + 1]) for i in range(len(e) - 1)]


def test_rn_volumes_fill_the_node_shell(oracle_mod):
    errs = []
    for n in (8, 16, 32):
        m = mesh(n, 2 * n, 2 * n)
        o = oracle_mod.Oracle(m, 0, 0)
        exact = 4 * math.pi / 3 * (m.rC[-1] ** 3 - m.rC[0] ** 3)
        errs.append(abs(o.rn_volumes().sum() - exact) / exact)
    assert min(orders(errs)) > 1.8, errs


@pytest.mark.parametrize("stretch", [False, True])
def test_pn_volumes_fill_the_shell(oracle_mod, stretch):
    m = phi_stretched(mesh(6, 8, 12)) if stretch else mesh(6, 8, 12)
    o = oracle_mod.Oracle(m, 0, 0)
    np.testing.assert_allclose(o.pn_volumes().sum(), o.volumes().sum(), rtol=1e-14)


@pytest.mark.parametrize("which", ["rn", "pn", "pn-stretched"])
def test_constant_symmetry_conservation(oracle_mod, which):
    m = phi_stretched(mesh(7, 8, 10)) if which == "pn-stretched" else mesh(7, 8, 10)
    which = which[:2]
    o = oracle_mod.Oracle(m, 1, 1)
    sh = o.rn_shape if which == "rn" else o.shape
    ap = o.rn_apply if which == "rn" else o.pn_apply
    vol = o.rn_volumes() if which == "rn" else o.pn_volumes()
    kappa, c = rand(sh, 3)
    assert np.array_equal(ap(kappa, c, np.ones((1,) + sh))[0], c)
    rng = np.random.default_rng(4)
    for bc in ((0, 1), (0, 0), (1, 1)):
        ob = oracle_mod.Oracle(m, *bc)
        apb = ob.rn_apply if which == "rn" else ob.pn_apply
        u, w = rng.standard_normal((2, 1) + sh)
        Lu, Lw = apb(kappa, c, u), apb(kappa, c, w)
        dot = lambda a, b: float((vol[None] * a * b).sum())
        assert abs(dot(Lu, w) - dot(u, Lw)) <= 1e-14 * math.sqrt(dot(Lu, Lu) * dot(w, w))
    z = ap(kappa, np.zeros(sh), rng.standard_normal((1,) + sh))
    terms = (vol[None] * z).ravel()
    assert abs(terms.sum()) <= 1e-13 * np.abs(terms).sum()


@pytest.mark.parametrize("which", ["rn", "pn"])
def test_dense_spd_and_pcg(oracle_mod, which):
    m = mesh(4, 4, 6)
    o = oracle_mod.Oracle(m, 0, 1)
    sh = o.rn_shape if which == "rn" else o.shape
    ap = o.rn_apply if which == "rn" else o.pn_apply
    vol = (o.rn_volumes() if which == "rn" else o.pn_volumes()).ravel()
    kappa, c = rand(sh, 5)
    n = int(np.prod(sh))
    A = np.stack([ap(kappa, c, e.reshape((1,) + sh)).ravel() for e in np.eye(n)], axis=1)
    VA = vol[:, None] * A
    assert np.abs(VA - VA.T).max() <= 1e-14 * np.abs(VA).max()
    S = np.sqrt(vol)[:, None] * A / np.sqrt(vol)[None, :]
    assert np.linalg.eigvalsh(0.5 * (S + S.T)).min() > 0
    f = np.random.default_rng(6).standard_normal((1,) + sh)
    pcg = o.rn_pcg if which == "rn" else o.pn_pcg
    rc, x, it, rel, _ = pcg(kappa, c, f, np.zeros_like(f), 1e-13, 1000)
    xd = np.linalg.solve(A, f.ravel())
    assert rc == oracle_mod.OK and np.abs(x.ravel() - xd).max() <= 1e-10 * np.abs(xd).max()


def test_rn_mms_second_order(oracle_mod):
    """C1's manufactured solution at the r nodes, Dirichlet values at the
    boundary nodes rF_0 and rF_nr, kappa = r^2 at the nodes."""
    e2, em = [], []
    for n in (8, 16, 32):
        m = mesh(n, n + n // 2, 2 * n, R=4.0)
        o = oracle_mod.Oracle(m, 0, 0)
        sh = o.rn_shape
        R, T, P = np.meshgrid(m.rF[1:-1], m.tC, m.pC, indexing="ij")
        kappa = R ** 2
        f = W.mms_forcing(R, T, P)[None]
        Tb, Pb = np.meshgrid(m.tC, m.pC, indexing="ij")
        ubi = W.mms_solution(m.rF[0], Tb, Pb)[None]
        ubo = W.mms_solution(m.rF[-1], Tb, Pb)[None]
        rhs = o.rn_dirichlet_rhs(kappa, f, ubi, ubo)
        rc, x, it, rel, _ = o.rn_pcg(kappa, np.zeros(sh), rhs, np.zeros_like(rhs), 1e-13, 20000)
        assert rc == oracle_mod.OK
        V = o.rn_volumes()
        e = x[0] - W.mms_solution(R, T, P)
        e2.append(math.sqrt((V * e * e).sum() / V.sum()))
        em.append(np.abs(e).max())
    assert min(orders(e2)) > 1.8 and min(orders(em)) > 1.7, (e2, em)


@pytest.mark.parametrize("stretch", [False, True])
def test_pn_mms_second_order(oracle_mod, stretch):
    """C1's manufactured solution at the phi nodes (rC, tC, pF_k); also on a
    non-uniform phi mesh"""
    e2 = []
    for n in (8, 16, 32):
        m = mesh(n, n + n // 2, 2 * n, R=4.0)
        m = phi_stretched(m) if stretch else m
        o = oracle_mod.Oracle(m, 0, 0)
        R, T, P = np.meshgrid(m.rC, m.tC, m.pF[:-1], indexing="ij")
        f = W.mms_forcing(R, T, P)[None]
        Tb, Pb = np.meshgrid(m.tC, m.pF[:-1], indexing="ij")
        ubi = W.mms_solution(m.rF[0], Tb, Pb)[None]
        ubo = W.mms_solution(m.rF[-1], Tb, Pb)[None]
        rhs = o.pn_dirichlet_rhs(R ** 2, f, ubi, ubo)
        rc, x, it, rel, _ = o.pn_pcg(R ** 2, np.zeros(o.shape), rhs, np.zeros_like(rhs), 1e-13, 20000)
        V = o.pn_volumes()
        e = x[0] - W.mms_solution(R, T, P)
        e2.append(math.sqrt((V * e * e).sum() / V.sum()))
    assert min(orders(e2)) > 1.8, e2
