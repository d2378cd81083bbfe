"""Pins for the oracle's per-radius array reduction (the paper's Listings 3-5,
"sum0(i)=sum0(i)+array(i,j)*...", P:428-445 / P:592-645; reading R27: the
elided factor is an angular weight w[j][k]):

* a field constant on each r-plane, with the normalised angular area weights,
  returns that constant;
* the polar-cap phi average (weights dp_k / 2 pi on the first theta row) of
  U(r) (1 + sin(theta) cos(phi)) returns U(r) (the cos(phi) mode averages out
  on the uniform periodic phi mesh);
* against numpy's einsum on random data (a library routine).
"""
import math

import numpy as np

from paper_conf_ipps_caplansl23_b200 import workloads as W


def test_plane_constant_returns_the_constant(oracle_mod):
    m = W.stretched_mesh(6, 10, 16)
    o = oracle_mod.Oracle(m, 0, 1)
    c = np.random.default_rng(1).uniform(-2, 2, size=(2, 6))
    x = np.broadcast_to(c[:, :, None, None], (2, 6, 10, 16)).copy()
    area = (np.sin(m.tC) * np.diff(m.tF))[:, None] * np.diff(m.pF)[None, :]
    w = area / area.sum()
    np.testing.assert_allclose(o.radial_sums(x, w), c, rtol=1e-14, atol=1e-15)


def test_polar_cap_phi_average(oracle_mod):
    m = W.stretched_mesh(5, 12, 32)
    o = oracle_mod.Oracle(m, 0, 1)
    r, t, p = np.meshgrid(m.rC, m.tC, m.pC, indexing="ij")
    U = np.exp(-r) * (2.0 + r)
    x = (U * (1.0 + np.sin(t) * np.cos(p)))[None]
    w = np.zeros((12, 32))
    w[0] = np.diff(m.pF) / (2.0 * math.pi)
    np.testing.assert_allclose(o.radial_sums(x, w)[0], U[:, 0, 0], rtol=1e-14)


def test_matches_einsum(oracle_mod):
    m = W.stretched_mesh(7, 9, 14)
    o = oracle_mod.Oracle(m, 0, 1)
    rng = np.random.default_rng(3)
    x = rng.standard_normal((3, 7, 9, 14))
    w = rng.standard_normal((9, 14))
    np.testing.assert_allclose(o.radial_sums(x, w), np.einsum("mijk,jk->mi", x, w), rtol=1e-13,
                               atol=1e-13)
