"""Degenerate and boundary cases of the GPU path vs the oracle: a single
theta row, the minimal phi ring (np = 2), theta walls instead of poles,
Neumann-Neumann with a mass term, Dirichlet on both r-ends, one-plane slabs."""
import math

import numpy as np
import pytest

from paper_conf_ipps_caplansl23_b200 import workloads as W

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def mp():
    if not torch.cuda.is_available():
        pytest.skip("needs a GPU")
    from paper_conf_ipps_caplansl23_b200 import build
    build.build()
    from paper_conf_ipps_caplansl23_b200 import maspcg
    return maspcg


def walled_mesh(nr, nt, np_):
    """theta in [0.3, 2.8]: no pole, zero-flux theta walls (R5)."""
    m = W.stretched_mesh(nr, nt, np_)
    tF = np.linspace(0.3, 2.8, nt + 1)
    m.tF, m.tC = tF, 0.5 * (tF[1:] + tF[:-1])
    m.pole_north = m.pole_south = False
    return m


CASES = [
    ("one theta row", lambda: W.stretched_mesh(6, 1, 8), (0, 1)),
    ("np = 2", lambda: W.stretched_mesh(5, 6, 2), (0, 1)),
    ("theta walls", lambda: walled_mesh(7, 9, 12), (0, 1)),
    ("Neumann-Neumann + mass", lambda: W.stretched_mesh(6, 10, 16), (1, 1)),
    ("Dirichlet both ends", lambda: W.stretched_mesh(6, 10, 16), (0, 0)),
    ("one r-plane", lambda: W.stretched_mesh(1, 10, 16), (0, 0)),
]


@pytest.mark.parametrize("name,mk,bc", CASES, ids=[c[0] for c in CASES])
@pytest.mark.parametrize("ncomp", [1, 3])
def test_edge_case_apply_and_pcg(mp, oracle_mod, name, mk, bc, ncomp):
    mesh = mk()
    shape = mesh.shape
    rng = np.random.default_rng(11)
    kappa = rng.uniform(0.5, 2.0, size=shape)
    c = rng.uniform(0.1, 1.0, size=shape)
    d = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    g = mp.Grid(mesh)
    op = mp.Operator(g, ncomp, d(kappa), d(c), *bc)
    o = oracle_mod.Oracle(mesh, *bc)
    V = o.volumes()[None]
    x = rng.standard_normal((ncomp,) + shape)
    y = torch.empty_like(d(x))
    op.apply(d(x), y)
    yo = o.apply(kappa, c, x)
    assert math.sqrt((V * (y.cpu().numpy() - yo) ** 2).sum() / (V * yo ** 2).sum()) <= 1e-13
    f = rng.standard_normal((ncomp,) + shape)
    xg = torch.zeros_like(d(f))
    st, it, rel, _ = op.solve(d(f), xg, 1e-12, 2000)
    rc, xo, ito, _, _ = o.pcg(kappa, c, f, np.zeros_like(f), 1e-12, 2000)
    assert st == mp.MAS_OK and rc == oracle_mod.OK
    assert abs(it - ito) <= 1
    assert math.sqrt((V * (xg.cpu().numpy() - xo) ** 2).sum() / (V * xo ** 2).sum()) <= 1e-10
