"""NEXT-2 vector-Laplacian curvature terms on the GPU (mas_op_set_curvature)
against the oracle's mas_ref_op_apply_curv / mas_ref_pcg_solve_curv (pinned in
tests/test_oracle_curv_pins.py): matvec rel L2_V <= 1e-13 and elementwise
1e-13 * 2 D max|x| (D + the curvature diagonal); PCG iterations +-1, x <=
1e-10; graph == host loop; 2 virtual r-slab ranks; switching off restores
the plain operator."""
import math
import threading

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


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a, dtype=np.float64)).cuda()


def rel_l2_V(V, a, b):
    V = V[None]
    return math.sqrt((V * (a - b) ** 2).sum() / max((V * b ** 2).sum(), 1e-300))


@pytest.mark.parametrize("shape", [(16, 24, 32), (9, 13, 70), (33, 8, 64), (5, 17, 130)])
@pytest.mark.parametrize("bc", [(0, 1), (1, 1)])
def test_curv_apply_matches_oracle(mp, oracle_mod, shape, bc):
    mesh = W.stretched_mesh(*shape)
    rng = np.random.default_rng(2)
    kappa, c = rng.uniform(0.5, 2.0, size=shape), rng.uniform(0.1, 1.0, size=shape)
    x = W.random_field((3,) + shape, 42)
    g = mp.Grid(mesh)
    op = mp.Operator(g, 3, dev(kappa), dev(c), *bc)
    op.set_curvature(True)
    y = torch.empty((3,) + shape, dtype=torch.float64, device="cuda")
    op.apply(dev(x), y)
    o = oracle_mod.Oracle(mesh, *bc)
    yo = o.apply_curv(kappa, c, x)
    yg = y.cpu().numpy()
    V = o.volumes()
    assert rel_l2_V(V, yg, yo) <= 1e-13
    R, T = np.meshgrid(mesh.rC, mesh.tC, indexing="ij")
    curv = kappa * (1.0 / (R * np.sin(T)) ** 2)[:, :, None] + kappa * (2.0 / R ** 2)[:, :, None]
    scale = 2.0 * (o.diag(kappa, c) + curv)[None] * np.abs(x).max()
    assert (np.abs(yg - yo) / scale).max() <= 1e-13
    # off again: the plain operator
    op.set_curvature(False)
    op.apply(dev(x), y)
    assert rel_l2_V(V, y.cpu().numpy(), o.apply(kappa, c, x)) <= 1e-13


def solve(mp, prob, prof=False, dist=None):
    g = mp.Grid(prob.mesh, dist=dist)
    op = mp.Operator(g, 3, dev(prob.kappa), dev(prob.c), prob.bc_inner, prob.bc_outer)
    op.set_curvature(True)
    op.set_profiling(prof)
    f = dev(prob.f)
    x = dev(prob.x0)
    st, it, rel, hist = op.solve(f, x, prob.tol, prob.maxit, True)
    torch.cuda.synchronize()
    return st, x.cpu().numpy(), it, hist, op, g


@pytest.mark.parametrize("shape", [(16, 24, 64), (33, 8, 66), (40, 20, 64)])
def test_curv_pcg_matches_oracle(mp, oracle_mod, shape):
    prob = W.viscosity_problem(*shape)
    o = oracle_mod.Oracle.for_problem(prob)
    rc, xo, ito, relo, histo = o.pcg_curv(prob.kappa, prob.c, prob.f, prob.x0, prob.tol, prob.maxit)
    st, x, it, hist, op, g = solve(mp, prob)
    assert rc == oracle_mod.OK and st == mp.MAS_OK
    assert abs(it - ito) <= 1, (it, ito)
    assert rel_l2_V(o.volumes(), x, xo) <= 1e-10
    np.testing.assert_allclose(hist[:10], histo[:10], rtol=1e-9, atol=0)
    b = solve(mp, prob, prof=True)  # the host-driven loop: same bits
    assert b[2] == it
    np.testing.assert_array_equal(b[1], x)
    with pytest.raises(mp.MasError):
        op.set_single_reduction(True)


def test_curv_virtual_ranks(mp, oracle_mod):
    prob = W.viscosity_problem(26, 16, 64, warm=False)
    vid = mp.virtual_ranks_id(9901)
    res, errs = {}, []

    def rank_main(r):
        try:
            torch.cuda.set_device(0)
            with torch.cuda.stream(torch.cuda.Stream()):
                g = mp.Grid(prob.mesh, dist=(2, r, vid))
                sl = slice(g.i0, g.i0 + g.nl)
                op = mp.Operator(g, 3, dev(prob.kappa[sl]), dev(prob.c[sl]), prob.bc_inner,
                                 prob.bc_outer)
                op.set_curvature(True)
                x = dev(prob.x0[:, sl])
                st, it, rel, _ = op.solve(dev(prob.f[:, sl]), x, prob.tol, prob.maxit)
                torch.cuda.current_stream().synchronize()
                res[r] = (g.i0, g.nl, st, it, x.cpu().numpy())
                op.close()
                g.close()
        except Exception as e:  # noqa: BLE001
            errs.append((r, repr(e)))

    th = [threading.Thread(target=rank_main, args=(r,)) for r in range(2)]
    for t in th:
        t.start()
    for t in th:
        t.join(timeout=600)
    assert not errs, errs
    o = oracle_mod.Oracle.for_problem(prob)
    rc, xo, ito, _, _ = o.pcg_curv(prob.kappa, prob.c, prob.f, prob.x0, prob.tol, prob.maxit)
    assert res[0][3] == res[1][3] and abs(res[0][3] - ito) <= 1
    xg = np.empty_like(xo)
    for r in range(2):
        i0, nl, st, it, x = res[r]
        assert st == mp.MAS_OK
        xg[:, i0:i0 + nl] = x
    assert rel_l2_V(o.volumes(), xg, xo) <= 1e-10
