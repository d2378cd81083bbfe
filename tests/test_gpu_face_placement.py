"""NEXT-2 face-centred placements on the GPU (mas_op_setup_placed with
MAS_PLACE_R_NODE / MAS_PLACE_PHI_NODE: the unchanged kernels on other 1-D
tables) against the oracle's mas_ref_rn_* / mas_ref_pn_* (pinned in
tests/test_oracle_face_pins.py): matvec rel L2_V and elementwise 1e-13,
diagonal / Dirichlet helper 1e-14, PCG iterations +-1 and x <= 1e-10,
phi nodes on 2 virtual r-slab ranks."""
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


def host(t):
    torch.cuda.synchronize()
    return t.cpu().numpy()


def rel_l2_V(V, a, b):
    V = V[None] if a.ndim == 4 else V
    return math.sqrt((V * (a - b) ** 2).sum() / max((V * b ** 2).sum(), 1e-300))


def oracle_fns(o, which):
    if which == "rn":
        return o.rn_shape, o.rn_apply, o.rn_diag, o.rn_dirichlet_rhs, o.rn_volumes(), o.rn_pcg
    return o.shape, o.pn_apply, o.pn_diag, o.pn_dirichlet_rhs, o.pn_volumes(), o.pn_pcg


@pytest.mark.parametrize("shape", [(16, 24, 32), (9, 13, 70), (33, 8, 64), (2, 3, 4)])
@pytest.mark.parametrize("ncomp", [1, 3])
@pytest.mark.parametrize("bc", [(0, 1), (0, 0), (1, 1)])
@pytest.mark.parametrize("which", ["rn", "pn"])
def test_face_apply_diag_rhs(mp, oracle_mod, shape, ncomp, bc, which):
    mesh = W.stretched_mesh(*shape)
    o = oracle_mod.Oracle(mesh, *bc)
    sh, ap, dg, drhs, V, _ = oracle_fns(o, which)
    rng = np.random.default_rng(1)
    kappa, c = rng.uniform(0.5, 2.0, size=sh), rng.uniform(0.1, 1.0, size=sh)
    x = W.random_field((ncomp,) + sh, 42)
    pl = mp.MAS_PLACE_R_NODE if which == "rn" else mp.MAS_PLACE_PHI_NODE
    g = mp.Grid(mesh)
    op = mp.Operator(g, ncomp, dev(kappa), dev(c), *bc, placement=pl)
    y = torch.empty((ncomp,) + sh, dtype=torch.float64, device="cuda")
    op.apply(dev(x), y)
    yo = ap(kappa, c, x)
    yg = host(y)
    assert rel_l2_V(V, yg, yo) <= 1e-13
    scale = 2.0 * dg(kappa, c)[None] * np.abs(x).max()
    assert (np.abs(yg - yo) / scale).max() <= 1e-13
    D = torch.empty(sh, dtype=torch.float64, device="cuda")
    op.diag(D)
    np.testing.assert_allclose(host(D), dg(kappa, c), rtol=1e-14, atol=0)
    f = rng.standard_normal((ncomp,) + sh)
    ub = rng.standard_normal((ncomp,) + sh[1:])
    fd = dev(f)
    op.dirichlet_rhs(dev(ub), dev(ub), fd)
    np.testing.assert_allclose(host(fd), drhs(kappa, f, ub, ub), rtol=1e-14, atol=1e-14 * np.abs(f).max())
    assert abs(op.dot(dev(x), dev(x)) - (V[None] * x * x).sum()) <= 1e-13 * (V[None] * x * x).sum()
    op.close()
    g.close()


@pytest.mark.parametrize("ncomp", [1, 3])
def test_phi_nodes_nonuniform_phi(mp, oracle_mod, ncomp):
    """A non-uniform periodic phi mesh: the dual phi cells differ from the
    cell-centred ones (on a uniform mesh they coincide, so only this case
    tells the phi-node tables from the cell tables)."""
    import dataclasses
    m0 = W.stretched_mesh(12, 10, 48)
    s = np.arange(49, dtype=np.float64) / 48
    pF = 2.0 * math.pi * s + 0.6 * np.sin(2.0 * math.pi * s)
    pF[0], pF[-1] = 0.0, 2.0 * math.pi
    mesh = dataclasses.replace(m0, pF=pF, pC=0.5 * (pF[1:] + pF[:-1]))
    for which in ("pn", "cell"):
        o = oracle_mod.Oracle(mesh, 0, 1)
        sh = o.shape
        rng = np.random.default_rng(3)
        kappa, c = rng.uniform(0.5, 2.0, size=sh), rng.uniform(0.1, 1.0, size=sh)
        x = W.random_field((ncomp,) + sh, 7)
        pl = mp.MAS_PLACE_PHI_NODE if which == "pn" else mp.MAS_PLACE_CELL
        g = mp.Grid(mesh)
        op = mp.Operator(g, ncomp, dev(kappa), dev(c), 0, 1, placement=pl)
        y = torch.empty((ncomp,) + sh, dtype=torch.float64, device="cuda")
        op.apply(dev(x), y)
        yo = (o.pn_apply if which == "pn" else o.apply)(kappa, c, x)
        V = o.pn_volumes() if which == "pn" else o.volumes()
        assert rel_l2_V(V, host(y), yo) <= 1e-13, which
        op.close()
        g.close()


def mms_at(mesh, which):
    """C1's manufactured problem at the nodes of the placement."""
    r = mesh.rF[1:-1] if which == "rn" else mesh.rC
    p = mesh.pF[:-1] if which == "pn" else mesh.pC
    R, T, P = np.meshgrid(r, mesh.tC, p, indexing="ij")
    Tb, Pb = np.meshgrid(mesh.tC, p, indexing="ij")
    return (R ** 2, W.mms_forcing(R, T, P)[None], W.mms_solution(mesh.rF[0], Tb, Pb)[None],
            W.mms_solution(mesh.rF[-1], Tb, Pb)[None])


@pytest.mark.parametrize("which", ["rn", "pn"])
@pytest.mark.parametrize("shape", [(16, 24, 32), (33, 17, 66)])
def test_face_pcg_matches_oracle(mp, oracle_mod, which, shape):
    mesh = W.stretched_mesh(*shape, 1.0, 2.0, 4.0)
    o = oracle_mod.Oracle(mesh, 0, 0)
    sh, ap, dg, drhs, V, pcg = oracle_fns(o, which)
    kappa, f, ubi, ubo = mms_at(mesh, which)
    c = np.zeros(sh)
    rhs = drhs(kappa, f, ubi, ubo)
    rc, xo, ito, _, histo = pcg(kappa, c, rhs, np.zeros_like(rhs), 1e-12, 20000)
    pl = mp.MAS_PLACE_R_NODE if which == "rn" else mp.MAS_PLACE_PHI_NODE
    g = mp.Grid(mesh)
    op = mp.Operator(g, 1, dev(kappa), dev(c), 0, 0, placement=pl)
    fd = dev(f)
    op.dirichlet_rhs(dev(ubi), dev(ubo), fd)
    x = torch.zeros((1,) + sh, dtype=torch.float64, device="cuda")
    st, it, rel, hist = op.solve(fd, x, 1e-12, 20000, True)
    assert rc == oracle_mod.OK and st == mp.MAS_OK and abs(it - ito) <= 1, (it, ito)
    assert rel_l2_V(V, host(x), xo) <= 1e-10
    np.testing.assert_allclose(hist[:10], histo[:10], rtol=1e-9, atol=0)


def test_phi_nodes_on_virtual_ranks_and_refusals(mp, oracle_mod):
    mesh = W.stretched_mesh(26, 16, 64, 1.0, 2.0, 4.0)
    o = oracle_mod.Oracle(mesh, 0, 0)
    kappa, f, ubi, ubo = mms_at(mesh, "pn")
    rhs = o.pn_dirichlet_rhs(kappa, f, ubi, ubo)
    rc, xo, ito, _, _ = o.pn_pcg(kappa, np.zeros(o.shape), rhs, np.zeros_like(rhs), 1e-12, 20000)
    vid = mp.virtual_ranks_id(8801)
    res, errs = {}, []

    def rank_main(r):
        try:
            torch.cuda.set_device(0)
            with torch.cuda.stream(torch.cuda.Stream()):
                g = mp.Grid(mesh, dist=(2, r, vid))
                sl = slice(g.i0, g.i0 + g.nl)
                op = mp.Operator(g, 1, dev(kappa[sl]), None, 0, 0, placement=mp.MAS_PLACE_PHI_NODE)
                fd = dev(f[:, sl])
                op.dirichlet_rhs(dev(ubi), dev(ubo), fd)
                x = torch.zeros((1, g.nl) + o.shape[1:], dtype=torch.float64, device="cuda")
                st, it, rel, _ = op.solve(fd, x, 1e-12, 20000)
                torch.cuda.current_stream().synchronize()
                res[r] = (g.i0, g.nl, st, it, x.cpu().numpy())
                # an r-node op needs one rank
                try:
                    mp.Operator(g, 1, dev(np.ones((mesh.shape[0] - 1,) + o.shape[1:])), None, 0, 0,
                                placement=mp.MAS_PLACE_R_NODE)
                    res[("rn", r)] = "created"
                except mp.MasError as e:
                    res[("rn", r)] = e.status
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
    assert res[0][3] == res[1][3] and abs(res[0][3] - ito) <= 1
    xg = np.empty_like(xo)
    for r in range(2):
        i0, nl, st, it, x = res[r]
        assert st == mp.MAS_OK
        xg[:, i0:i0 + nl] = x
    assert rel_l2_V(o.pn_volumes(), xg, xo) <= 1e-10
    # r nodes need one rank: the library refuses them on an r-slab grid
    assert res[("rn", 0)] == mp.MAS_ERR_ARG and res[("rn", 1)] == mp.MAS_ERR_ARG
