"""NEXT-2 theta-node placement with pole unknowns on the GPU
(mas_op_setup_placed(MAS_PLACE_THETA_NODE), k_pole_avg = the paper's per-
radius sum0 reduction) through the C ABI, against the oracle's mas_ref_tn_*
(pinned in tests/test_oracle_tnode_pins.py).

Tolerances (north_star): matvec rel L2_V <= 1e-13 and elementwise
|dy| <= 1e-13 * 2 D max|x|; diagonal / Dirichlet helper 1e-14; PCG at tol:
iterations +-1, x <= 1e-10 (unconditional); fixed iterations: x <= 1e-10.
The pole rows of every GPU output are phi-constant bitwise."""
import math
import threading

import numpy as np
import pytest

from paper_conf_ipps_caplansl23_b200 import workloads as W

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")
_key = [5000]


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


def poles_constant(a):
    for row in (0, -1):
        blk = a[..., row, :]
        if not np.array_equal(blk, np.broadcast_to(blk[..., :1], blk.shape)):
            return False
    return True


SHAPES = [(16, 24, 32), (9, 13, 70), (33, 8, 64), (5, 17, 130), (3, 2, 4)]


@pytest.mark.parametrize("shape", SHAPES)
@pytest.mark.parametrize("ncomp", [1, 3])
@pytest.mark.parametrize("bc", [(0, 1), (0, 0), (1, 1)])
def test_tn_apply_matches_oracle(mp, oracle_mod, shape, ncomp, bc):
    mesh = W.stretched_mesh(*shape)
    sh = (shape[0], shape[1] + 1, shape[2])
    rng = np.random.default_rng(1)
    kappa, c = rng.uniform(0.5, 2.0, size=sh), rng.uniform(0.1, 1.0, size=sh)
    x = W.replicate_poles(W.random_field((ncomp,) + sh, 42))
    g = mp.Grid(mesh)
    op = mp.Operator(g, ncomp, dev(kappa), dev(c), *bc, placement=mp.MAS_PLACE_THETA_NODE)
    y = torch.empty((ncomp,) + sh, dtype=torch.float64, device="cuda")
    op.apply(dev(x), y)
    o = oracle_mod.Oracle(mesh, *bc)
    yo = o.tn_apply(kappa, c, x)
    V = o.tn_volumes()
    yg = host(y)
    assert rel_l2_V(V, yg, yo) <= 1e-13
    scale = 2.0 * o.tn_diag(kappa, c)[None] * np.abs(x).max()
    assert (np.abs(yg - yo) / scale).max() <= 1e-13
    assert poles_constant(yg)
    # diagonal and the Dirichlet helper
    D = torch.empty(sh, dtype=torch.float64, device="cuda")
    op.diag(D)
    np.testing.assert_allclose(host(D), o.tn_diag(kappa, c), rtol=1e-14, atol=0)
    f = W.replicate_poles(rng.standard_normal((ncomp,) + sh))
    ub = W.replicate_poles(rng.standard_normal((ncomp,) + sh[1:]))
    fd = dev(f)
    op.dirichlet_rhs(dev(ub), dev(ub), fd)
    np.testing.assert_allclose(host(fd), o.tn_dirichlet_rhs(kappa, f, ub, ub), rtol=1e-14,
                               atol=1e-14 * np.abs(f).max())
    # the V-weighted dot over theta-node slots
    assert abs(op.dot(dev(x), dev(x)) - o.tn_dot(x, x)) <= 1e-13 * o.tn_dot(x, x)
    op.close()
    g.close()


def tn_solve(mp, prob, tol=None, maxit=None, prof=False):
    g = mp.Grid(prob.mesh)
    op = mp.Operator(g, prob.ncomp, dev(prob.kappa), dev(prob.c), prob.bc_inner, prob.bc_outer,
                     placement=mp.MAS_PLACE_THETA_NODE)
    op.set_profiling(prof)
    f = dev(prob.f)
    if prob.ub_inner is not None:
        op.dirichlet_rhs(dev(prob.ub_inner), None, f)
    x = dev(prob.x0)
    st, it, rel, hist = op.solve(f, x, prob.tol if tol is None else tol,
                                 prob.maxit if maxit is None else maxit, True)
    return st, host(x), it, rel, hist, op, g


def oracle_tn(oracle_mod, prob, tol=None, maxit=None):
    o = oracle_mod.Oracle.for_problem(prob)
    f = o.tn_dirichlet_rhs(prob.kappa, prob.f, prob.ub_inner, prob.ub_outer)
    return o.tn_pcg(prob.kappa, prob.c, f, prob.x0, prob.tol if tol is None else tol,
                    prob.maxit if maxit is None else maxit) + (o.tn_volumes(),)


@pytest.mark.parametrize("shape", [(16, 24, 64), (9, 13, 70), (40, 17, 130)])
def test_tn_pcg_matches_oracle_at_tol(mp, oracle_mod, shape):
    prob = W.tnode_conduction_problem(*shape)
    rc, xo, ito, relo, histo, V = oracle_tn(oracle_mod, prob)
    st, x, it, rel, hist, op, g = tn_solve(mp, prob)
    assert rc == oracle_mod.OK and st == mp.MAS_OK and rel <= prob.tol
    assert abs(it - ito) <= 1, (it, ito)
    assert rel_l2_V(V, x, xo) <= 1e-10
    assert poles_constant(x)
    np.testing.assert_allclose(hist[:10], histo[:10], rtol=1e-9, atol=0)


@pytest.mark.parametrize("k", [1, 2, 7, 40])
def test_tn_pcg_fixed_iterations(mp, oracle_mod, k):
    prob = W.tnode_conduction_problem(12, 16, 32)
    rc, xo, ito, _, _, V = oracle_tn(oracle_mod, prob, tol=0.0, maxit=k)
    st, x, it, rel, hist, op, g = tn_solve(mp, prob, tol=0.0, maxit=k)
    assert st == mp.MAS_NOT_CONVERGED and it == ito == k
    assert rel_l2_V(V, x, xo) <= 1e-10


def test_tn_graph_equals_host_loop_and_refusals(mp, oracle_mod):
    prob = W.tnode_conduction_problem(20, 16, 64)
    a = tn_solve(mp, prob)
    b = tn_solve(mp, prob, prof=True)
    assert (a[0], a[2]) == (b[0], b[2])
    np.testing.assert_array_equal(a[1], b[1])
    np.testing.assert_array_equal(np.asarray(a[4]), np.asarray(b[4]))
    op = a[5]
    with pytest.raises(mp.MasError):
        op.set_single_reduction(True)
    with pytest.raises(mp.MasError):
        op.enable_p2p()
    with pytest.raises(mp.MasError):
        op.set_aniso(dev(np.ones(op.N)), dev(np.zeros(3 * op.N)))
    # a grid without both poles has no theta-node placement
    m = W.stretched_mesh(4, 8, 8)
    tF = np.linspace(0.3, 2.8, 9)
    m.tF, m.tC = tF, 0.5 * (tF[1:] + tF[:-1])
    m.pole_north = m.pole_south = False
    g = mp.Grid(m)
    with pytest.raises(mp.MasError) as e:
        mp.Operator(g, 1, dev(np.ones((4, 9, 8))), None, 0, 1, placement=mp.MAS_PLACE_THETA_NODE)
    assert e.value.status == mp.MAS_ERR_ARG


@pytest.mark.parametrize("P", [2, 3])
def test_tn_virtual_ranks(mp, oracle_mod, P):
    """r-slabs of the theta-node operator on P virtual ranks (the NCCL-loop
    placement of the seams and allreduces; the pole pass is rank-local)."""
    prob = W.tnode_conduction_problem(13 * P, 16, 64, warm=False)
    _key[0] += 1
    vid = mp.virtual_ranks_id(_key[0])
    res, errs = {}, []

    def rank_main(r):
        try:
            torch.cuda.set_device(0)
            with torch.cuda.stream(torch.cuda.Stream()):
                g = mp.Grid(prob.mesh, dist=(P, r, vid))
                sl = slice(g.i0, g.i0 + g.nl)
                op = mp.Operator(g, 1, dev(prob.kappa[sl]), dev(prob.c[sl]), prob.bc_inner,
                                 prob.bc_outer, placement=mp.MAS_PLACE_THETA_NODE)
                f = dev(prob.f[:, sl])
                op.dirichlet_rhs(dev(prob.ub_inner), None, f)
                x = dev(prob.x0[:, sl])
                st, it, rel, _ = op.solve(f, x, prob.tol, prob.maxit)
                torch.cuda.current_stream().synchronize()
                res[r] = (g.i0, g.nl, st, it, x.cpu().numpy())
                op.close()
                g.close()
        except Exception as e:  # noqa: BLE001
            errs.append((r, repr(e)))

    th = [threading.Thread(target=rank_main, args=(r,)) for r in range(P)]
    for t in th:
        t.start()
    for t in th:
        t.join(timeout=600)
    assert not errs, errs
    rc, xo, ito, _, _, V = oracle_tn(oracle_mod, prob)
    its = {res[r][3] for r in range(P)}
    assert len(its) == 1 and abs(its.pop() - ito) <= 1
    xg = np.empty_like(xo)
    for r in range(P):
        i0, nl, st, it, x = res[r]
        assert st == mp.MAS_OK
        xg[:, i0:i0 + nl] = x
    assert rel_l2_V(V, xg, xo) <= 1e-10
