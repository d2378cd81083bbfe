"""GPU <-> oracle parity, through the C ABI (lib/libmaspcg.so) on a B200.

Tolerances (north_star): matvec relative L2_V <= 1e-13; PCG at
the same tol: iteration counts within +-1 and x within 1e-10 relative L2_V;
fixed-iteration mode (tol = 0, maxit = k): x within 1e-10; residual
histories within 1e-9 relative over the first 10 iterations and 2e-2 after
(the oracle's own sensitivity to a 1-ulp perturbation).
"""
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


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a, dtype=np.float64)).cuda()


def host(t):
    torch.cuda.synchronize()
    return t.cpu().numpy()


def rel_l2_V(V, a, b):
    V = V[None] if a.ndim == 4 else V
    return math.sqrt((V * (a - b) ** 2).sum() / max((V * b ** 2).sum(), 1e-300))


def make(mp, mesh, ncomp, kappa, c, bci, bco):
    g = mp.Grid(mesh)
    op = mp.Operator(g, ncomp, dev(kappa), dev(c) if c is not None else None, bci, bco)
    return g, op


SHAPES = [
    (16, 24, 32),    # C1 shape
    (9, 13, 70),     # ragged: theta not a multiple of 8, phi not of 64, odd nr
    (33, 8, 64),     # r crosses several chunks; exactly one tile
    (5, 17, 130),    # several ragged tiles in phi
    (1, 3, 4),       # tiny: one plane
]


def rand_problem(shape, seed):
    rng = np.random.default_rng(seed)
    kappa = rng.uniform(0.5, 2.0, size=shape)
    c = rng.uniform(0.1, 1.0, size=shape)
    return kappa, c


@pytest.mark.parametrize("shape", SHAPES)
@pytest.mark.parametrize("ncomp", [1, 3])
@pytest.mark.parametrize("bc", [(0, 1), (0, 0), (1, 1)])
def test_apply_matches_oracle(mp, oracle_mod, shape, ncomp, bc):
    mesh = W.stretched_mesh(*shape)
    kappa, c = rand_problem(shape, 1)
    x = W.random_field((ncomp,) + shape, 42)
    g, op = make(mp, mesh, ncomp, kappa, c, *bc)
    y = torch.empty((ncomp,) + shape, dtype=torch.float64, device="cuda")
    op.apply(dev(x), y)
    o = oracle_mod.Oracle(mesh, *bc)
    yo = o.apply(kappa, c, x)
    V = o.volumes()
    yg = host(y)
    assert rel_l2_V(V, yg, yo) <= 1e-13
    # elementwise: |L x| <= (c + 2 sum_f G_f / V) max|x| <= 2 D_P max|x|, so the
    # per-cell error is bounded relative to that cell's own scale (V spans
    # ~1e5 on these meshes, which the V-weighted norm alone would hide)
    scale = 2.0 * o.diag(kappa, c)[None] * np.abs(x).max()
    assert (np.abs(yg - yo) / scale).max() <= 1e-13
    # host-pointer path of the same ABI call
    yh = np.empty_like(x)
    op.apply(np.ascontiguousarray(x), yh)
    assert rel_l2_V(V, yh, yo) <= 1e-13
    assert (np.abs(yh - yo) / scale).max() <= 1e-13


@pytest.mark.parametrize("shape", SHAPES[:3])
def test_diag_dirichlet_rhs_dot(mp, oracle_mod, shape):
    mesh = W.stretched_mesh(*shape)
    kappa, c = rand_problem(shape, 2)
    g, op = make(mp, mesh, 1, kappa, c, 0, 0)
    o = oracle_mod.Oracle(mesh, 0, 0)
    D = torch.empty(shape, dtype=torch.float64, device="cuda")
    op.diag(D)
    np.testing.assert_allclose(host(D), o.diag(kappa, c), rtol=1e-14, atol=0)
    rng = np.random.default_rng(3)
    f = rng.standard_normal((1,) + shape)
    ubi = rng.standard_normal((1,) + shape[1:])
    ubo = rng.standard_normal((1,) + shape[1:])
    fd = dev(f)
    op.dirichlet_rhs(dev(ubi), dev(ubo), fd)
    np.testing.assert_allclose(host(fd), o.dirichlet_rhs(kappa, f, ubi, ubo), rtol=1e-14,
                               atol=1e-14 * np.abs(f).max())
    a, b = rng.standard_normal((2, 1) + shape)
    assert abs(op.dot(dev(a), dev(b)) - o.dot(a, b)) <= 1e-13 * math.sqrt(o.dot(a, a) * o.dot(b, b))


def test_setup_rejects_bad_coefficients(mp):
    mesh = W.stretched_mesh(4, 8, 8)
    kappa, c = rand_problem((4, 8, 8), 4)
    g = mp.Grid(mesh)
    bad = kappa.copy()
    bad[1, 2, 3] = -1.0
    with pytest.raises(mp.MasError) as e:
        mp.Operator(g, 1, dev(bad), dev(c), 0, 1)
    assert e.value.status == mp.MAS_ERR_ARG
    bad = c.copy()
    bad[0, 0, 0] = float("nan")
    with pytest.raises(mp.MasError):
        mp.Operator(g, 1, dev(kappa), dev(bad), 0, 1)
    # kappa = 0 with c = 0 and Neumann-Neumann => D = 0
    with pytest.raises(mp.MasError):
        mp.Operator(g, 1, dev(np.zeros_like(kappa)), None, 1, 1)


def gpu_solve(mp, prob, tol=None, maxit=None, x0=None, want_hist=True):
    g, op = make(mp, prob.mesh, prob.ncomp, prob.kappa, prob.c, prob.bc_inner, prob.bc_outer)
    f = dev(prob.f)
    ubi = dev(prob.ub_inner) if prob.ub_inner is not None else None
    ubo = dev(prob.ub_outer) if prob.ub_outer is not None else None
    if ubi is not None or ubo is not None:
        op.dirichlet_rhs(ubi, ubo, f)
    x = dev(prob.x0 if x0 is None else x0)
    st, it, rel, hist = op.solve(f, x, prob.tol if tol is None else tol,
                                 prob.maxit if maxit is None else maxit, want_hist)
    return st, host(x), it, rel, hist, op


def small_problems():
    return [
        W.mms_problem(16, 24, 32),
        W.conduction_problem(16, 24, 64),
        W.viscosity_problem(16, 24, 64),
        W.conduction_problem(9, 13, 70, warm=False),
        W.viscosity_problem(33, 8, 66, warm=False),
    ]


@pytest.mark.parametrize("idx", range(5))
def test_pcg_matches_oracle_at_tol(mp, oracle_mod, idx):
    prob = small_problems()[idx]
    rc, xo, ito, relo, histo = oracle_mod.solve_problem(prob)
    st, x, it, rel, hist, op = gpu_solve(mp, prob)
    assert rc == oracle_mod.OK and st == mp.MAS_OK
    assert abs(it - ito) <= 1, (it, ito)
    assert rel <= prob.tol
    V = oracle_mod.Oracle.for_problem(prob).volumes()
    assert rel_l2_V(V, x, xo) <= 1e-10  # unconditional (north_star: x <= 1e-10)
    # Residual histories: CG amplifies rounding differences; the oracle run
    # against itself with a 1e-16 relative perturbation of f already differs
    # by 1e-4..3e-3 after ~20 iterations on these stiff problems (DESIGN.md
    # §6.2).  So: 1e-9 over the first 10 iterations; after that within 4x the
    # oracle's own envelope on this very problem, the running max over four
    # independently perturbed oracle solves (one perturbation alone samples
    # the rounding spread too thinly for a tight factor).
    n = min(len(hist), len(histo))
    np.testing.assert_allclose(hist[:10], histo[:10], rtol=1e-9, atol=0)
    f0 = prob.f.copy()
    env = np.zeros(n)
    for seed in (7, 8, 9, 10):
        prob.f = f0 * (1.0 + 1e-16 * np.random.default_rng(seed).standard_normal(f0.shape))
        _, _, _, _, histp = oracle_mod.solve_problem(prob)
        m = min(n, len(histp))
        env[:m] = np.maximum(env[:m], np.abs(histp[:m] - histo[:m]) / histo[:m])
    prob.f = f0
    env = np.maximum.accumulate(env)
    dev_ = np.abs(hist[:n] - histo[:n]) / histo[:n]
    assert (dev_ <= 4.0 * env + 1e-9).all(), (dev_.max(), env.max(), (dev_ / (env + 1e-30)).max())


@pytest.mark.parametrize("k", [1, 2, 7, 40])
def test_pcg_fixed_iterations(mp, oracle_mod, k):
    prob = W.viscosity_problem(12, 16, 32)
    rc, xo, ito, _, _ = oracle_mod.solve_problem(prob, tol=0.0, maxit=k)
    st, x, it, rel, hist, _ = gpu_solve(mp, prob, tol=0.0, maxit=k)
    assert rc == oracle_mod.NOT_CONVERGED and st == mp.MAS_NOT_CONVERGED
    assert it == ito == k
    V = oracle_mod.Oracle.for_problem(prob).volumes()
    assert rel_l2_V(V, x, xo) <= 1e-10
    # the host-driven loop (profiling on) reaches the same maxit decision, bitwise
    g2, op2 = make(mp, prob.mesh, prob.ncomp, prob.kappa, prob.c, prob.bc_inner, prob.bc_outer)
    f2 = dev(prob.f)
    if prob.ub_inner is not None or prob.ub_outer is not None:
        op2.dirichlet_rhs(dev(prob.ub_inner) if prob.ub_inner is not None else None,
                          dev(prob.ub_outer) if prob.ub_outer is not None else None, f2)
    op2.set_profiling(True)
    x2 = dev(prob.x0)
    st2, it2, _, hist2 = op2.solve(f2, x2, 0.0, k, True)
    assert (st2, it2) == (st, it)
    np.testing.assert_array_equal(host(x2), x)
    np.testing.assert_array_equal(np.asarray(hist2), np.asarray(hist))


def test_pcg_edge_cases(mp, oracle_mod):
    prob = W.conduction_problem(8, 16, 32)
    # zero rhs -> x = 0, 0 iterations
    prob.f[:] = 0.0
    prob.ub_inner = None
    st, x, it, rel, hist, _ = gpu_solve(mp, prob)
    assert st == mp.MAS_OK and it == 0 and (x == 0).all()
    # maxit = 0 with a nonzero residual -> NOT_CONVERGED, x unchanged
    prob = W.conduction_problem(8, 16, 32)
    st, x, it, rel, hist, _ = gpu_solve(mp, prob, maxit=0)
    assert st == mp.MAS_NOT_CONVERGED and it == 0
    np.testing.assert_array_equal(x, prob.x0)
    # exact start: x0 = oracle solution at tol 1e-14 -> stops at k = 0 with tol 1e-8
    rc, xo, _, _, _ = oracle_mod.solve_problem(prob, tol=1e-14)
    st, x, it, rel, hist, _ = gpu_solve(mp, prob, tol=1e-8, x0=xo)
    assert st == mp.MAS_OK and it == 0


def test_mass_only_one_iteration(mp):
    shape = (6, 10, 20)
    mesh = W.stretched_mesh(*shape)
    c = np.random.default_rng(5).uniform(0.1, 3, size=shape)
    f = np.random.default_rng(6).standard_normal((3,) + shape)
    g = mp.Grid(mesh)
    op = mp.Operator(g, 3, dev(np.zeros(shape)), dev(c), 0, 1)
    x = torch.zeros((3,) + shape, dtype=torch.float64, device="cuda")
    st, it, rel, _ = op.solve(dev(f), x, 1e-12, 50)
    assert st == mp.MAS_OK and it == 1
    np.testing.assert_allclose(host(x), f / c[None], rtol=4e-16, atol=0)


def test_host_pointer_solve_equals_device_solve(mp):
    prob = W.conduction_problem(10, 16, 32)
    st, xd, it, rel, _, op = gpu_solve(mp, prob)
    f = np.ascontiguousarray(prob.f).copy()
    op.dirichlet_rhs(prob.ub_inner, None, f)
    xh = np.ascontiguousarray(prob.x0).copy()
    st2, it2, rel2, _ = op.solve(f, xh, prob.tol, prob.maxit)
    assert (st2, it2) == (st, it)
    np.testing.assert_array_equal(xh, xd)


def test_deterministic_repeat(mp):
    prob = W.viscosity_problem(12, 16, 64)
    a = gpu_solve(mp, prob)
    b = gpu_solve(mp, prob)
    assert a[2] == b[2]
    np.testing.assert_array_equal(a[1], b[1])


@pytest.mark.parametrize("mk", ["viscosity", "conduction"])
def test_p2p_transport_one_rank_is_bitwise_identical(mp, mk):
    """mas_op_enable_p2p on one GPU: the mailbox allreduce runs against the
    rank itself inside the CUDA-graph loop (0 + v = v exactly), so the solve
    must be bit-identical to the plain path, over repeated solves (epochs)."""
    prob = (W.viscosity_problem(12, 16, 64) if mk == "viscosity" else
            W.conduction_problem(10, 16, 32))
    st, xd, it, rel, hist, op = gpu_solve(mp, prob)
    op.enable_p2p()
    assert op.transport == "p2p"
    f = dev(prob.f)
    op.dirichlet_rhs(None if prob.ub_inner is None else dev(prob.ub_inner), None, f)
    for _ in range(3):
        x = dev(prob.x0)
        st2, it2, rel2, hist2 = op.solve(f, x, prob.tol, prob.maxit, True)
        assert (st2, it2, rel2) == (st, it, rel)
        np.testing.assert_array_equal(host(x), xd)
        np.testing.assert_array_equal(np.asarray(hist2), np.asarray(hist))
    # fixed-iteration and zero-rhs paths through the mailbox
    x = dev(prob.x0)
    assert op.solve(f, x, 0.0, 5)[:2] == (mp.MAS_NOT_CONVERGED, 5)
    z = torch.zeros_like(f)
    st3, it3, _, _ = op.solve(z, x, prob.tol, prob.maxit)
    assert (st3, it3) == (mp.MAS_OK, 0) and float(x.abs().max()) == 0.0


@pytest.mark.parametrize("mk", ["viscosity", "conduction", "mms"])
def test_graph_loop_equals_host_loop_bitwise(mp, mk):
    """The single-GPU solve runs as one CUDA graph (device-side while node);
    with profiling on, the same kernels are launched one by one from the
    host.  Both must give the same bits, iteration count and history."""
    prob = {"viscosity": lambda: W.viscosity_problem(20, 16, 64),
            "conduction": lambda: W.conduction_problem(40, 16, 32),
            "mms": lambda: W.mms_problem(16, 24, 32)}[mk]()
    st, xg, it, rel, hist, op = gpu_solve(mp, prob)
    f = dev(prob.f)
    ubi = dev(prob.ub_inner) if prob.ub_inner is not None else None
    ubo = dev(prob.ub_outer) if prob.ub_outer is not None else None
    if ubi is not None or ubo is not None:
        op.dirichlet_rhs(ubi, ubo, f)
    op.set_profiling(True)
    x = dev(prob.x0)
    st2, it2, rel2, hist2 = op.solve(f, x, prob.tol, prob.maxit, True)
    assert (st2, it2, rel2) == (st, it, rel)
    np.testing.assert_array_equal(host(x), xg)
    np.testing.assert_array_equal(np.asarray(hist2), np.asarray(hist))
