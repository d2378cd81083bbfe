"""GPU <-> oracle parity of the field-aligned conduction term L_par (SURVEY.md
§8(f) NEXT-4, readings R21-R26), through the C ABI on a B200.

Same bars as the isotropic path: apply relative L2_V <= 1e-13,
diagonal <= 1e-13, PCG iterations +-1 and x <= 1e-10 at the same tol,
fixed-iteration x <= 1e-10.  The oracle evaluates W kpar (b.g)(b.dg) per
corner; the library precomputes sqrt(W kpar) b / (4 h) per corner, so the two
agree to rounding, not bitwise.
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


SHAPES = [
    (16, 24, 32),
    (9, 13, 70),     # ragged theta / phi tiles, odd nr
    (33, 8, 64),     # several r chunks, one tile
    (5, 17, 130),    # several ragged phi tiles
    (2, 3, 4),       # tiny
]


def rand_fields(shape, seed):
    rng = np.random.default_rng(seed)
    kappa = rng.uniform(0.5, 2.0, size=shape)
    c = rng.uniform(0.1, 1.0, size=shape)
    kpar = rng.uniform(0.5, 4.0, size=shape)
    b = rng.standard_normal((3,) + shape)
    b /= np.linalg.norm(b, axis=0)
    return kappa, c, kpar, b


def setup(mp, mesh, kappa, c, kpar, b, bc=(0, 1)):
    g = mp.Grid(mesh)
    op = mp.Operator(g, 1, dev(kappa), dev(c), *bc)
    op.set_aniso(dev(kpar), dev(b))
    return g, op


@pytest.mark.parametrize("shape", SHAPES)
@pytest.mark.parametrize("bc", [(0, 1), (0, 0)])
def test_apply_and_diag_match_oracle(mp, oracle_mod, shape, bc):
    mesh = W.stretched_mesh(*shape)
    kappa, c, kpar, b = rand_fields(shape, 1)
    g, op = setup(mp, mesh, kappa, c, kpar, b, bc)
    x = W.random_field((1,) + shape, 42)
    y = torch.empty((1,) + shape, dtype=torch.float64, device="cuda")
    op.apply(dev(x), y)
    o = oracle_mod.Oracle(mesh, *bc)
    yo = o.apply(kappa, c, x) + o.aniso_apply(kpar, b, x)
    V = o.volumes()
    assert rel_l2_V(V, host(y), yo) <= 1e-13
    # the L_par part alone (kappa = 0, c = 0 except a tiny mass for D > 0)
    D = torch.empty(shape, dtype=torch.float64, device="cuda")
    op.diag(D)
    Do = o.diag(kappa, c) + o.aniso_diag(kpar, b)
    np.testing.assert_allclose(host(D), Do, rtol=1e-13, atol=0)


@pytest.mark.parametrize("shape", [(16, 24, 64), (24, 20, 70), (40, 32, 128), (7, 40, 192)])
def test_apply_repeatable_and_per_cell(mp, oracle_mod, shape):
    """Race sentinel for k_aniso's shared-memory hand-offs (the two-parity
    corner-row exchange between consumer warps, the halo warp's extra column,
    the ring slot released before the consumer barrier): 30 repeated applies
    are bitwise identical, and every cell of c x + L_par x is within 1e-12 of
    a local scale of the oracle: 2 max|x| times the largest diagonal D_Q of
    the cell's 27-cell neighbourhood (the V-weighted operator is a Gram
    matrix, so |L_PQ| <= sqrt(V_Q/V_P) sqrt(D_P D_Q); a stale or half-written
    value in one cell is an O(1) error there, even where the V-weighted norm
    hides it).
    Shapes: one phi tile (64), a ragged phi tile (70 = 64 + 6), ragged theta
    tiles, several tiles per block segment (192 = 3 phi tiles)."""
    mesh = W.stretched_mesh(*shape)
    _, c, kpar, b = rand_fields(shape, 3)
    kappa = np.zeros(shape)
    g, op = setup(mp, mesh, kappa, c, kpar, b)
    xh = W.random_field((1,) + shape, 11)
    x = dev(xh)
    y0 = torch.empty_like(x)
    op.apply(x, y0)
    for _ in range(30):
        y = torch.empty_like(x)
        op.apply(x, y)
        assert torch.equal(y, y0)
    o = oracle_mod.Oracle(mesh, 0, 1)
    yo = o.apply(kappa, c, xh) + o.aniso_apply(kpar, b, xh)
    D = o.diag(kappa, c) + o.aniso_diag(kpar, b)
    Dp = np.pad(D, ((1, 1), (1, 1), (0, 0)), mode="edge")
    Dp = np.concatenate([Dp[:, :, -1:], Dp, Dp[:, :, :1]], axis=2)  # periodic phi
    n0, n1, n2 = shape
    Dn = np.max([Dp[a:a + n0, b_:b_ + n1, e:e + n2] for a in range(3) for b_ in range(3) for e in range(3)],
                axis=0)
    scale = 2.0 * Dn[None] * np.abs(xh).max()
    assert (np.abs(host(y0) - yo) / scale).max() <= 1e-12


def test_pure_field_aligned_apply(mp, oracle_mod):
    """kappa = 0: the result is c x + L_par x alone (no 7-point term to hide a
    wrong corner term behind)."""
    shape = (12, 20, 70)
    mesh = W.stretched_mesh(*shape)
    _, c, kpar, b = rand_fields(shape, 2)
    kappa = np.zeros(shape)
    g, op = setup(mp, mesh, kappa, c, kpar, b)
    x = W.random_field((1,) + shape, 7)
    y = torch.empty((1,) + shape, dtype=torch.float64, device="cuda")
    op.apply(dev(x), y)
    o = oracle_mod.Oracle(mesh, 0, 1)
    yo = c[None] * x + o.aniso_apply(kpar, b, x)
    assert rel_l2_V(o.volumes(), host(y), yo) <= 1e-13


def test_switch_off_restores_isotropic_operator(mp, oracle_mod):
    shape = (8, 16, 64)
    mesh = W.stretched_mesh(*shape)
    kappa, c, kpar, b = rand_fields(shape, 3)
    g, op = setup(mp, mesh, kappa, c, kpar, b)
    op.set_aniso(None, None)
    x = W.random_field((1,) + shape, 8)
    y = torch.empty((1,) + shape, dtype=torch.float64, device="cuda")
    op.apply(dev(x), y)
    o = oracle_mod.Oracle(mesh, 0, 1)
    assert rel_l2_V(o.volumes(), host(y), o.apply(kappa, c, x)) <= 1e-13
    D = torch.empty(shape, dtype=torch.float64, device="cuda")
    op.diag(D)
    np.testing.assert_allclose(host(D), o.diag(kappa, c), rtol=1e-14, atol=0)


def test_host_pointer_inputs_bitwise_equal(mp):
    shape = (8, 16, 64)
    mesh = W.stretched_mesh(*shape)
    kappa, c, kpar, b = rand_fields(shape, 4)
    g, op = setup(mp, mesh, kappa, c, kpar, b)
    g2 = mp.Grid(mesh)
    op2 = mp.Operator(g2, 1, dev(kappa), dev(c), 0, 1)
    op2.set_aniso(np.ascontiguousarray(kpar), np.ascontiguousarray(b))
    x = dev(W.random_field((1,) + shape, 9))
    y1 = torch.empty_like(x)
    y2 = torch.empty_like(x)
    op.apply(x, y1)
    op2.apply(x, y2)
    assert torch.equal(y1, y2)


def test_rejects_bad_inputs(mp):
    shape = (6, 8, 16)
    mesh = W.stretched_mesh(*shape)
    kappa, c, kpar, b = rand_fields(shape, 5)
    g = mp.Grid(mesh)
    op3 = mp.Operator(g, 3, dev(kappa), dev(c), 0, 1)
    with pytest.raises(mp.MasError) as e:
        op3.set_aniso(dev(kpar), dev(b))
    assert e.value.status == mp.MAS_ERR_ARG
    op = mp.Operator(g, 1, dev(kappa), dev(c), 0, 1)
    bad = kpar.copy()
    bad[3, 4, 5] = -1.0
    with pytest.raises(mp.MasError):
        op.set_aniso(dev(bad), dev(b))
    bb = b.copy()
    bb[1, 2, 3, 4] = np.nan
    with pytest.raises(mp.MasError):
        op.set_aniso(dev(kpar), dev(bb))
    # boundary-corner entries (i = 0 or j = 0) are ignored (R25)
    kk = kpar.copy()
    kk[0, :, :] = -5.0
    kk[:, 0, :] = np.nan
    op.set_aniso(dev(kk), dev(b))


def _solve_pair(mp, oracle_mod, prob, tol, maxit, prof=False):
    g = mp.Grid(prob.mesh)
    op = mp.Operator(g, 1, dev(prob.kappa), dev(prob.c), prob.bc_inner, prob.bc_outer)
    op.set_aniso(dev(prob.kpar), dev(prob.bhat))
    if prof:
        op.set_profiling(True)
    f = dev(prob.f)
    op.dirichlet_rhs(dev(prob.ub_inner) if prob.ub_inner is not None else None, None, f)
    x = dev(prob.x0)
    st, it, rel, hist = op.solve(f, x, tol, maxit, want_hist=True)
    rc, xo, ito, relo, histo = oracle_mod.solve_problem(prob, tol=tol, maxit=maxit)
    return st, it, host(x), hist, rc, xo, ito, histo, op


@pytest.mark.parametrize("shape", [(16, 16, 32), (24, 20, 70), (40, 32, 128)])
def test_pcg_matches_oracle(mp, oracle_mod, shape):
    prob = W.aniso_conduction_problem(*shape)
    st, it, x, hist, rc, xo, ito, histo, _ = _solve_pair(mp, oracle_mod, prob, 1e-12, 20000)
    assert st == mp.MAS_OK and rc == oracle_mod.OK
    assert abs(it - ito) <= 1, (it, ito)
    V = oracle_mod.Oracle.for_problem(prob).volumes()
    assert rel_l2_V(V, x, xo) <= 1e-10  # unconditional (north_star: x <= 1e-10)
    n = min(10, len(hist), len(histo))
    np.testing.assert_allclose(hist[:n], histo[:n], rtol=1e-9)


@pytest.mark.parametrize("k", [1, 2, 7, 40])
def test_fixed_iterations_match_oracle(mp, oracle_mod, k):
    prob = W.aniso_conduction_problem(16, 24, 64)
    st, it, x, hist, rc, xo, ito, histo, _ = _solve_pair(mp, oracle_mod, prob, 0.0, k)
    assert it == ito == k
    V = oracle_mod.Oracle.for_problem(prob).volumes()
    assert rel_l2_V(V, x, xo) <= 1e-10


def test_graph_loop_equals_host_loop_bitwise(mp, oracle_mod):
    """The profiled solve runs the host-driven loop (A, L_par, B per
    iteration with events); the default runs the CUDA-graph while loop."""
    prob = W.aniso_conduction_problem(16, 24, 64)
    a = _solve_pair(mp, oracle_mod, prob, 1e-12, 5000, prof=False)
    b = _solve_pair(mp, oracle_mod, prob, 1e-12, 5000, prof=True)
    assert a[1] == b[1]
    assert np.array_equal(a[2], b[2])
    assert b[8].aniso_time() > 0.0


@pytest.mark.parametrize("shape", [(1, 8, 16), (6, 1, 16), (5, 6, 2), (3, 2, 130)])
def test_degenerate_grids(mp, oracle_mod, shape):
    """One r-plane or one theta row: every corner is on the boundary, L_par = 0;
    np = 2: the phi-wrap boxes cover the whole row; a 2-row theta band with a
    ragged phi tile.  Apply and diagonal against the oracle."""
    mesh = W.stretched_mesh(*shape)
    kappa, c, kpar, b = rand_fields(shape, 21)
    g, op = setup(mp, mesh, kappa, c, kpar, b)
    x = W.random_field((1,) + shape, 22)
    y = torch.empty((1,) + shape, dtype=torch.float64, device="cuda")
    op.apply(dev(x), y)
    o = oracle_mod.Oracle(mesh, 0, 1)
    yo = o.apply(kappa, c, x) + o.aniso_apply(kpar, b, x)
    assert rel_l2_V(o.volumes(), host(y), yo) <= 1e-13
    if shape[0] == 1 or shape[1] == 1:
        assert np.array_equal(o.aniso_apply(kpar, b, x), np.zeros_like(x))
    D = torch.empty(shape, dtype=torch.float64, device="cuda")
    op.diag(D)
    np.testing.assert_allclose(host(D), o.diag(kappa, c) + o.aniso_diag(kpar, b), rtol=1e-13, atol=0)


def test_aniso_on_the_p2p_mailbox_loop_one_gpu(mp, oracle_mod):
    """The P2P transport on one GPU (the mailbox runs against itself, the loop
    is one CUDA graph): kernel A publishes its sigma to slot A, k_aniso its
    part to slot C, kernel B sums both; the init sums come from k_aniso<RESID>.
    Bitwise equal to the plain single-GPU loop (both add the two parts in the
    same order), and the oracle's iteration count."""
    prob = W.aniso_conduction_problem(16, 24, 64)
    a = _solve_pair(mp, oracle_mod, prob, 1e-12, 5000)
    g = mp.Grid(prob.mesh)
    op = mp.Operator(g, 1, dev(prob.kappa), dev(prob.c), prob.bc_inner, prob.bc_outer)
    op.enable_p2p()
    op.set_aniso(dev(prob.kpar), dev(prob.bhat))
    f = dev(prob.f)
    op.dirichlet_rhs(dev(prob.ub_inner), None, f)
    for _ in range(2):  # repeated solves: mailbox epochs
        x = dev(prob.x0)
        st, it, rel, _ = op.solve(f, x, 1e-12, 5000)
        assert st == mp.MAS_OK and it == a[1]
        assert np.array_equal(host(x), a[2])


@pytest.mark.parametrize("shape", [(16, 24, 64), (24, 20, 70)])
def test_fused_lpar_kernel_matches_oracle(mp, oracle_mod, shape, monkeypatch):
    """The opt-in fused form (MAS_LPAR_FUSED=1: the iteration's L_par inside
    kernel A, corners staged per plane with the diagonal halo cells): PCG
    against the oracle (+-1, x <= 1e-10), graph == host loop bitwise, and the
    fixed-iteration iterates (k = 7) within 1e-10."""
    monkeypatch.setenv("MAS_LPAR_FUSED", "1")
    prob = W.aniso_conduction_problem(*shape)
    a = _solve_pair(mp, oracle_mod, prob, 1e-12, 5000, prof=False)
    assert a[8].aniso_fused
    b = _solve_pair(mp, oracle_mod, prob, 1e-12, 5000, prof=True)
    assert a[1] == b[1]
    assert np.array_equal(a[2], b[2])
    rc, xo, ito, _, _ = oracle_mod.solve_problem(prob)
    V = oracle_mod.Oracle.for_problem(prob).volumes()
    assert abs(a[1] - ito) <= 1
    assert rel_l2_V(V, a[2], xo) <= 1e-10
    rc, xo7, ito7, _, _ = oracle_mod.solve_problem(prob, tol=0.0, maxit=7)
    c = _solve_pair(mp, oracle_mod, prob, 0.0, 7, prof=False)
    assert c[1] == 7 and rel_l2_V(V, c[2], xo7) <= 1e-10
