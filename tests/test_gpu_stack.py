"""NEXT-2 staggered viscosity step as ONE solve on the GPU (mas_stack_*,
reading R34): v_r at r nodes, v_theta at theta nodes (pole unknowns), v_phi at
phi nodes, each its own operator, one PCG on the stacked vector with the
summed inner products -- against the oracle's mas_ref_stacked_pcg_solve
(pinned in tests/test_oracle_stacked_pins.py).

Tolerances (north_star): at tol, iterations within max(1, the oracle's own
1-ulp sensitivity) and x <= 1e-10 in the stacked V-norm (unconditional); at a
fixed iteration count x <= 1e-10.  Structural checks are bitwise: one block =
mas_pcg_solve, two identical blocks = one block, graph loop = host loop,
repeated solves through the cached graph."""
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


def pshape(shape, pl):
    nr, nt, np_ = shape
    return {0: (nr, nt, np_), 1: (nr, nt + 1, np_), 2: (nr - 1, nt, np_), 3: (nr, nt, np_)}[pl]


def make_blocks(shape, spec, seed=0):
    """spec: [(placement, ncomp, bc)] -> per block (placement, ncomp, bc, kappa,
    c, f, x0) on the stretched mesh of `shape`; blocks scaled differently."""
    out = []
    for q, (pl, ncomp, bc) in enumerate(spec):
        sh = pshape(shape, pl)
        rng = np.random.default_rng(seed + 10 * q)
        kappa = rng.uniform(0.5, 2.0, size=sh) * 4.0 ** q
        c = rng.uniform(0.1, 1.0, size=sh)
        f = rng.standard_normal((ncomp,) + sh) * 2.0 ** q
        x0 = 0.1 * rng.standard_normal((ncomp,) + sh)
        if pl == 1:
            c, f, x0 = W.replicate_poles(c), W.replicate_poles(f), W.replicate_poles(x0)
        out.append((pl, ncomp, bc, kappa, c, f, x0))
    return out


def gpu_stack(mp, mesh, blocks, tol, maxit, hist=False):
    g = mp.Grid(mesh)
    ops = [mp.Operator(g, nc, dev(k), dev(c), *bc, placement=pl) for pl, nc, bc, k, c, f, x0 in blocks]
    sk = mp.Stack(ops)
    xs = [dev(b[6]) for b in blocks]
    st, it, rel, h = sk.solve([dev(b[5]) for b in blocks], xs, tol, maxit, hist)
    out = [host(x) for x in xs]
    sk.close()
    for o in ops:
        o.close()
    g.close()
    return st, it, rel, out, h


def oracle_stack(om, mesh, blocks, tol, maxit, fscale=None):
    ob = []
    for q, (pl, nc, bc, kappa, c, f, x0) in enumerate(blocks):
        ff = f if fscale is None else f * fscale[q]
        ob.append((om.Oracle(mesh, *bc), pl, kappa, c, ff, x0))
    return om.stacked_pcg(ob, tol, maxit), ob


def volumes(om, ob):
    out = []
    for o, pl, *_ in ob:
        out.append({0: o.volumes, 1: o.tn_volumes, 2: o.rn_volumes, 3: o.pn_volumes}[pl]()[None])
    return out


def stacked_rel(V, xg, xo):
    num = sum((v * (a - b) ** 2).sum() for v, a, b in zip(V, xg, xo))
    den = sum((v * b ** 2).sum() for v, b in zip(V, xo))
    return math.sqrt(num / den)


STAGGERED = [(2, 1, (0, 0)), (1, 1, (0, 1)), (3, 1, (0, 1))]  # v_r, v_theta, v_phi


@pytest.mark.parametrize("shape", [(16, 24, 32), (9, 13, 70), (33, 8, 64), (4, 3, 4)])
def test_staggered_stack_vs_oracle(mp, oracle_mod, shape):
    mesh = W.stretched_mesh(*shape)
    blocks = make_blocks(shape, STAGGERED, seed=shape[0])
    tol, maxit = 1e-10, 5000
    st, it, rel, xg, hist = gpu_stack(mp, mesh, blocks, tol, maxit, hist=True)
    (rc, xo, ito, relo, histo), ob = oracle_stack(oracle_mod, mesh, blocks, tol, maxit)
    assert st == mp.MAS_OK and rc == oracle_mod.OK and rel <= tol
    env = 0
    for sd in range(2):
        rng = np.random.default_rng(100 + sd)
        fs = [1.0 + 1e-16 * rng.standard_normal()] * len(blocks)
        (_, _, itp, _, _), _ = oracle_stack(oracle_mod, mesh, blocks, tol, maxit, fscale=fs)
        env = max(env, abs(itp - ito))
    assert abs(it - ito) <= max(1, env), (it, ito, env)
    assert stacked_rel(volumes(oracle_mod, ob), xg, xo) <= 1e-10
    np.testing.assert_allclose(hist[0], histo[0], rtol=1e-12)
    for b, x in zip(blocks, xg):  # theta nodes: the pole rows stay one value per radius
        if b[0] == 1:
            for row in (0, -1):
                assert np.array_equal(x[..., row, :], np.broadcast_to(x[..., row, :1], x[..., row, :].shape))


def test_mixed_stack_fixed_iterations_vs_oracle(mp, oracle_mod):
    """cell-centred 3-component block + phi-node block + r-node 3-component
    block, 7 iterations exactly (tol 0): x <= 1e-10 of the oracle's 7th
    iterate, NOT_CONVERGED from both."""
    shape = (12, 16, 64)
    mesh = W.stretched_mesh(*shape)
    blocks = make_blocks(shape, [(0, 3, (0, 1)), (3, 1, (1, 1)), (2, 3, (0, 0))], seed=5)
    st, it, rel, xg, _ = gpu_stack(mp, mesh, blocks, 0.0, 7)
    (rc, xo, ito, _, _), ob = oracle_stack(oracle_mod, mesh, blocks, 0.0, 7)
    assert st == mp.MAS_NOT_CONVERGED and rc == oracle_mod.NOT_CONVERGED and it == ito == 7
    assert stacked_rel(volumes(oracle_mod, ob), xg, xo) <= 1e-10


def test_one_block_is_mas_pcg_solve_bitwise(mp):
    shape = (20, 16, 64)
    mesh = W.stretched_mesh(*shape)
    for spec in ([(1, 1, (0, 1))], [(0, 3, (0, 1))], [(2, 1, (0, 0))]):
        blocks = make_blocks(shape, spec, seed=7)
        st, it, rel, xg, h = gpu_stack(mp, mesh, blocks, 1e-11, 3000, hist=True)
        pl, nc, bc, k, c, f, x0 = blocks[0]
        g = mp.Grid(mesh)
        op = mp.Operator(g, nc, dev(k), dev(c), *bc, placement=pl)
        x = dev(x0)
        st1, it1, rel1, h1 = op.solve(dev(f), x, 1e-11, 3000, True)
        assert (st, it, rel) == (st1, it1, rel1)
        assert np.array_equal(xg[0], host(x)) and np.array_equal(h, h1)
        op.close()
        g.close()


def test_two_identical_blocks_are_one_block_bitwise(mp):
    shape = (16, 24, 64)
    mesh = W.stretched_mesh(*shape)
    one = make_blocks(shape, [(3, 1, (0, 1))], seed=9)
    st1, it1, _, x1, _ = gpu_stack(mp, mesh, one, 1e-11, 3000)
    st2, it2, _, x2, _ = gpu_stack(mp, mesh, one + one, 1e-11, 3000)
    assert st1 == st2 == mp.MAS_OK and it1 == it2
    assert np.array_equal(x2[0], x1[0]) and np.array_equal(x2[1], x1[0])


def test_graph_loop_equals_host_loop_and_repeats(mp, monkeypatch):
    shape = (16, 24, 32)
    mesh = W.stretched_mesh(*shape)
    blocks = make_blocks(shape, STAGGERED, seed=11)
    a = gpu_stack(mp, mesh, blocks, 1e-10, 3000, hist=True)
    monkeypatch.setenv("MAS_NO_GRAPH", "1")  # read at operator setup
    b = gpu_stack(mp, mesh, blocks, 1e-10, 3000, hist=True)
    monkeypatch.delenv("MAS_NO_GRAPH")
    assert a[:3] == b[:3]
    for xa, xb in zip(a[3], b[3]):
        assert np.array_equal(xa, xb)
    assert np.array_equal(a[4], b[4])
    # repeated solves through one stack (the cached graph), and a moved x
    g = mp.Grid(mesh)
    ops = [mp.Operator(g, nc, dev(k), dev(c), *bc, placement=pl) for pl, nc, bc, k, c, f, x0 in blocks]
    sk = mp.Stack(ops)
    rhs = [dev(bk[5]) for bk in blocks]
    for rep in range(3):
        xs = [dev(bk[6]) for bk in blocks]
        st, it, rel, _ = sk.solve(rhs, xs, 1e-10, 3000)
        assert (st, it, rel) == a[:3]
        for xd, xa in zip(xs, a[3]):
            assert np.array_equal(host(xd), xa)
    sk.close()
    for o in ops:
        o.close()
    g.close()


def test_zero_rhs_and_refusals(mp):
    shape = (8, 8, 64)
    mesh = W.stretched_mesh(*shape)
    blocks = make_blocks(shape, STAGGERED, seed=13)
    zero = [b[:5] + (np.zeros_like(b[5]), b[6]) for b in blocks]
    st, it, rel, xg, _ = gpu_stack(mp, mesh, zero, 1e-10, 100)
    assert st == mp.MAS_OK and it == 0 and all(not x.any() for x in xg)
    g = mp.Grid(mesh)
    pl, nc, bc, k, c, f, x0 = blocks[2]
    op = mp.Operator(g, nc, dev(k), dev(c), *bc, placement=pl)
    op2 = mp.Operator(g, nc, dev(k), dev(c), *bc, placement=pl)
    with pytest.raises(mp.MasError):
        mp.Stack([op, op])                      # the same operator twice
    with pytest.raises(mp.MasError):
        mp.Stack([])
    sk = mp.Stack([op, op2])
    # host arrays: staged through the ops' device buffers, same result as device arrays
    xh = [x0.copy(), x0.copy()]
    st_h, it_h, rel_h, _ = sk.solve([f, f], xh, 1e-10, 500)
    xd = [dev(x0), dev(x0)]
    st_d, it_d, rel_d, _ = sk.solve([dev(f), dev(f)], xd, 1e-10, 500)
    assert (st_h, it_h, rel_h) == (st_d, it_d, rel_d) and st_h == mp.MAS_OK
    assert np.array_equal(xh[0], host(xd[0])) and np.array_equal(xh[1], host(xd[1]))
    sk.close()
    op2.close()
    c1 = make_blocks(shape, [(0, 1, (0, 1))], seed=1)[0]
    opc = mp.Operator(g, 1, dev(c1[3]), dev(c1[4]), 0, 1)
    opc.set_single_reduction(True)
    with pytest.raises(mp.MasError):
        mp.Stack([op, opc])                     # the single-reduction loop
    opc.close()
    opa = mp.Operator(g, 1, dev(c1[3]), dev(c1[4]), 0, 1)
    opa.set_aniso(dev(np.ones(shape)), dev(np.ones((3,) + shape) / math.sqrt(3.0)))
    with pytest.raises(mp.MasError):
        mp.Stack([op, opa])                     # the field-aligned term
    opa.close()
    op.close()
    g.close()
