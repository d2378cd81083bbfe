"""Parity at BASELINE.json's full sizes, in bench.py's launch configuration
(single GPU, the CUDA-graph PCG loop, chunked stencil work items):

* C3 (3-component viscosity, 256x256x512) and C2 (conduction, 128x128x256)
  matvec: GPU mas_op_apply vs the oracle evaluated cell by cell
  (mas_ref_op_apply_cells) on ~20k sampled cells that include every boundary
  class (poles, r-boundaries, phi wrap, tile and chunk edges): <= 1e-13
  relative to the local scale;
* the full solves: the oracle runs the same PCG at full size (seconds on the
  box's host cores): iterations within max(1, the oracle's own 1-ulp
  sensitivity) (R20), x <= 1e-10 relative L2_V; and the true
  residual of the GPU solution, computed by the oracle, is at the level the
  recursive residual reports.
"""
import math

import numpy as np
import pytest

from paper_conf_ipps_caplansl23_b200 import workloads as W

pytestmark = [pytest.mark.gpu, pytest.mark.slow]
torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def mp():
    if not torch.cuda.is_available():
        pytest.skip("needs a GPU")
    from paper_conf_ipps_caplansl23_b200 import build
    build.build()
    from paper_conf_ipps_caplansl23_b200 import maspcg
    return maspcg


def sample_cells(shape, ncomp, n=20000, seed=5):
    nr, nt, np_ = shape
    rng = np.random.default_rng(seed)
    i = rng.integers(0, nr, n)
    j = rng.integers(0, nt, n)
    k = rng.integers(0, np_, n)
    # force boundary classes: r faces, poles, phi wrap, tile/chunk edges
    special = []
    for ii in (0, 1, nr - 2, nr - 1, 31, 32, 63, 64):
        for jj in (0, 1, nt - 2, nt - 1, 7, 8):
            for kk in (0, 1, np_ - 1, 63, 64):
                if ii < nr and jj < nt and kk < np_:
                    special.append((ii, jj, kk))
    sp = np.array(special).T
    i, j, k = (np.concatenate([a, b]) for a, b in zip((i, j, k), sp))
    m = rng.integers(0, ncomp, len(i))
    P = (i * nt + j) * np_ + k
    return np.unique(m * (nr * nt * np_) + P)


@pytest.mark.parametrize("cfg", ["C2", "C3"])
def test_fullsize_matvec_sampled(mp, oracle_mod, cfg):
    kind, nr, nt, np_ = {"C2": ("conduction", 128, 128, 256), "C3": ("viscosity", 256, 256, 512)}[cfg]
    prob = W.make(kind, nr=nr, nt=nt, np_=np_)
    x = W.random_field((prob.ncomp,) + prob.shape, 42)
    g = mp.Grid(prob.mesh)
    d = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    op = mp.Operator(g, prob.ncomp, d(prob.kappa), d(prob.c), prob.bc_inner, prob.bc_outer)
    y = torch.empty_like(d(x))
    op.apply(d(x), y)
    yg = y.cpu().numpy().ravel()
    idx = sample_cells(prob.shape, prob.ncomp)
    o = oracle_mod.Oracle.for_problem(prob)
    yo = o.apply_cells(prob.kappa, prob.c, x, idx)
    # local scale: |c u| + (1/V) sum_f G_f |u_P| + |u_N| ~ D_P * max|x|
    D = o.diag(prob.kappa, prob.c).ravel()
    scale = D[idx % D.size] * 2.0
    err = np.abs(yg[idx] - yo) / scale
    assert err.max() <= 1e-13, err.max()


@pytest.mark.parametrize("cfg", ["C2", "C3"])
def test_fullsize_pcg_vs_oracle(mp, oracle_mod, cfg):
    kind, nr, nt, np_ = {"C2": ("conduction", 128, 128, 256), "C3": ("viscosity", 256, 256, 512)}[cfg]
    prob = W.make(kind, nr=nr, nt=nt, np_=np_)
    d = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    g = mp.Grid(prob.mesh)
    op = mp.Operator(g, prob.ncomp, d(prob.kappa), d(prob.c), prob.bc_inner, prob.bc_outer)
    f = d(prob.f)
    if prob.ub_inner is not None:
        op.dirichlet_rhs(d(prob.ub_inner), None, f)
    x = d(prob.x0)
    st, it, rel, hist = op.solve(f, x, prob.tol, prob.maxit, True)
    assert st == mp.MAS_OK and rel <= prob.tol
    xg = x.cpu().numpy()
    fh = f.cpu().numpy()
    rc, xo, ito, relo, _ = oracle_mod.solve_problem(prob)
    assert rc == oracle_mod.OK
    o = oracle_mod.Oracle.for_problem(prob)
    # The oracle's own sensitivity: near tol the residual curve of these
    # stiff problems is flat (ratio ~0.9-1.0 per iteration), and a 1e-16
    # relative perturbation of f moves the oracle's own count (C2: 173 ->
    # 171).  Band = max(1, that envelope) (R20); x must agree to
    # 1e-10 regardless of the count.
    fo = o.dirichlet_rhs(prob.kappa, prob.f, prob.ub_inner, prob.ub_outer)
    env = 0
    for s in range(2):
        fp = fo * (1.0 + 1e-16 * np.random.default_rng(s).standard_normal(fo.shape))
        _, _, itp, _, _ = o.pcg(prob.kappa, prob.c, fp, prob.x0, prob.tol, prob.maxit)
        env = max(env, abs(itp - ito))
    assert abs(it - ito) <= max(1, env), (it, ito, env)
    V = o.volumes()[None]
    assert math.sqrt((V * (xg - xo) ** 2).sum() / (V * xo ** 2).sum()) <= 1e-10
    # the oracle's rhs equals the library's rhs (Dirichlet helper parity)
    assert math.sqrt((V * (fh - fo) ** 2).sum() / (V * fo ** 2).sum()) <= 1e-14
    # true residual of the GPU solution, by the oracle
    r = fo - o.apply(prob.kappa, prob.c, xg)
    true_rel = math.sqrt((V * r * r).sum() / (V * fo * fo).sum())
    assert true_rel <= 10 * prob.tol, true_rel


# ---------------------------------------------------------------------------
# C2a: field-aligned conduction (NEXT-4) at its bench size, bench launch
# configuration (k_aniso r-chunks sized for one resident wave)
# ---------------------------------------------------------------------------
def test_fullsize_c2a_apply_and_solve(mp, oracle_mod):
    prob = W.aniso_conduction_problem(128, 128, 256)
    o = oracle_mod.Oracle.for_problem(prob)
    d = lambda a: torch.from_numpy(np.array(a)).cuda()
    g = mp.Grid(prob.mesh)
    op = mp.Operator(g, 1, d(prob.kappa), d(prob.c), prob.bc_inner, prob.bc_outer)
    op.set_aniso(d(prob.kpar), d(prob.bhat))
    x = W.random_field((1,) + prob.shape, 42)
    y = torch.empty((1,) + prob.shape, dtype=torch.float64, device="cuda")
    op.apply(d(x), y)
    yo = o.apply(prob.kappa, prob.c, x) + o.aniso_apply(prob.kpar, prob.bhat, x)
    V = o.volumes()[None]
    yg = y.cpu().numpy()
    assert math.sqrt((V * (yg - yo) ** 2).sum() / (V * yo ** 2).sum()) <= 1e-13
    # the full solve, warm start as in bench.py
    f = d(prob.f)
    op.dirichlet_rhs(d(prob.ub_inner), None, f)
    xs = d(prob.x0)
    st, it, rel, _ = op.solve(f, xs, prob.tol, prob.maxit)
    rc, xo, ito, relo, _ = oracle_mod.solve_problem(prob)
    assert st == mp.MAS_OK and rc == oracle_mod.OK
    assert abs(it - ito) <= 1, (it, ito)
    xg = xs.cpu().numpy()
    assert math.sqrt((V * (xg - xo) ** 2).sum() / (V * xo ** 2).sum()) <= 1e-10  # unconditional (north_star: x <= 1e-10)


# ---------------------------------------------------------------------------
# the round-2 bench configurations at full size: the single-reduction loop
# (bench --solver cg1) on C2 and C3, and C2t (theta nodes with pole rows)
# ---------------------------------------------------------------------------
@pytest.mark.parametrize("cfg", ["C2", "C3"])
def test_fullsize_single_reduction_vs_oracle(mp, oracle_mod, cfg):
    kind, nr, nt, np_ = {"C2": ("conduction", 128, 128, 256), "C3": ("viscosity", 256, 256, 512)}[cfg]
    prob = W.make(kind, nr=nr, nt=nt, np_=np_)
    d = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    g = mp.Grid(prob.mesh)
    op = mp.Operator(g, prob.ncomp, d(prob.kappa), d(prob.c), prob.bc_inner, prob.bc_outer)
    op.set_single_reduction(True)
    f = d(prob.f)
    if prob.ub_inner is not None:
        op.dirichlet_rhs(d(prob.ub_inner), None, f)
    x = d(prob.x0)
    st, it, rel, _ = op.solve(f, x, prob.tol, prob.maxit)
    assert st == mp.MAS_OK and rel <= prob.tol
    xg = x.cpu().numpy()
    rc, xo, ito, _, _ = oracle_mod.solve_problem(prob, cg1=True)
    assert rc == oracle_mod.OK
    # NEXT-1's band: +-2 iterations, x <= 1e-9
    assert abs(it - ito) <= 2, (it, ito)
    V = oracle_mod.Oracle.for_problem(prob).volumes()[None]
    assert math.sqrt((V * (xg - xo) ** 2).sum() / (V * xo ** 2).sum()) <= 1e-9


def test_fullsize_theta_nodes_vs_oracle(mp, oracle_mod):
    prob = W.tnode_conduction_problem(128, 128, 256)
    d = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    g = mp.Grid(prob.mesh)
    op = mp.Operator(g, 1, d(prob.kappa), d(prob.c), prob.bc_inner, prob.bc_outer,
                     placement=mp.MAS_PLACE_THETA_NODE)
    f = d(prob.f)
    op.dirichlet_rhs(d(prob.ub_inner), None, f)
    x = d(prob.x0)
    st, it, rel, _ = op.solve(f, x, prob.tol, prob.maxit)
    assert st == mp.MAS_OK
    o = oracle_mod.Oracle.for_problem(prob)
    fo = o.tn_dirichlet_rhs(prob.kappa, prob.f, prob.ub_inner, None)
    rc, xo, ito, _, _ = o.tn_pcg(prob.kappa, prob.c, fo, prob.x0, prob.tol, prob.maxit)
    env = 0  # the oracle's own 1-ulp sensitivity (R20)
    for sd in range(2):
        fp = fo * (1.0 + 1e-16 * np.random.default_rng(sd).standard_normal(fo.shape))
        _, _, itp, _, _ = o.tn_pcg(prob.kappa, prob.c, fp, prob.x0, prob.tol, prob.maxit)
        env = max(env, abs(itp - ito))
    assert abs(it - ito) <= max(1, env), (it, ito, env)
    V = o.tn_volumes()[None]
    xg = x.cpu().numpy()
    assert math.sqrt((V * (xg - xo) ** 2).sum() / (V * xo ** 2).sum()) <= 1e-10
    for row in (0, -1):  # one value per pole and radius
        assert np.array_equal(xg[0, :, row, :], np.broadcast_to(xg[0, :, row, :1], xg[0, :, row, :].shape))


def test_fullsize_staggered_stack_vs_oracle(mp, oracle_mod):
    """NEXT-2 R34 at C2's grid: C3's viscous fields on the staggered mesh
    (v_r r nodes, v_theta theta nodes, v_phi phi nodes), one PCG on the
    stacked vector: iterations within max(1, the oracle's envelope), x <= 1e-10
    in the stacked V-norm."""
    mesh, dt, blocks = W.staggered_viscosity_blocks(128, 128, 256)
    d = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    g = mp.Grid(mesh)
    ops = [mp.Operator(g, 1, d(k), d(c), W.DIRICHLET, W.NEUMANN, placement=pl) for pl, k, c, f, x0 in blocks]
    sk = mp.Stack(ops)
    xs = [d(b[4]) for b in blocks]
    tol = 1e-12
    st, it, rel, _ = sk.solve([d(b[3]) for b in blocks], xs, tol, 20000)
    assert st == mp.MAS_OK and rel <= tol
    xg = [x.cpu().numpy() for x in xs]
    o = oracle_mod.Oracle(mesh, W.DIRICHLET, W.NEUMANN)

    def run(scale):
        return oracle_mod.stacked_pcg([(o, pl, k, c, f * scale, x0) for pl, k, c, f, x0 in blocks], tol, 20000)

    rc, xo, ito, _, _ = run(1.0)
    assert rc == oracle_mod.OK
    _, _, itp, _, _ = run(1.0 + 2.2e-16)
    env = abs(itp - ito)
    assert abs(it - ito) <= max(1, env), (it, ito, env)
    V = [{1: o.tn_volumes, 2: o.rn_volumes, 3: o.pn_volumes}[b[0]]()[None] for b in blocks]
    num = sum((v * (a - b) ** 2).sum() for v, a, b in zip(V, xg, xo))
    den = sum((v * b ** 2).sum() for v, b in zip(V, xo))
    assert math.sqrt(num / den) <= 1e-10
    sk.close()
    for op in ops:
        op.close()
    g.close()
