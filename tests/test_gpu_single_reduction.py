"""NEXT-1 single-reduction PCG on the GPU (mas_op_set_single_reduction),
through the C ABI, against the oracle's Chronopoulos-Gear recurrence
(mas_ref_pcg_solve_cg1, pinned in tests/test_oracle_cg1_pins.py).

Band ("its own parity band"): iterations within +-2 of
the oracle's CG1 and of the oracle's standard PCG, x within 1e-9 relative
L2_V of both (in practice the same recurrence agrees like the two-kernel
loop: see the asserts on the history); fixed iteration counts: x within
1e-10 of the oracle's CG1."""
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


def rel_l2_V(V, a, b):
    V = V[None]
    return math.sqrt((V * (a - b) ** 2).sum() / max((V * b ** 2).sum(), 1e-300))


def make(mp, prob):
    g = mp.Grid(prob.mesh)
    op = mp.Operator(g, prob.ncomp, dev(prob.kappa), dev(prob.c), prob.bc_inner, prob.bc_outer)
    op.set_single_reduction(True)
    assert op.single_reduction
    f = dev(prob.f)
    ubi = None if prob.ub_inner is None else dev(prob.ub_inner)
    ubo = None if prob.ub_outer is None else dev(prob.ub_outer)
    if ubi is not None or ubo is not None:
        op.dirichlet_rhs(ubi, ubo, f)
    return g, op, f


def gsolve(mp, prob, tol=None, maxit=None, x0=None, prof=False):
    g, op, f = make(mp, prob)
    op.set_profiling(prof)
    x = dev(prob.x0 if x0 is None else x0)
    st, it, rel, hist = op.solve(f, x, prob.tol if tol is None else tol,
                                 prob.maxit if maxit is None else maxit, True)
    torch.cuda.synchronize()
    return st, x.cpu().numpy(), it, rel, hist, op, g


def problems():
    return [W.mms_problem(16, 24, 32), W.conduction_problem(16, 24, 64),
            W.viscosity_problem(16, 24, 64), W.conduction_problem(9, 13, 70, warm=False),
            W.viscosity_problem(33, 8, 66, warm=False), W.conduction_problem(40, 17, 130)]


@pytest.mark.parametrize("idx", range(6))
def test_single_reduction_matches_oracle_at_tol(mp, oracle_mod, idx):
    prob = problems()[idx]
    rc, xo, ito, relo, histo = oracle_mod.solve_problem(prob, cg1=True)
    rs, xs, its, _, _ = oracle_mod.solve_problem(prob)
    st, x, it, rel, hist, op, g = gsolve(mp, prob)
    assert rc == oracle_mod.OK and st == mp.MAS_OK and rel <= prob.tol
    assert abs(it - ito) <= 2 and abs(it - its) <= 2, (it, ito, its)
    V = oracle_mod.Oracle.for_problem(prob).volumes()
    assert rel_l2_V(V, x, xo) <= 1e-9
    assert rel_l2_V(V, x, xs) <= 1e-9
    n = min(10, len(hist), len(histo))
    np.testing.assert_allclose(hist[:n], histo[:n], rtol=1e-9, atol=0)


@pytest.mark.parametrize("k", [1, 2, 7, 40])
@pytest.mark.parametrize("mk", ["viscosity", "conduction"])
def test_single_reduction_fixed_iterations(mp, oracle_mod, k, mk):
    prob = W.viscosity_problem(12, 16, 32) if mk == "viscosity" else W.conduction_problem(12, 16, 32)
    rc, xo, ito, _, _ = oracle_mod.solve_problem(prob, tol=0.0, maxit=k, cg1=True)
    st, x, it, rel, hist, op, g = gsolve(mp, prob, tol=0.0, maxit=k)
    assert rc == oracle_mod.NOT_CONVERGED and st == mp.MAS_NOT_CONVERGED
    assert it == ito == k
    V = oracle_mod.Oracle.for_problem(prob).volumes()
    assert rel_l2_V(V, x - prob.x0, xo - prob.x0) <= 1e-10
    # the host-driven loop (profiling; also the virtual-rank / NCCL loops) must
    # launch the kernel that takes the maxit decision and give the same bits
    st2, x2, it2, rel2, hist2, _, _ = gsolve(mp, prob, tol=0.0, maxit=k, prof=True)
    assert (st2, it2) == (st, it)
    np.testing.assert_array_equal(x2, x)
    np.testing.assert_array_equal(np.asarray(hist2), np.asarray(hist))


@pytest.mark.parametrize("mk", ["viscosity", "mms"])
def test_single_reduction_graph_equals_host_loop(mp, mk):
    prob = W.viscosity_problem(20, 16, 64) if mk == "viscosity" else W.mms_problem(16, 24, 32)
    a = gsolve(mp, prob)
    b = gsolve(mp, prob, prof=True)
    assert a[2] == b[2] and a[0] == b[0]
    np.testing.assert_array_equal(a[1], b[1])
    np.testing.assert_array_equal(np.asarray(a[4]), np.asarray(b[4]))
    assert b[5].kernel_times()[0] > 0.0
    # repeated solves through the cached graph
    c = gsolve(mp, prob)
    np.testing.assert_array_equal(a[1], c[1])


def test_single_reduction_edge_cases(mp, oracle_mod):
    prob = W.conduction_problem(8, 16, 32)
    prob.f[:] = 0.0
    prob.ub_inner = None
    st, x, it, rel, hist, op, g = gsolve(mp, prob)
    assert st == mp.MAS_OK and it == 0 and (x == 0).all()
    prob = W.conduction_problem(8, 16, 32)
    st, x, it, rel, hist, op, g = gsolve(mp, prob, maxit=0)
    assert st == mp.MAS_NOT_CONVERGED and it == 0
    np.testing.assert_array_equal(x, prob.x0)
    rc, xo, _, _, _ = oracle_mod.solve_problem(prob, tol=1e-14)
    st, x, it, rel, hist, op, g = gsolve(mp, prob, tol=1e-8, x0=xo)
    assert st == mp.MAS_OK and it == 0
    # mass only: exactly one iteration, x = f / c
    shape = (6, 10, 20)
    c = np.random.default_rng(5).uniform(0.1, 3, size=shape)
    f = np.random.default_rng(6).standard_normal((3,) + shape)
    gg = mp.Grid(W.stretched_mesh(*shape))
    o = mp.Operator(gg, 3, dev(np.zeros(shape)), dev(c), 0, 1)
    o.set_single_reduction(True)
    xx = torch.zeros((3,) + shape, dtype=torch.float64, device="cuda")
    st, it, rel, _ = o.solve(dev(f), xx, 1e-12, 50)
    assert st == mp.MAS_OK and it == 1
    np.testing.assert_allclose(xx.cpu().numpy(), f / c[None], rtol=4e-16, atol=0)


def test_single_reduction_switch_and_refusals(mp, oracle_mod):
    prob = W.viscosity_problem(12, 16, 64)
    st, x, it, rel, hist, op, g = gsolve(mp, prob)
    op.set_single_reduction(False)
    assert not op.single_reduction
    f = dev(prob.f)
    xs = dev(prob.x0)
    st2, it2, _, _ = op.solve(f, xs, prob.tol, prob.maxit)
    rs, xo, its, _, _ = oracle_mod.solve_problem(prob)
    assert abs(it2 - its) <= 1  # the two-kernel loop again
    # field-aligned term and single reduction refuse each other
    pa = W.aniso_conduction_problem(16, 16, 32)
    ga = mp.Grid(pa.mesh)
    oa = mp.Operator(ga, 1, dev(pa.kappa), dev(pa.c), pa.bc_inner, pa.bc_outer)
    oa.set_aniso(dev(pa.kpar), dev(pa.bhat))
    with pytest.raises(mp.MasError) as e:
        oa.set_single_reduction(True)
    assert e.value.status == mp.MAS_ERR_ARG
    oa.set_aniso(None, None)
    oa.set_single_reduction(True)
    with pytest.raises(mp.MasError):
        oa.set_aniso(dev(pa.kpar), dev(pa.bhat))
    # the single-reduction loop over the P2P transport: switched on before
    # mas_op_enable_p2p (which then maps its buffers), refused after it
    gp = mp.Grid(prob.mesh)
    op2 = mp.Operator(gp, prob.ncomp, dev(prob.kappa), dev(prob.c), prob.bc_inner, prob.bc_outer)
    op2.enable_p2p()
    with pytest.raises(mp.MasError):
        op2.set_single_reduction(True)
    op3 = mp.Operator(gp, prob.ncomp, dev(prob.kappa), dev(prob.c), prob.bc_inner, prob.bc_outer)
    op3.set_single_reduction(True)
    op3.enable_p2p()
    assert op3.transport == "p2p" and op3.single_reduction


@pytest.mark.parametrize("mk", ["viscosity", "conduction"])
def test_single_reduction_one_rank_nccl(mp, oracle_mod, mk):
    """The r-slab loop (seams of r, w, s; ONE ncclAllReduce of 3 doubles per
    iteration; the decision in the next kernel) on a 1-rank NCCL communicator."""
    prob = W.viscosity_problem(24, 16, 64) if mk == "viscosity" else W.conduction_problem(40, 16, 32)
    g = mp.Grid(prob.mesh, dist=(1, 0, mp.mas_comm_unique_id()))
    op = mp.Operator(g, prob.ncomp, dev(prob.kappa), dev(prob.c), prob.bc_inner, prob.bc_outer)
    op.set_single_reduction(True)
    f = dev(prob.f)
    if prob.ub_inner is not None:
        op.dirichlet_rhs(dev(prob.ub_inner), None, f)
    x = dev(prob.x0)
    st, it, rel, hist = op.solve(f, x, prob.tol, prob.maxit, True)
    rc, xo, ito, _, histo = oracle_mod.solve_problem(prob, cg1=True)
    V = oracle_mod.Oracle.for_problem(prob).volumes()
    assert st == mp.MAS_OK and abs(it - ito) <= 2
    assert rel_l2_V(V, x.cpu().numpy(), xo) <= 1e-9
    np.testing.assert_allclose(hist[:10], histo[:10], rtol=1e-9, atol=0)


@pytest.mark.parametrize("P", [2, 3])
def test_single_reduction_virtual_ranks(mp, oracle_mod, P):
    """r-slabs on P virtual ranks: every rank stops at the same iteration;
    iterations +-2 and x <= 1e-9 against the oracle's monolithic CG1."""
    import threading
    prob = W.viscosity_problem(13 * P, 16, 64, warm=False)
    vid = mp.virtual_ranks_id(7700 + P)
    res, errs = {}, []

    def rank_main(r):
        try:
            torch.cuda.set_device(0)
            with torch.cuda.stream(torch.cuda.Stream()):
                g = mp.Grid(prob.mesh, dist=(P, r, vid))
                sl = slice(g.i0, g.i0 + g.nl)
                op = mp.Operator(g, 3, dev(prob.kappa[sl]), dev(prob.c[sl]), prob.bc_inner,
                                 prob.bc_outer)
                op.set_single_reduction(True)
                x = dev(prob.x0[:, sl])
                st, it, rel, _ = op.solve(dev(prob.f[:, sl]), x, prob.tol, prob.maxit)
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
    rc, xo, ito, _, _ = oracle_mod.solve_problem(prob, cg1=True)
    its = {res[r][3] for r in range(P)}
    assert len(its) == 1, its
    assert abs(its.pop() - ito) <= 2
    xg = np.empty_like(xo)
    for r in range(P):
        i0, nl, st, it, x = res[r]
        assert st == mp.MAS_OK
        xg[:, i0:i0 + nl] = x
    assert rel_l2_V(oracle_mod.Oracle.for_problem(prob).volumes(), xg, xo) <= 1e-9


@pytest.mark.parametrize("mk", ["viscosity", "conduction"])
def test_single_reduction_p2p_one_rank_bitwise(mp, mk):
    """The mailbox reduction against the rank itself (0 + v = v): the P2P
    single-reduction loop equals the plain one bit for bit, over repeated
    solves (epochs), in the CUDA-graph loop."""
    prob = W.viscosity_problem(12, 16, 64) if mk == "viscosity" else W.conduction_problem(10, 16, 32)
    st, x, it, rel, hist, op, g = gsolve(mp, prob)
    op2 = mp.Operator(g, prob.ncomp, dev(prob.kappa), dev(prob.c), prob.bc_inner, prob.bc_outer)
    op2.set_single_reduction(True)
    op2.enable_p2p()
    f = dev(prob.f)
    if prob.ub_inner is not None:
        op2.dirichlet_rhs(dev(prob.ub_inner), None, f)
    for _ in range(3):
        x2 = dev(prob.x0)
        st2, it2, rel2, hist2 = op2.solve(f, x2, prob.tol, prob.maxit, True)
        assert (st2, it2, rel2) == (st, it, rel)
        np.testing.assert_array_equal(x2.cpu().numpy(), x)
        np.testing.assert_array_equal(np.asarray(hist2), np.asarray(hist))


@pytest.mark.parametrize("P", [2, 3])
def test_single_reduction_p2p_virtual_ranks(mp, oracle_mod, P):
    """r-slabs on P virtual ranks with the P2P transport: the kernels sum the
    3 partials in the mailbox (rank order), the halos are read in place; the
    same bits as the NCCL loop of the virtual ranks (its allreduce also sums
    in rank order), and the oracle's CG1 band."""
    import threading
    prob = W.viscosity_problem(13 * P, 16, 64, warm=False)
    out = {}
    for p2p in (False, True):
        vid = mp.virtual_ranks_id(7800 + 10 * P + int(p2p))
        res, errs = {}, []

        def rank_main(r):
            try:
                torch.cuda.set_device(0)
                with torch.cuda.stream(torch.cuda.Stream()):
                    g = mp.Grid(prob.mesh, dist=(P, r, vid))
                    sl = slice(g.i0, g.i0 + g.nl)
                    op = mp.Operator(g, 3, dev(prob.kappa[sl]), dev(prob.c[sl]), prob.bc_inner,
                                     prob.bc_outer)
                    op.set_single_reduction(True)
                    if p2p:
                        op.enable_p2p()
                    x = dev(prob.x0[:, sl])
                    st, it, rel, _ = op.solve(dev(prob.f[:, sl]), x, prob.tol, prob.maxit)
                    torch.cuda.current_stream().synchronize()
                    res[r] = (g.i0, g.nl, st, it, x.cpu().numpy(), op.transport)
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
        assert {res[r][5] for r in range(P)} == {"p2p" if p2p else "nccl"}
        out[p2p] = res
    rc, xo, ito, _, _ = oracle_mod.solve_problem(prob, cg1=True)
    for p2p in (False, True):
        its = {out[p2p][r][3] for r in range(P)}
        assert len(its) == 1 and abs(next(iter(its)) - ito) <= 2
    xs = {}
    for p2p in (False, True):
        xg = np.empty_like(xo)
        for r in range(P):
            i0, nl, st, it, x, _ = out[p2p][r]
            assert st == mp.MAS_OK
            xg[:, i0:i0 + nl] = x
        xs[p2p] = xg
    assert out[True][0][3] == out[False][0][3]
    np.testing.assert_array_equal(xs[True], xs[False])
    assert rel_l2_V(oracle_mod.Oracle.for_problem(prob).volumes(), xs[True], xo) <= 1e-9
