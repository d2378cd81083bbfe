"""The multi-rank (r-slab) path of the library on ONE B200: P ranks run as P
host threads, each with its own CUDA stream, connected by the library's
"virtual ranks" transport (comm.cpp) instead of NCCL.  Everything else is the
production multi-rank code: the slab partition, ghost-plane kernels,
seam/allreduce placement in the host-driven PCG loop and the stop handshake.

Parity: P slabs vs the oracle on the same global problem:
matvec <= 1e-13, PCG iterations +-1 and x <= 1e-10.
"""
import math
import threading

import numpy as np
import pytest

from paper_conf_ipps_caplansl23_b200 import workloads as W

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")

_key = [1000]


@pytest.fixture(scope="module")
def mp():
    if not torch.cuda.is_available():
        pytest.skip("needs a GPU")
    from paper_conf_ipps_caplansl23_b200 import build
    build.build()
    from paper_conf_ipps_caplansl23_b200 import maspcg
    return maspcg


def assemble(out, key):
    """Global [comp][r][theta][phi] field from the ranks' local blocks."""
    nc = out[0][key].shape[0]
    nr = max(r["i0"] + r["nl"] for r in out)
    nt = max(r["j0"] + r["ntl"] for r in out)
    g = np.full((nc, nr, nt, out[0][key].shape[3]), np.nan)
    for r in out:
        g[:, r["i0"]:r["i0"] + r["nl"], r["j0"]:r["j0"] + r["ntl"]] = r[key]
    assert not np.isnan(g).any()
    return g


def run_ranks(mp, prob, P, x_apply, want_solve=True, maxit=None, tol=None, p2p=False,
              solves=1, ptheta=1):
    _key[0] += 1
    vid = mp.virtual_ranks_id(_key[0])
    res, errs = {}, []

    def rank_main(r):
        try:
            torch.cuda.set_device(0)
            s = torch.cuda.Stream()
            with torch.cuda.stream(s):
                g = mp.Grid(prob.mesh, dist=(P, r, vid), ptheta=ptheta)
                i0, nl, j0, ntl = g.i0, g.nl, g.j0, g.ntl
                sl = (slice(i0, i0 + nl), slice(j0, j0 + ntl))     # [r, theta] of a field
                slc = (slice(None),) + sl                           # [comp, r, theta]
                d = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
                op = mp.Operator(g, prob.ncomp, d(prob.kappa[sl]), d(prob.c[sl]), prob.bc_inner,
                                 prob.bc_outer)
                if p2p:
                    op.enable_p2p()
                    assert op.transport == "p2p"
                y = torch.empty((prob.ncomp, nl, ntl, prob.shape[2]), dtype=torch.float64,
                                device="cuda")
                op.apply(d(x_apply[slc]), y)
                out = {"i0": i0, "nl": nl, "j0": j0, "ntl": ntl, "y": None, "dot": None}
                torch.cuda.current_stream().synchronize()
                out["y"] = y.cpu().numpy()
                out["dot"] = op.dot(d(x_apply[slc]), d(x_apply[slc]))
                if want_solve:
                    f = d(prob.f[slc])
                    ubi = d(prob.ub_inner[:, j0:j0 + ntl]) if prob.ub_inner is not None else None
                    op.dirichlet_rhs(ubi, None, f)
                    for _ in range(solves):  # repeated solves: mailbox epochs
                        x = d(prob.x0[slc])
                        st, it, rel, hist = op.solve(f, x, prob.tol if tol is None else tol,
                                                     prob.maxit if maxit is None else maxit, True)
                        torch.cuda.current_stream().synchronize()
                    out.update(st=st, it=it, rel=rel, x=x.cpu().numpy(), launches=op.launch_count,
                               hist=np.asarray(hist))
                op.close()
                g.close()
                res[r] = out
        except Exception as e:  # noqa: BLE001
            errs.append((r, repr(e)))

    th = [threading.Thread(target=rank_main, args=(r,)) for r in range(P)]
    for t in th:
        t.start()
    for t in th:
        t.join(timeout=600)
    assert not errs, errs
    assert len(res) == P
    return [res[r] for r in range(P)]


@pytest.mark.parametrize("P", [2, 3, 4])
def test_virtual_ranks_apply_dot_and_pcg(mp, oracle_mod, P):
    prob = W.viscosity_problem(13, 16, 64, warm=False)
    x = W.random_field((3,) + prob.shape, 42)
    out = run_ranks(mp, prob, P, x)
    o = oracle_mod.Oracle.for_problem(prob)
    V = o.volumes()[None]
    # matvec, assembled from the slabs
    y = assemble(out, "y")
    yo = o.apply(prob.kappa, prob.c, x)
    assert math.sqrt((V * (y - yo) ** 2).sum() / (V * yo ** 2).sum()) <= 1e-13
    # global dot through the allreduce
    for r in out:
        assert abs(r["dot"] - o.dot(x, x)) <= 1e-13 * o.dot(x, x)
    # PCG
    rc, xo, ito, _, _ = oracle_mod.solve_problem(prob)
    its = {r["it"] for r in out}
    assert len(its) == 1, its  # every rank stopped at the same iteration
    it = its.pop()
    assert all(r["st"] == mp.MAS_OK for r in out)
    assert abs(it - ito) <= 1
    xg = assemble(out, "x")
    assert math.sqrt((V * (xg - xo) ** 2).sum() / (V * xo ** 2).sum()) <= 1e-10  # unconditional (north_star: x <= 1e-10)


@pytest.mark.parametrize("P", [2, 3])
def test_virtual_ranks_seam_overlap_split_kernel(mp, oracle_mod, P):
    """Slabs of >= 12 planes use >= 3 chunks: kernel A runs the interior
    chunks while the seams are in flight, then the two edge chunks."""
    prob = W.viscosity_problem(15 * P, 16, 64, warm=False)
    x = W.random_field((3,) + prob.shape, 44)
    out = run_ranks(mp, prob, P, x)
    rc, xo, ito, _, _ = oracle_mod.solve_problem(prob)
    its = {r["it"] for r in out}
    assert len(its) == 1 and abs(its.pop() - ito) <= 1
    V = oracle_mod.Oracle.for_problem(prob).volumes()[None]
    xg = assemble(out, "x")
    assert math.sqrt((V * (xg - xo) ** 2).sum() / (V * xo ** 2).sum()) <= 1e-10
    # the split kernel A shows up as one extra launch per iteration
    assert all(r["launches"] >= 3 * r["it"] for r in out)


def test_virtual_ranks_conduction_dirichlet_and_fixed_iterations(mp, oracle_mod):
    prob = W.conduction_problem(10, 24, 32)
    x = W.random_field((1,) + prob.shape, 43)
    out = run_ranks(mp, prob, 3, x, tol=0.0, maxit=25)
    rc, xo, ito, _, _ = oracle_mod.solve_problem(prob, tol=0.0, maxit=25)
    assert all(r["st"] == mp.MAS_NOT_CONVERGED and r["it"] == 25 for r in out)
    xg = assemble(out, "x")
    V = oracle_mod.Oracle.for_problem(prob).volumes()[None]
    assert math.sqrt((V * (xg - xo) ** 2).sum() / (V * xo ** 2).sum()) <= 1e-10


# ---------------------------------------------------------------------------
# P2P transport (mas_op_enable_p2p): mailbox allreduce fused into the reducing
# kernels' last blocks and in-place reads of the neighbours' edge planes.  On
# one GPU the virtual ranks' buffers are plain device pointers of one process;
# the kernels run exactly the code of the multi-GPU path.
# ---------------------------------------------------------------------------
@pytest.mark.parametrize("P", [2, 3, 4])
def test_virtual_ranks_p2p_transport_matches_nccl_path_bitwise(mp, oracle_mod, P):
    """Both transports sum the ranks' partials in rank order, so the P2P loop
    must reproduce the NCCL-placement loop bit for bit (and the oracle).  Slabs
    of 8 planes: the NCCL loop does not split kernel A (which would change the
    block-partial summation order)."""
    prob = W.viscosity_problem(8 * P, 16, 64, warm=False)
    x = W.random_field((3,) + prob.shape, 45)
    ref = run_ranks(mp, prob, P, x)
    out = run_ranks(mp, prob, P, x, p2p=True, solves=2)
    assert [r["it"] for r in out] == [r["it"] for r in ref]
    assert all(r["st"] == mp.MAS_OK for r in out)
    for a, b in zip(out, ref):
        assert np.array_equal(a["x"], b["x"])
        assert np.array_equal(a["hist"], b["hist"])
    rc, xo, ito, _, _ = oracle_mod.solve_problem(prob)
    assert abs(out[0]["it"] - ito) <= 1
    V = oracle_mod.Oracle.for_problem(prob).volumes()[None]
    xg = assemble(out, "x")
    assert math.sqrt((V * (xg - xo) ** 2).sum() / (V * xo ** 2).sum()) <= 1e-10
    # no seam split: one kernel A and one kernel B per iteration
    assert all(r["launches"] <= 2 * r["it"] + 6 for r in out)


@pytest.mark.parametrize("P", [2, 4])
def test_virtual_ranks_p2p_long_slabs(mp, oracle_mod, P):
    prob = W.viscosity_problem(17 * P + 1, 16, 64, warm=False)
    x = W.random_field((3,) + prob.shape, 46)
    out = run_ranks(mp, prob, P, x, p2p=True)
    rc, xo, ito, _, _ = oracle_mod.solve_problem(prob)
    its = {r["it"] for r in out}
    assert len(its) == 1 and abs(its.pop() - ito) <= 1
    V = oracle_mod.Oracle.for_problem(prob).volumes()[None]
    xg = assemble(out, "x")
    assert math.sqrt((V * (xg - xo) ** 2).sum() / (V * xo ** 2).sum()) <= 1e-10


def test_virtual_ranks_p2p_dirichlet_fixed_iterations(mp, oracle_mod):
    prob = W.conduction_problem(10, 24, 32)
    x = W.random_field((1,) + prob.shape, 43)
    out = run_ranks(mp, prob, 3, x, tol=0.0, maxit=25, p2p=True)
    rc, xo, ito, _, _ = oracle_mod.solve_problem(prob, tol=0.0, maxit=25)
    assert all(r["st"] == mp.MAS_NOT_CONVERGED and r["it"] == 25 for r in out)
    xg = assemble(out, "x")
    V = oracle_mod.Oracle.for_problem(prob).volumes()[None]
    assert math.sqrt((V * (xg - xo) ** 2).sum() / (V * xo ** 2).sum()) <= 1e-10


# ---------------------------------------------------------------------------
# (r, theta) decomposition (NEXT-3): P = pr x ptheta ranks, theta fastest.
# Theta-ghost rows: packed and exchanged (setup, apply, init, NCCL loop) or
# read in place from the theta neighbours' arrays (P2P loop).
# ---------------------------------------------------------------------------
@pytest.mark.parametrize("P,ptheta,shape", [(2, 2, (9, 16, 64)), (4, 2, (12, 20, 64)),
                                            (3, 3, (7, 13, 66)), (6, 3, (10, 25, 32))])
def test_virtual_ranks_theta_split_matches_oracle(mp, oracle_mod, P, ptheta, shape):
    prob = W.viscosity_problem(*shape, warm=False)
    x = W.random_field((3,) + prob.shape, 47)
    o = oracle_mod.Oracle.for_problem(prob)
    V = o.volumes()[None]
    rc, xo, ito, _, _ = oracle_mod.solve_problem(prob)
    res = {}
    for p2p in (False, True):
        out = run_ranks(mp, prob, P, x, p2p=p2p, ptheta=ptheta)
        y = assemble(out, "y")
        yo = o.apply(prob.kappa, prob.c, x)
        assert math.sqrt((V * (y - yo) ** 2).sum() / (V * yo ** 2).sum()) <= 1e-13
        for r in out:
            assert abs(r["dot"] - o.dot(x, x)) <= 1e-13 * o.dot(x, x)
        its = {r["it"] for r in out}
        assert len(its) == 1, its
        it = its.pop()
        assert all(r["st"] == mp.MAS_OK for r in out) and abs(it - ito) <= 1
        xg = assemble(out, "x")
        assert math.sqrt((V * (xg - xo) ** 2).sum() / (V * xo ** 2).sum()) <= 1e-10  # unconditional (north_star: x <= 1e-10)
        res[p2p] = (it, xg)
    # both loops sum the same block partials in rank order
    assert res[False][0] == res[True][0]
    np.testing.assert_array_equal(res[False][1], res[True][1])


def test_virtual_ranks_theta_split_conduction_dirichlet_fixed_iterations(mp, oracle_mod):
    prob = W.conduction_problem(8, 24, 32)
    x = W.random_field((1,) + prob.shape, 48)
    rc, xo, ito, _, _ = oracle_mod.solve_problem(prob, tol=0.0, maxit=20)
    V = oracle_mod.Oracle.for_problem(prob).volumes()[None]
    for p2p in (False, True):
        out = run_ranks(mp, prob, 4, x, tol=0.0, maxit=20, p2p=p2p, ptheta=4)
        assert all(r["st"] == mp.MAS_NOT_CONVERGED and r["it"] == 20 for r in out)
        xg = assemble(out, "x")
        assert math.sqrt((V * (xg - xo) ** 2).sum() / (V * xo ** 2).sum()) <= 1e-10


def test_test_transports_need_opt_in(mp):
    """A production process (no MAS_TEST_TRANSPORTS=1) cannot select the
    virtual-rank test transport by its id: mas_grid_create returns
    MAS_ERR_ARG (comm.cpp)."""
    import os
    import subprocess
    import sys
    code = (
        "import sys; sys.path.insert(0, %r)\n"
        "import torch; torch.cuda.set_device(0)\n"
        "from paper_conf_ipps_caplansl23_b200 import maspcg as M, workloads as W\n"
        "m = W.stretched_mesh(4, 8, 8)\n"
        "try:\n"
        "    M.Grid(m, dist=(2, 0, M.virtual_ranks_id(4242)))\n"
        "    print('created')\n"
        "except M.MasError as e:\n"
        "    print('status', e.status)\n" % os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    env = {k: v for k, v in os.environ.items() if k != "MAS_TEST_TRANSPORTS"}
    out = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True, timeout=300)
    assert ("status %d" % mp.MAS_ERR_ARG) in out.stdout, (out.stdout, out.stderr[-2000:])
