"""The field-aligned conduction term (NEXT-4) on the r-slab multi-rank path, on
ONE B200: P ranks as host threads connected by the library's virtual-ranks
transport (comm.cpp), everything else the production multi-rank code (corner
plane seam at mas_op_set_aniso, p_k seams after every kernel A, rank-local
sigma partials + allreduce, init residual with x seams).

Parity against the oracle on the same global problem: apply <= 1e-13, PCG
iterations +-1 and x <= 1e-10; every rank stops at the same iteration.
"""
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


def run_ranks(mp, prob, P, x_apply, tol, maxit, p2p=False):
    _key[0] += 1
    vid = mp.virtual_ranks_id(_key[0])
    res, errs = {}, []

    def rank_main(r):
        try:
            torch.cuda.set_device(0)
            s = torch.cuda.Stream()
            with torch.cuda.stream(s):
                g = mp.Grid(prob.mesh, dist=(P, r, vid))
                i0, nl = g.i0, g.nl
                sl = slice(i0, i0 + nl)
                d = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
                op = mp.Operator(g, 1, d(prob.kappa[sl]), d(prob.c[sl]), prob.bc_inner,
                                 prob.bc_outer)
                if p2p:  # the mailbox loop: p_k read in place from the neighbours
                    op.enable_p2p()
                op.set_aniso(d(prob.kpar[sl]), d(prob.bhat[:, sl]))
                y = torch.empty((1, nl) + prob.shape[1:], dtype=torch.float64, device="cuda")
                op.apply(d(x_apply[:, sl]), y)
                D = torch.empty((nl,) + prob.shape[1:], dtype=torch.float64, device="cuda")
                op.diag(D)
                f = d(prob.f[:, sl])
                op.dirichlet_rhs(d(prob.ub_inner) if prob.ub_inner is not None else None, None, f)
                x = d(prob.x0[:, sl])
                st, it, rel, hist = op.solve(f, x, tol, maxit, True)
                torch.cuda.current_stream().synchronize()
                res[r] = {"i0": i0, "nl": nl, "y": y.cpu().numpy(), "D": D.cpu().numpy(),
                          "st": st, "it": it, "x": x.cpu().numpy()}
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
    return [res[r] for r in range(P)]


def assemble(out, key, axis):
    return np.concatenate([r[key] for r in out], axis=axis)


@pytest.mark.parametrize("p2p", [False, True])
@pytest.mark.parametrize("P,shape", [(2, (16, 16, 64)), (3, (20, 24, 70)), (4, (33, 16, 128))])
def test_aniso_virtual_ranks_match_oracle(mp, oracle_mod, P, shape, p2p):
    prob = W.aniso_conduction_problem(*shape)
    x = W.random_field((1,) + prob.shape, 42)
    out = run_ranks(mp, prob, P, x, prob.tol, prob.maxit, p2p)
    o = oracle_mod.Oracle.for_problem(prob)
    V = o.volumes()[None]
    y = assemble(out, "y", 1)
    yo = o.apply(prob.kappa, prob.c, x) + o.aniso_apply(prob.kpar, prob.bhat, x)
    assert math.sqrt((V * (y - yo) ** 2).sum() / (V * yo ** 2).sum()) <= 1e-13
    D = assemble(out, "D", 0)
    np.testing.assert_allclose(D, o.diag(prob.kappa, prob.c) + o.aniso_diag(prob.kpar, prob.bhat),
                               rtol=1e-13, atol=0)
    rc, xo, ito, _, _ = oracle_mod.solve_problem(prob)
    its = {r["it"] for r in out}
    assert len(its) == 1, its
    it = its.pop()
    assert all(r["st"] == mp.MAS_OK for r in out)
    assert abs(it - ito) <= 1, (it, ito)
    xg = assemble(out, "x", 1)
    assert math.sqrt((V * (xg - xo) ** 2).sum() / (V * xo ** 2).sum()) <= 1e-10  # unconditional (north_star: x <= 1e-10)


def test_aniso_virtual_ranks_fixed_iterations(mp, oracle_mod):
    prob = W.aniso_conduction_problem(18, 16, 64)
    out = run_ranks(mp, prob, 3, W.random_field((1,) + prob.shape, 1), 0.0, 12)
    rc, xo, ito, _, _ = oracle_mod.solve_problem(prob, tol=0.0, maxit=12)
    assert {r["it"] for r in out} == {12} and ito == 12
    V = oracle_mod.Oracle.for_problem(prob).volumes()[None]
    xg = assemble(out, "x", 1)
    assert math.sqrt((V * (xg - xo) ** 2).sum() / (V * xo ** 2).sum()) <= 1e-10
