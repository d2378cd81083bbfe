"""The breakdown exit of the PCG loop (sigma_k <= 0 in kernel B(k)) on the GPU:
status MAS_ERR_BREAKDOWN, iters = k, and x = the iterate before the breaking
step, x_{k-1}.  With the scalar operator's two-iteration x update (DESIGN.md
§5.2) an even k leaves x at x_{k-2} after kernel A(k), and kernel B completes
it.  A symmetric positive definite operator does not break down, so the
breakdown is forced with a test hook (MAS_TEST_BREAKDOWN_AT=k, honoured only
with MAS_TEST_TRANSPORTS=1); the reference is the same solve stopped after
k-1 iterations (tol 0, maxit k-1), itself pinned to the oracle by the
fixed-iteration parity tests -- compared bitwise, in the graph loop and in
the host loop."""
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


@pytest.mark.parametrize("kind", ["conduction", "viscosity"])
@pytest.mark.parametrize("graph", [True, False])
def test_forced_breakdown_returns_the_previous_iterate(mp, monkeypatch, kind, graph):
    prob = W.conduction_problem(10, 16, 64) if kind == "conduction" else W.viscosity_problem(12, 16, 64)
    if not graph:
        monkeypatch.setenv("MAS_NO_GRAPH", "1")  # read at operator setup
    g = mp.Grid(prob.mesh)
    op = mp.Operator(g, prob.ncomp, dev(prob.kappa), dev(prob.c), prob.bc_inner, prob.bc_outer)
    f = dev(prob.f)
    if prob.ub_inner is not None:
        op.dirichlet_rhs(dev(prob.ub_inner), None, f)
    for k in (1, 2, 3, 6, 7):
        monkeypatch.setenv("MAS_TEST_BREAKDOWN_AT", str(k))
        x = dev(prob.x0)
        st, it, rel, hist = op.solve(f, x, 1e-14, 1000, True)
        monkeypatch.delenv("MAS_TEST_BREAKDOWN_AT")
        assert st == mp.MAS_ERR_BREAKDOWN and it == k, (k, st, it)
        xr = dev(prob.x0)
        st_r, it_r, rel_r, hist_r = op.solve(f, xr, 0.0, k - 1, True)
        assert it_r == k - 1 and st_r in (mp.MAS_NOT_CONVERGED, mp.MAS_OK)
        assert np.array_equal(x.cpu().numpy(), xr.cpu().numpy()), (kind, k)
        assert rel == rel_r and np.array_equal(np.asarray(hist), np.asarray(hist_r)), (kind, k)
    op.close()
    g.close()
