"""The NCCL code path on one B200: mas_grid_create with a 1-rank mas_dist_t
and a real NCCL unique id creates a 1-rank NCCL communicator (ncclCommInitRank
+ ncclCommSplit), so the op runs the multi-GPU iteration loop: the comm
stream, the split kernel-A launch (interior chunks, then the edge chunks
behind the seam event), ncclAllReduce of sigma and (rho, ||r||^2), the init
allreduce, the NCCL-polling waits (ncclCommGetAsyncError) and mas_op_dot's
allreduce.  With one rank the seams have no neighbour, so ncclSend/ncclRecv
cannot run here; everything else of the NCCL transport does.

Parity (north_star): PCG iterations within +-1 and x within 1e-10 relative
L2_V of the oracle; the NCCL loop against the single-GPU graph loop on the
same op problem: iterations +-1, x within 1e-10 (the split kernel A sums
<p,q> in another order, so the bits may differ)."""
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
    return math.sqrt((V[None] * (a - b) ** 2).sum() / (V[None] * b ** 2).sum())


def solve(mp, prob, dist, p2p=False, aniso=False):
    g = mp.Grid(prob.mesh, dist=dist)
    op = mp.Operator(g, prob.ncomp, dev(prob.kappa), dev(prob.c), prob.bc_inner, prob.bc_outer)
    if aniso:
        op.set_aniso(dev(prob.kpar), dev(prob.bhat))
    if p2p:
        op.enable_p2p()
    f = dev(prob.f)
    if prob.ub_inner is not None:
        op.dirichlet_rhs(dev(prob.ub_inner), None, f)
    x = dev(prob.x0)
    st, it, rel, hist = op.solve(f, x, prob.tol, prob.maxit, True)
    torch.cuda.synchronize()
    return st, it, x.cpu().numpy(), op, g, f


@pytest.mark.parametrize("mk", ["viscosity", "conduction", "aniso"])
def test_one_rank_nccl_loop_matches_oracle(mp, oracle_mod, mk):
    prob = {"viscosity": lambda: W.viscosity_problem(24, 16, 64),
            "conduction": lambda: W.conduction_problem(40, 16, 32),
            "aniso": lambda: W.aniso_conduction_problem(24, 16, 64)}[mk]()
    dist = (1, 0, mp.mas_comm_unique_id())
    st, it, x, op, g, f = solve(mp, prob, dist, aniso=(mk == "aniso"))
    assert op.transport == "nccl"
    rc, xo, ito, _, _ = oracle_mod.solve_problem(prob)
    V = oracle_mod.Oracle.for_problem(prob).volumes()
    assert st == mp.MAS_OK and abs(it - ito) <= 1, (it, ito)
    assert rel_l2_V(V, x, xo) <= 1e-10
    # against the single-GPU graph loop on the same problem
    st1, it1, x1, op1, g1, _ = solve(mp, prob, None, aniso=(mk == "aniso"))
    assert abs(it - it1) <= 1 and rel_l2_V(V, x, x1) <= 1e-10
    # mas_op_dot through ncclAllReduce
    a = dev(prob.x0)
    assert abs(op.dot(a, a) - oracle_mod.Oracle.for_problem(prob).dot(prob.x0, prob.x0)) <= \
        1e-13 * oracle_mod.Oracle.for_problem(prob).dot(prob.x0, prob.x0)
    # the exchange-step measurement: no r-neighbour (0 seam bytes), a real allreduce
    seam_us, ar_us, seam_bytes = op.comm_bench(5)
    assert seam_bytes == 0.0 and ar_us > 0.0
    for o in (op, op1):
        o.close()
    g.close()
    g1.close()


def test_one_rank_nccl_comm_with_p2p_mailbox(mp, oracle_mod):
    """P2P transport set up over the 1-rank NCCL communicator (IPC records
    all-gathered through it): the mailbox runs against itself in the graph
    loop and matches the plain single-GPU graph loop bit for bit."""
    prob = W.viscosity_problem(12, 16, 64)
    dist = (1, 0, mp.mas_comm_unique_id())
    st, it, x, op, g, f = solve(mp, prob, dist, p2p=True)
    assert op.transport == "p2p" and st == mp.MAS_OK
    st1, it1, x1, op1, g1, _ = solve(mp, prob, None)
    assert it == it1
    np.testing.assert_array_equal(x, x1)
    op.close()
    op1.close()
    g.close()
    g1.close()
