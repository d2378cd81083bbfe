"""Small solves for compute-sanitizer (memcheck / racecheck / initcheck):
scalar and 3-component, ragged tiles, one chunk boundary, host-driven loop
and CUDA-graph loop."""
import os
os.environ.setdefault("MAS_TEST_TRANSPORTS", "1")  # virtual ranks (comm.cpp)
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_ipps_caplansl23_b200 import maspcg as M  # noqa: E402
from paper_conf_ipps_caplansl23_b200 import workloads as W  # noqa: E402

d = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
for prob in (W.conduction_problem(9, 13, 70), W.viscosity_problem(40, 10, 66)):
    g = M.Grid(prob.mesh)
    op = M.Operator(g, prob.ncomp, d(prob.kappa), d(prob.c), prob.bc_inner, prob.bc_outer)
    f = d(prob.f)
    if prob.ub_inner is not None:
        op.dirichlet_rhs(d(prob.ub_inner), None, f)
    y = torch.empty_like(f)
    op.apply(d(prob.x0), y)
    x = d(prob.x0)
    st, it, rel, _ = op.solve(f, x, 1e-10, 30)
    op.set_profiling(True)   # host-driven loop
    x = d(prob.x0)
    st2, it2, rel2, _ = op.solve(f, x, 1e-10, 30)
    torch.cuda.synchronize()
    print(prob.name, st, it, st2, it2)
    op.close()
    g.close()

# P2P transport on one rank (mailbox against itself, graph loop), then a 2x2
# (r, theta) decomposition on virtual ranks through both loops
import threading  # noqa: E402

prob = W.viscosity_problem(12, 16, 64)
g = M.Grid(prob.mesh)
op = M.Operator(g, prob.ncomp, d(prob.kappa), d(prob.c), prob.bc_inner, prob.bc_outer)
op.enable_p2p()
x = d(prob.x0)
print("p2p one rank", op.solve(d(prob.f), x, 1e-10, 30)[:2])
op.close()
g.close()

prob = W.conduction_problem(8, 20, 32)
for p2p in (False, True):
    vid = M.virtual_ranks_id(777 + p2p)
    out = {}

    def rank_main(r):
        torch.cuda.set_device(0)
        with torch.cuda.stream(torch.cuda.Stream()):
            gg = M.Grid(prob.mesh, dist=(4, r, vid), ptheta=2)
            sl = (slice(gg.i0, gg.i0 + gg.nl), slice(gg.j0, gg.j0 + gg.ntl))
            oo = M.Operator(gg, 1, d(prob.kappa[sl]), d(prob.c[sl]), prob.bc_inner, prob.bc_outer)
            if p2p:
                oo.enable_p2p()
            f = d(prob.f[(slice(None),) + sl])
            oo.dirichlet_rhs(d(prob.ub_inner[:, sl[1]]), None, f)
            xx = d(prob.x0[(slice(None),) + sl])
            out[r] = oo.solve(f, xx, 1e-10, 30)[:2]
            torch.cuda.synchronize()
            oo.close()
            gg.close()

    th = [threading.Thread(target=rank_main, args=(r,)) for r in range(4)]
    for t in th:
        t.start()
    for t in th:
        t.join()
    print("2x2 virtual ranks p2p" if p2p else "2x2 virtual ranks nccl-placement", out)
