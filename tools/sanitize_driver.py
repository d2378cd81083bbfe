"""Small solves for compute-sanitizer (memcheck / racecheck / initcheck):
scalar and 3-component, ragged tiles, one chunk boundary, host-driven loop
and CUDA-graph loop."""
import os
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
