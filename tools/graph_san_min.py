"""compute-sanitizer driver for the CUDA-graph solve loop (one GPU): C1 (MMS,
scalar), C2-shaped conduction, C3-shaped 3-component viscosity, the
field-aligned conduction term (C2a-shaped), the P2P mailbox on one rank, and
(with --c3full) one full-size C3 solve capped at a few iterations.  Every
solve goes through the graph loop (profiling off, MAS_NO_GRAPH unset) and is
repeated, so the cached graph is relaunched."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_ipps_caplansl23_b200 import maspcg as M  # noqa: E402
from paper_conf_ipps_caplansl23_b200 import workloads as W  # noqa: E402

d = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()


def run(prob, maxit=40, aniso=False, p2p=False, reps=2):
    g = M.Grid(prob.mesh)
    op = M.Operator(g, prob.ncomp, d(prob.kappa), d(prob.c), prob.bc_inner, prob.bc_outer)
    if aniso:
        op.set_aniso(d(prob.kpar), d(prob.bhat))
    if p2p:
        op.enable_p2p()
    f = d(prob.f)
    ubi = None if prob.ub_inner is None else d(prob.ub_inner)
    ubo = None if prob.ub_outer is None else d(prob.ub_outer)
    if ubi is not None or ubo is not None:
        op.dirichlet_rhs(ubi, ubo, f)
    res = []
    for _ in range(reps):
        x = d(prob.x0)
        st, it, rel, _ = op.solve(f, x, 1e-10, maxit)
        res.append((st, it))
    # a solve that converges inside iteration 1's kernels (exact start) and a
    # zero-rhs solve: the while loop must end from its early-exit paths
    x = d(prob.x0)
    res.append(op.solve(torch.zeros_like(f), x, 1e-10, maxit)[:2])
    torch.cuda.synchronize()
    print(prob.name, prob.mesh.shape, "aniso" if aniso else "", "p2p" if p2p else "", res, flush=True)
    op.close()
    g.close()


only = next((a.split("=", 1)[1] for a in sys.argv if a.startswith("--only=")), None)
cases = {
    "c1": lambda: run(W.mms_problem(16, 24, 32), maxit=300),
    "c2a": lambda: run(W.conduction_problem(9, 13, 70)),
    "c2b": lambda: run(W.conduction_problem(40, 24, 130)),
    "c3a": lambda: run(W.viscosity_problem(40, 10, 66)),
    "c3b": lambda: run(W.viscosity_problem(64, 64, 128), maxit=12),
    "aniso": lambda: run(W.aniso_conduction_problem(16, 24, 64), aniso=True),
    "p2p": lambda: run(W.viscosity_problem(12, 16, 64), p2p=True),
}
for name, fn in cases.items():
    if only is None or name in only.split(","):
        fn()
if "--c3full" in sys.argv:
    run(W.viscosity_problem(256, 256, 512), maxit=3, reps=1)
print("done")
