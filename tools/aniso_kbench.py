"""k_aniso<PCGA> device time at C2a from the kernel replay (mas_op_kernel_bench:
20 graph launches after an L2 flush each); prints one line.  For A/B builds
(diagnostic ones included: no parity check here)."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(sys.argv[0] if sys.argv[0] else __file__)))
sys.path.insert(0, os.getcwd())
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_ipps_caplansl23_b200 import maspcg as M  # noqa: E402
from paper_conf_ipps_caplansl23_b200 import workloads as W  # noqa: E402

d = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
prob = W.aniso_conduction_problem(128, 128, 256)
g = M.Grid(prob.mesh)
op = M.Operator(g, 1, d(prob.kappa), d(prob.c), prob.bc_inner, prob.bc_outer)
op.set_aniso(d(prob.kpar), d(prob.bhat))
res = []
for _ in range(3):
    a, b, c = op.kernel_bench(20)
    res.append(c)
print(sys.argv[1] if len(sys.argv) > 1 else "", "k_aniso us:", " ".join(f"{1e3 * v:.2f}" for v in res))
