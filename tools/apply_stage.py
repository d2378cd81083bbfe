"""Debug driver: one mas_op_apply of config C2 (isotropic) or C2a (aniso)."""
import sys
import os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
from paper_conf_ipps_caplansl23_b200 import maspcg as M
from paper_conf_ipps_caplansl23_b200 import workloads as W

prob = W.make(sys.argv[1], nr=128, nt=128, np_=256)
d = lambda a: torch.from_numpy(np.array(a)).cuda()
g = M.Grid(prob.mesh)
op = M.Operator(g, 1, d(prob.kappa), d(prob.c), prob.bc_inner, prob.bc_outer)
if prob.kpar is not None:
    op.set_aniso(d(prob.kpar), d(prob.bhat))
x = d(prob.x0); y = torch.empty_like(x)
op.apply(x, y)
torch.cuda.synchronize(); print("apply ok", flush=True)
